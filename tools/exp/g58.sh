#!/bin/bash
# same-run full candidate grid on the off-grid shapes with the final kernels (data for the next refit)
set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/g58_build.log 2>&1 || { echo build-failed; exit 1; }
out=gpurun_out/sweep_r1s_offgrid_full.jsonl; rm -f $out
for e in 20 21 22 23 24 25 26; do
  timeout 900 python tools/sweep.py --out $out --elems $e --perturb-only --ops mv,dot --kmin $((e-9)) --reps 7 >> gpurun_out/g58_sweep.log 2>&1
  timeout 900 python tools/sweep.py --out $out --elems $e --perturb-only --ops tmv --kmin 3 --kmax 9 --reps 7 >> gpurun_out/g58_sweep.log 2>&1
done
timeout 900 python tools/sweep.py --out $out --elems 26 --kmin 30 --ops mv,dot --extra 393216x171,3145728x22 --reps 7 >> gpurun_out/g58_sweep.log 2>&1
timeout 900 python tools/sweep.py --out $out --elems 26 --kmin 30 --ops tmv --extra 14x5162220,98x691870 --reps 7 >> gpurun_out/g58_sweep.log 2>&1
gzip -f $out; ls -la $out.gz
