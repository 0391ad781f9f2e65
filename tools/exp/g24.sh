#!/bin/bash
set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/g24_build.log 2>&1 || { echo build-failed; tail -30 gpurun_out/g24_build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_rowtile.py tests/test_gpu_mis.py -x -q > gpurun_out/g24_pytest.log 2>&1
echo "pytest rc=$?"; tail -5 gpurun_out/g24_pytest.log
out=gpurun_out/sweep_r1f_tmvrt.jsonl
rm -f $out
for e in 20 21 22 23 24 25 26; do
  timeout 900 python tools/sweep.py --out $out --elems $e --perturb-only --ops tmv --kmin 3 --kmax 9 --reps 7 --flat-only >> gpurun_out/g24_sweep.log 2>&1
done
timeout 900 python tools/sweep.py --out $out --elems 26 --kmin 30 --ops tmv --extra 14x5162220,98x691870 --reps 7 --flat-only >> gpurun_out/g24_sweep.log 2>&1
wc -l $out
