#!/bin/bash
set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/g36_build.log 2>&1 || { echo build-failed; exit 1; }
timeout 900 python -m pytest tests/test_gpu_mis.py -x -q > gpurun_out/g36_pytest.log 2>&1
echo "pytest rc=$?"; tail -2 gpurun_out/g36_pytest.log
out=gpurun_out/sweep_r1k_shift.jsonl; rm -f $out
for e in 20 21 22 23 24 25 26; do
  timeout 1200 python tools/sweep.py --out $out --elems $e --perturb-only --ops mv --kmin 3 --reps 7 --shift-only >> gpurun_out/g36_sweep.log 2>&1
done
timeout 900 python tools/sweep.py --out $out --elems 26 --kmin 30 --ops mv --extra 12x5592406,96x699051,768x87382,6144x10923,49152x1366 --reps 7 --shift-only >> gpurun_out/g36_sweep.log 2>&1
wc -l $out
