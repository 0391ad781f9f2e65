#!/bin/bash
# funnel TMV kernel with the interior fast path: full candidate grid on the R+1 shapes
set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/g27_build.log 2>&1 || { echo build-failed; tail -30 gpurun_out/g27_build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_mis.py tests/test_gpu_random.py -x -q > gpurun_out/g27_pytest.log 2>&1
echo "pytest rc=$?"; tail -2 gpurun_out/g27_pytest.log
out=gpurun_out/sweep_r1g_tmvmis.jsonl
rm -f $out
for e in 20 21 22 23 24 25 26; do
  timeout 1200 python tools/sweep.py --out $out --elems $e --perturb-only --ops tmv --kmin 10 --reps 7 >> gpurun_out/g27_sweep.log 2>&1
done
timeout 900 python tools/sweep.py --out $out --elems 26 --kmin 30 --ops tmv --extra 393217x170,3145729x21,49153x1365,6145x10922 --reps 7 >> gpurun_out/g27_sweep.log 2>&1
wc -l $out
