#!/bin/bash
# rowtile kernel + flat TMV fix: parity, then sweeps of the new candidates on the perturbed shapes
set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/g21_build.log 2>&1 || { echo build-failed; tail -30 gpurun_out/g21_build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_rowtile.py tests/test_gpu_mis.py -x -q > gpurun_out/g21_pytest.log 2>&1
echo "pytest rc=$?"; tail -5 gpurun_out/g21_pytest.log
run() { echo "== $*"; timeout 60 python tools/run_one.py "$@" 2>&1 | tail -1; }
{
run tmv 9 8388608 TMV_REGTILE --params 0,0,0,4 --reps 10
run tmv 129 524288 TMV_REGTILE --params 0,0,0,4 --reps 10
run mv 262144 257 MV_WPR --params 32,0,0,0,4,0,0 --reps 10
run mv 524288 129 MV_SUBWARP --params 8,0,0,0,4,0,0 --reps 10
run mv 131072 513 MV_WPR --params 32,0,0,0,4,0,0 --reps 10
run dot 524288 129 MV_SUBWARP --params 8,0,0,0,4,0,0 --reps 10
run mv 8388608 9 MV_SUBWARP --params 1,0,0,0,4,512,0 --reps 10
} > gpurun_out/g21_times.txt 2>&1
timeout 1200 python tools/sweep.py --out gpurun_out/sweep_r1f_rowtile.jsonl --elems 20,21,22,23,24,25,26 --perturb-only \
    --ops mv,dot --rowtile-only --kmin 11 --reps 7 > gpurun_out/g21_sweep_rt.log 2>&1
echo "sweep rt rc=$?"
timeout 600 python tools/sweep.py --out gpurun_out/sweep_r1f_flat.jsonl --elems 20,21,22,23,24,25,26 --perturb-only \
    --ops tmv --flat-only --kmin 3 --kmax 8 --reps 7 > gpurun_out/g21_sweep_flat.log 2>&1
echo "sweep flat rc=$?"
