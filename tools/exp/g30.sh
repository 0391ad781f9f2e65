#!/bin/bash
set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/g30_build.log 2>&1 || { echo build-failed; exit 1; }
timeout 600 python -m pytest tests/test_gpu_rowtile.py -x -q > gpurun_out/g30_pytest.log 2>&1
echo "pytest rc=$?"; tail -1 gpurun_out/g30_pytest.log
out=gpurun_out/sweep_r1h_tmvrt.jsonl; rm -f $out
for e in 24 25 26; do
  timeout 900 python tools/sweep.py --out $out --elems $e --perturb-only --ops tmv --kmin 3 --kmax 9 --reps 7 --rowtile-only >> gpurun_out/g30_sweep.log 2>&1
done
timeout 900 python bench.py --workload offgrid --steps 50 --warmup 5 > gpurun_out/r1h_bench_offgrid.json 2> gpurun_out/g30_bench.err
echo "bench rc=$?"; cut -c1-300 gpurun_out/r1h_bench_offgrid.json
timeout 600 python bench.py --workload offgrid --impl reference --steps 3 --warmup 3 > gpurun_out/r1h_bench_offgrid_reference.json 2>> gpurun_out/g30_bench.err
echo "ref rc=$?"
bash tools/profile_workload.sh offgrid 42 r1h > gpurun_out/g30_prof.log 2>&1
echo "prof rc=$?"; ls gpurun_out | grep r1h
