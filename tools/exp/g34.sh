#!/bin/bash
# round evidence after the staged row tiles / PDL change
set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke(); print('smoke ok')" > gpurun_out/r1i_smoke.log 2>&1; echo "smoke rc=$?"
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/r1i_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/r1i_pytest_gpu.log
timeout 900 python bench.py > gpurun_out/r1i_bench.json 2> gpurun_out/r1i_bench.err; echo "bench rc=$?"
timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/r1i_bench_reference.json 2>> gpurun_out/r1i_bench.err; echo "ref rc=$?"
timeout 900 python bench.py --workload offgrid > gpurun_out/r1i_bench_offgrid.json 2>> gpurun_out/r1i_bench.err; echo "offgrid rc=$?"
timeout 900 python bench.py --workload offgrid --impl reference --steps 3 --warmup 3 > gpurun_out/r1i_bench_offgrid_reference.json 2>> gpurun_out/r1i_bench.err
bash tools/profile_bench.sh r1i > gpurun_out/r1i_prof.log 2>&1; echo "prof rc=$?"
bash tools/profile_workload.sh offgrid 42 r1i > gpurun_out/r1i_prof2.log 2>&1; echo "prof2 rc=$?"
for f in r1i_bench r1i_bench_offgrid; do python -c "import json,sys; d=json.loads(open(sys.argv[1]).read()); print(sys.argv[1], round(d['value']), d['roofline']['frac'], d['e2e']['value'], d['clocks'])" gpurun_out/$f.json; done
