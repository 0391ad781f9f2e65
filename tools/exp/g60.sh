#!/bin/bash
set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke(); print('smoke ok')" > gpurun_out/r1s_smoke.log 2>&1; echo "smoke rc=$?"
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/r1s_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/r1s_pytest_gpu.log
timeout 900 python bench.py > gpurun_out/r1s_bench.json 2> gpurun_out/r1s_bench.err; echo "bench rc=$?"
timeout 900 python bench.py --workload offgrid > gpurun_out/r1s_bench_offgrid.json 2>> gpurun_out/r1s_bench.err; echo "offgrid rc=$?"
for f in r1s_bench r1s_bench_offgrid; do python -c "import json,sys; d=json.loads(open(sys.argv[1]).read()); print(sys.argv[1], round(d['value']), d['roofline']['frac'], d['roofline']['median_frac'], d['roofline']['min_frac'], d['e2e']['value'], d['clocks'])" gpurun_out/$f.json; done
