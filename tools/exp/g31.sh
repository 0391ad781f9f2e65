#!/bin/bash
set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/g31_build.log 2>&1 || { echo build-failed; exit 1; }
B="python bench.py --workload offgrid --steps 20 --warmup 5 --no-e2e --no-cpu-baseline"
f() { python -c "import json,sys; d=json.loads(open(sys.argv[1]).read()); print(sys.argv[1], round(d['value']), round(d['ms_per_step'],3), round(d['kernel_sum_ms'],3))" $1; }
$B --streams 1 > gpurun_out/g31_s1.json 2>/dev/null; f gpurun_out/g31_s1.json
ADAPTIC_PDL=0 $B --streams 1 > gpurun_out/g31_s1_nopdl.json 2>/dev/null; f gpurun_out/g31_s1_nopdl.json
$B --streams 1 --kernel-events-in-timed --detail gpurun_out/g31_detail.jsonl > gpurun_out/g31_s1_inner.json 2>/dev/null; f gpurun_out/g31_s1_inner.json
python bench.py --steps 20 --warmup 5 --no-e2e --no-cpu-baseline --streams 1 > gpurun_out/g31_sweep_s1.json 2>/dev/null; f gpurun_out/g31_sweep_s1.json
