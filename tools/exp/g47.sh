#!/bin/bash
set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/g48_build.log 2>&1 || { echo build-failed; exit 1; }
f() { python -c "import json,sys; d=json.loads(open(sys.argv[1]).read()); print(sys.argv[1], round(d['value']), round(d['ms_per_step'],3), round(d.get('kernel_sum_ms') or 0,3), d['clocks']['sm_mhz'])" $1; }
for rep in 1 2; do
for kb in 1 0; do
  for w in sweep offgrid; do
    ADAPTIC_EXCLUSIVE=$kb timeout 300 python bench.py --workload $w --steps 100 --warmup 5 --no-e2e --no-cpu-baseline > gpurun_out/g48_${w}_${kb}_$rep.json 2>/dev/null; f gpurun_out/g48_${w}_${kb}_$rep.json
  done
done; done
