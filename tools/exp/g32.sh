#!/bin/bash
set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/g32_build.log 2>&1 || { echo build-failed; exit 1; }
f() { python -c "import json,sys; d=json.loads(open(sys.argv[1]).read()); print(sys.argv[1], round(d['value']), round(d['ms_per_step'],3), round(d.get('kernel_sum_ms') or 0,3))" $1; }
for w in sweep offgrid blas1 stencil multi dot; do
  for pdl in 1 0; do
    ADAPTIC_PDL=$pdl timeout 300 python bench.py --workload $w --steps 30 --warmup 5 --no-e2e --no-cpu-baseline > gpurun_out/g32_${w}_pdl$pdl.json 2>/dev/null; f gpurun_out/g32_${w}_pdl$pdl.json
  done
done
