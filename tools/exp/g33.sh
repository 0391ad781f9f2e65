#!/bin/bash
set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/g33_build.log 2>&1 || { echo build-failed; exit 1; }
f() { python -c "import json,sys; d=json.loads(open(sys.argv[1]).read()); print(sys.argv[1], round(d['value']), round(d['ms_per_step'],3), round(d.get('kernel_sum_ms') or 0,3))" $1; }
for w in sweep offgrid; do
  for st in 1 2 3; do
    timeout 300 python bench.py --workload $w --steps 30 --warmup 5 --no-e2e --no-cpu-baseline --streams $st > gpurun_out/g33_${w}_s$st.json 2>/dev/null; f gpurun_out/g33_${w}_s$st.json
  done
done
timeout 600 python -m pytest tests -m gpu -q -x -k "batch or stream" > gpurun_out/g33_pytest.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/g33_pytest.log
