#!/bin/bash
set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/g35_build.log 2>&1 || { echo build-failed; exit 1; }
timeout 900 python -m pytest tests/test_gpu_mis.py tests/test_gpu_random.py tests/test_gpu_parity.py -x -q > gpurun_out/g35_pytest.log 2>&1
echo "pytest rc=$?"; tail -2 gpurun_out/g35_pytest.log
f() { python -c "import json,sys; d=json.loads(open(sys.argv[1]).read()); print(sys.argv[1], round(d['value']), round(d['ms_per_step'],3), round(d.get('kernel_sum_ms') or 0,3), d['roofline']['median_frac'])" $1; }
timeout 300 python bench.py --workload offgrid --steps 30 --warmup 5 --no-e2e --no-cpu-baseline --detail gpurun_out/g35_detail.jsonl > gpurun_out/g35_offgrid.json 2>/dev/null; f gpurun_out/g35_offgrid.json
out=gpurun_out/sweep_r1j_mvmis.jsonl; rm -f $out
for e in 20 22 24 26; do
  timeout 1200 python tools/sweep.py --out $out --elems $e --perturb-only --ops mv --kmin 3 --kmax $((e-10)) --reps 7 >> gpurun_out/g35_sweep.log 2>&1
done
wc -l $out
