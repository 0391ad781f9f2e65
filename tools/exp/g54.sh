#!/bin/bash
set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/g54_build.log 2>&1 || { echo build-failed; exit 1; }
timeout 900 python -m pytest tests/test_gpu_rowtile.py tests/test_gpu_mis.py tests/test_gpu_parity.py -x -q > gpurun_out/g54_pytest.log 2>&1
echo "pytest rc=$?"; tail -1 gpurun_out/g54_pytest.log
for a in "tmv 9 8388608 TMV_REGTILE --params 0,0,0,0,4,512,44" "tmv 9 8388608 TMV_REGTILE --params 0,0,0,0,4,512,0" "tmv 513 131072 TMV_REGTILE --params 0,0,0,0,4,512,20" "tmv 129 524288 AUTO" "mv 262144 257 AUTO" "mv 524288 129 MV_TPR --params 128,0,1,4" "mv 2097152 32 AUTO" "dot 524288 129 AUTO"; do
  echo "$a $(timeout 60 python tools/run_one.py $a --reps 30 2>&1 | tail -1 | cut -c1-50)"
done
f() { python -c "import json,sys; d=json.loads(open(sys.argv[1]).read()); print(sys.argv[1], round(d['value']), round(d['ms_per_step'],3), round(d.get('kernel_sum_ms') or 0,3), d['roofline']['median_frac'], d['clocks']['sm_mhz'])" $1; }
for w in sweep offgrid; do timeout 300 python bench.py --workload $w --steps 100 --warmup 5 --no-e2e --no-cpu-baseline > gpurun_out/g54_$w.json 2>/dev/null; f gpurun_out/g54_$w.json; done
