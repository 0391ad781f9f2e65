#!/bin/bash
set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/g46_build.log 2>&1 || { echo build-failed; exit 1; }
timeout 900 python -m pytest tests/test_gpu_rowtile.py -x -q > gpurun_out/g46_pytest.log 2>&1
echo "pytest rc=$?"; tail -2 gpurun_out/g46_pytest.log
out=gpurun_out/sweep_r1n_tmvrt4.jsonl; rm -f $out
for e in 20 21 22 23 24 25 26; do
  timeout 900 python tools/sweep.py --out $out --elems $e --perturb-only --ops tmv --kmin 10 --kmax 11 --reps 7 --rowtile-only >> gpurun_out/g46_sweep.log 2>&1
done
python - <<'PY'
import json,collections
rows=[json.loads(l) for l in open('gpurun_out/sweep_r1n_tmvrt4.jsonl')]
by=collections.defaultdict(list)
for r in rows: by[(r['R'],r['C'])].append(r)
for k,rs in sorted(by.items(), key=lambda t:(t[0][0]*t[0][1],t[0][0])):
    a=[r for r in rs if r['req']=='AUTO'][0]
    b=max((r for r in rs if r['req']!='AUTO'), key=lambda r:r['GBps'])
    print(k, 'AUTO', a['variant'], round(a['GBps']), 'best tile', round(b['GBps']), b['params'])
PY
