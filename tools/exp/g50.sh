#!/bin/bash
set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/g50_build.log 2>&1 || { echo build-failed; exit 1; }
out=gpurun_out/sweep_r1o_rowtile_vec.jsonl; rm -f $out
for e in 20 21 22 23 24 25 26; do
  timeout 900 python tools/sweep.py --out $out --elems $e --ops mv,dot --kmin $((e-10)) --reps 7 --rowtile-only >> gpurun_out/g50_sweep.log 2>&1
done
python - <<'PY'
import json,collections
rows=[json.loads(l) for l in open('gpurun_out/sweep_r1o_rowtile_vec.jsonl')]
by=collections.defaultdict(list)
for r in rows: by[(r['op'],r['R'],r['C'])].append(r)
for k,rs in sorted(by.items(), key=lambda t:(t[0][0],t[0][1]*t[0][2],t[0][1])):
    if k[1]*k[2] < (1<<25): continue
    a=[r for r in rs if r['req']=='AUTO'][0]
    f=[r for r in rs if r['req']!='AUTO']
    if not f: continue
    b=max(f, key=lambda r:r['GBps'])
    print(k, 'AUTO', a['variant'], round(a['GBps']), 'best tile', round(b['GBps']), b['params'])
PY
