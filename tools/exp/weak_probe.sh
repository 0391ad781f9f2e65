#!/bin/bash
set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || echo build-failed
run() { echo "== $*"; python tools/run_one.py "$@" 2>&1 | tail -1; }
{
run tmv 9 8388608 AUTO --reps 10
run tmv 9 8388608 TMV_REGTILE --params 0,0,0,4 --reps 10
run tmv 129 524288 AUTO --reps 10
run tmv 513 131072 AUTO --reps 10
run mv 262144 257 AUTO --reps 10
run mv 524288 129 AUTO --reps 10
run mv 131072 513 AUTO --reps 10
run dot 524288 129 AUTO --reps 10
} > gpurun_out/weak_times.txt 2>&1
i=0
for args in "tmv 9 8388608 TMV_REGTILE --params 0,0,0,4" "tmv 9 8388608 AUTO" "mv 262144 257 AUTO" "mv 524288 129 AUTO" "tmv 129 524288 AUTO"; do
  i=$((i+1))
  ncu --set full --clock-control none -k regex:"mv_" -c 1 -o /tmp/weak$i -f python tools/run_one.py $args --reps 2 > /dev/null 2>&1
  ncu -i /tmp/weak$i.ncu-rep --page raw --csv > gpurun_out/weak${i}_raw.csv 2>/dev/null
  ncu -i /tmp/weak$i.ncu-rep --page details --csv > gpurun_out/weak${i}_details.csv 2>/dev/null
done
echo done
