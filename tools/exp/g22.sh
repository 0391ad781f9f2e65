#!/bin/bash
set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/g22_build.log 2>&1 || { echo build-failed; exit 1; }
i=0
for args in "tmv 9 8388608 TMV_REGTILE --params 0,0,0,2" "tmv 129 524288 TMV_REGTILE --params 0,0,0,2" "mv 262144 257 MV_SUBWARP --params 16,0,0,0,4,256,47" "mv 8388608 9 MV_SUBWARP --params 1,0,0,0,4,256,1365"; do
  i=$((i+1))
  ncu --set full --import-source on --clock-control none -k regex:"mv_" -c 1 -o /tmp/g22_$i -f python tools/run_one.py $args --reps 2 > /dev/null 2>&1
  ncu -i /tmp/g22_$i.ncu-rep --page raw --csv > gpurun_out/g22_${i}_raw.csv 2>/dev/null
  ncu -i /tmp/g22_$i.ncu-rep --page details --csv > gpurun_out/g22_${i}_details.csv 2>/dev/null
  ncu -i /tmp/g22_$i.ncu-rep --page source --csv --print-source sass > gpurun_out/g22_${i}_sass.csv 2>/dev/null
done
echo done
