#!/bin/bash
set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/g38_build.log 2>&1 || { echo build-failed; exit 1; }
for shape in "513 131072" "257 262144" "9 8388608"; do
for p in 0,0,0,0,4,1024,4 0,0,0,0,4,1024,16 0,0,0,0,4,1024,28 0,0,0,0,4,512,44 0,0,0,0,4,512,0 0,0,0,0,4,256,0; do
  echo "== $shape $p $(timeout 60 python tools/run_one.py tmv $shape TMV_REGTILE --params $p --reps 20 2>&1 | tail -1 | cut -c1-60)"
done; done > gpurun_out/g40_times.txt 2>&1
echo done
for a in "mv 262144 257 MV_SUBWARP --params 16,0,0,0,4,256,47" "mv 524288 129 MV_TPR --params 128,0,1,4" "mv 1048576 65 AUTO" "dot 524288 129 AUTO"; do echo "== $a $(timeout 60 python tools/run_one.py $a --reps 20 2>&1 | tail -1 | cut -c1-60)"; done >> gpurun_out/g40_times.txt
