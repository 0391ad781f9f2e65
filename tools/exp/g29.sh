#!/bin/bash
set -u
mkdir -p gpurun_out/memcheck
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/g29_build.log 2>&1 || { echo build-failed; exit 1; }
export PYTORCH_NO_CUDA_MEMORY_CACHING=1
timeout 1500 compute-sanitizer --tool memcheck --error-exitcode 9 python -m pytest tests/test_gpu_rowtile.py -x -q > gpurun_out/memcheck/r1g_memcheck_rowtile.log 2>&1
echo "memcheck rc=$?"; tail -3 gpurun_out/memcheck/r1g_memcheck_rowtile.log
timeout 900 compute-sanitizer --tool racecheck --error-exitcode 9 python -m pytest tests/test_gpu_rowtile.py -x -q -k "exact or deterministic" > gpurun_out/memcheck/r1g_racecheck_rowtile.log 2>&1
echo "racecheck rc=$?"; tail -3 gpurun_out/memcheck/r1g_racecheck_rowtile.log
timeout 900 compute-sanitizer --tool synccheck --error-exitcode 9 python -m pytest tests/test_gpu_rowtile.py -x -q -k "exact or deterministic" > gpurun_out/memcheck/r1g_synccheck_rowtile.log 2>&1
echo "synccheck rc=$?"; tail -3 gpurun_out/memcheck/r1g_synccheck_rowtile.log
unset PYTORCH_NO_CUDA_MEMORY_CACHING
i=0
for args in "tmv 513 131072 TMV_REGTILE --params 0,0,0,0,4,1024,20" "tmv 257 262144 TMV_REGTILE --params 0,0,0,0,4,512,44"; do
  i=$((i+1))
  ncu --set full --import-source on --clock-control none -k regex:"mv_" -c 1 -o /tmp/g29_$i -f python tools/run_one.py $args --reps 2 > /dev/null 2>&1
  ncu -i /tmp/g29_$i.ncu-rep --page details --csv > gpurun_out/g29_${i}_details.csv 2>/dev/null
  ncu -i /tmp/g29_$i.ncu-rep --page source --csv --print-source sass > gpurun_out/g29_${i}_sass.csv 2>/dev/null
  ncu -i /tmp/g29_$i.ncu-rep --page raw --csv > gpurun_out/g29_${i}_raw.csv 2>/dev/null
done
echo done
