#!/bin/bash
# ncu evidence for a non-default bench workload (run under gpurun).  Writes into gpurun_out/:
#   launches_<w>_<tag>.csv      ncu launch list (gpu__time_duration.sum, --clock-control none)
#   full_<w>_<tag>_raw.csv      ncu --set full raw page of the first N kernels of one step
#   detail_<w>_<tag>.jsonl      the bench's per-problem list (same order)
# Usage: tools/profile_workload.sh <workload> <n-kernels-per-step> [tag]
set -u
w=$1; n=$2; tag=${3:-r1}
mkdir -p gpurun_out
python bench.py --workload $w --steps 20 --warmup 3 --streams 1 --no-e2e --no-cpu-baseline \
    --detail gpurun_out/detail_${w}_${tag}.jsonl > gpurun_out/bench_${w}_forprof.json 2>/dev/null
ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"b1_|mv_|mv4_|ring|bicg_|st_direct|st_tile" --csv \
    --log-file gpurun_out/launches_${w}_${tag}.csv \
    python bench.py --workload $w --steps 2 --warmup 3 --streams 1 --no-e2e --no-cpu-baseline > /dev/null 2>&1
ncu --set full --clock-control none -k regex:"b1_|mv_|mv4_|ring|bicg_|st_direct|st_tile" -c $n -o /tmp/full_${w}_${tag} -f \
    python bench.py --workload $w --steps 1 --warmup 3 --streams 1 --no-e2e --no-cpu-baseline > /dev/null 2>&1
ncu -i /tmp/full_${w}_${tag}.ncu-rep --page raw --csv > gpurun_out/full_${w}_${tag}_raw.csv 2>/dev/null
echo "profile $w done"
