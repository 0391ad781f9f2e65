#!/bin/bash
# Profile the bench step on one GPU (run under gpurun).  Writes into gpurun_out/:
#   launches.csv        ncu launch list (gpu__time_duration.sum per kernel; cold, serialised)
#   bench_full.ncu-rep  ncu --set full of the 42 kernels of one step (warm-up step 1)
#   detail_prof.jsonl   the bench's per-problem plan/variant list (same order as the captures)
# Usage: tools/profile_bench.sh [round-tag]
set -u
tag=${1:-r1}
mkdir -p gpurun_out
python bench.py --steps 20 --warmup 3 --no-e2e --no-cpu-baseline --detail gpurun_out/detail_prof.jsonl \
    > gpurun_out/bench_forprof.json 2> gpurun_out/bench_forprof.err
ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"mv_|tmv_|mv4_|ring" --csv \
    --log-file gpurun_out/launches_${tag}.csv \
    python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
# the full report of 42 kernels exceeds gpurun's 64 MiB copy-back: keep it in /tmp, bring back
# the raw-page CSV (all metrics, one row per kernel) and the source page of the first kernel
ncu --set full --clock-control none --import-source on -k regex:"mv_|tmv_|mv4_|ring" -c 42 \
    -o /tmp/bench_full_${tag} -f \
    python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_full_${tag}.log 2>&1
ncu -i /tmp/bench_full_${tag}.ncu-rep --page raw --csv > gpurun_out/bench_full_${tag}_raw.csv 2>/dev/null
ncu -i /tmp/bench_full_${tag}.ncu-rep --page details --csv > gpurun_out/bench_full_${tag}_details.csv 2>/dev/null
ls -la /tmp/bench_full_${tag}.ncu-rep
echo "profile done"
