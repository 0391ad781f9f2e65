# ncu evidence of the offgrid step at the final table (after the last TMV refit)
set -x
timeout 900 bash tools/profile_workload.sh offgrid 42 r2w > gpurun_out/profile_offgrid_r2w.log 2>&1
