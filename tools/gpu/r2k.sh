# Round-2 final evidence at the last kernel commit: every workload's bench line (N = 1), the
# oracle arm, and ncu launch lists + full captures of the default and offgrid steps.
set -x
mkdir -p gpurun_out/r2k
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv
for w in sweep offgrid multi dot rowshard splitk config0 blas1 bicgstab stencil small; do
  timeout 400 python bench.py --workload $w --detail gpurun_out/r2k/$w.detail.jsonl > gpurun_out/r2k/$w.json 2> gpurun_out/r2k/$w.err
done
timeout 300 python bench.py --workload dot --dtype i32 --detail gpurun_out/r2k/dot_i32.detail.jsonl > gpurun_out/r2k/dot_i32.json 2> gpurun_out/r2k/dot_i32.err
timeout 400 python bench.py --impl reference > gpurun_out/r2k/reference.json 2> gpurun_out/r2k/reference.err
timeout 120 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2k/smoke.log 2>&1
timeout 900 bash tools/profile_bench.sh r2k > gpurun_out/r2k/profile_bench.log 2>&1
timeout 900 bash tools/profile_workload.sh offgrid 42 r2k > gpurun_out/r2k/profile_offgrid.log 2>&1
ls -la gpurun_out
