# FINAL evidence of round 2 at the last kernel/planner commit: full GPU tests + smoke, every
# workload's bench line, the oracle arm, ncu launch lists + full captures (default, offgrid).
set -x
mkdir -p gpurun_out/r2z
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r2z/pytest_gpu.log 2>&1; echo pytest $? >> gpurun_out/r2z/pytest_gpu.log
timeout 120 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2z/smoke.log 2>&1
for w in sweep offgrid multi dot rowshard splitk config0 blas1 bicgstab stencil small; do
  timeout 400 python bench.py --workload $w --detail gpurun_out/r2z/$w.detail.jsonl > gpurun_out/r2z/$w.json 2> gpurun_out/r2z/$w.err
done
timeout 300 python bench.py --workload dot --dtype i32 --detail gpurun_out/r2z/dot_i32.detail.jsonl > gpurun_out/r2z/dot_i32.json 2> gpurun_out/r2z/dot_i32.err
timeout 400 python bench.py --impl reference > gpurun_out/r2z/reference.json 2> gpurun_out/r2z/reference.err
timeout 900 bash tools/profile_bench.sh r2z > gpurun_out/r2z/profile_bench.log 2>&1
timeout 900 bash tools/profile_workload.sh offgrid 42 r2z > gpurun_out/r2z/profile_offgrid.log 2>&1
