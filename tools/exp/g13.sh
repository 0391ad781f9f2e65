mkdir -p gpurun_out
timeout 300 python -m pytest -q -x tests/test_gpu_stencil.py > gpurun_out/g13_st_alone.log 2>&1
CUDA_LAUNCH_BLOCKING=1 timeout 600 python -m pytest -q tests/test_gpu_mv_tile.py tests/test_gpu_stencil.py > gpurun_out/g13_both_blocking.log 2>&1
tail -n 3 gpurun_out/g13_st_alone.log gpurun_out/g13_both_blocking.log
