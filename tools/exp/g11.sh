mkdir -p gpurun_out
timeout 600 python -m pytest -q tests/test_gpu_mv_tile.py tests/test_gpu_stencil.py > gpurun_out/g11_tests.log 2>&1
rm -f gpurun_out/sweep_tile.jsonl
timeout 1200 python tools/sweep.py --out gpurun_out/sweep_tile.jsonl --ops mv --elems 20,22,24,26 --tile-only \
    --extra 2048x1048576,16384x32768,32768x32768,65536x32768,65536x65536,131072x32768 > gpurun_out/g11_sweep.log 2>&1
timeout 600 python bench.py --workload stencil > gpurun_out/g11_bench_stencil.json 2> gpurun_out/g11_bench_stencil.err
tail -n 3 gpurun_out/g11_tests.log
