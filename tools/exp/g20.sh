mkdir -p gpurun_out
timeout 900 python -m pytest -q tests/test_gpu_stencil.py tests/test_gpu_random.py > gpurun_out/g20_tests.log 2>&1
rm -f gpurun_out/sweep_st4.jsonl
timeout 900 python tools/sweep_stencil.py --elems 24,26 --out gpurun_out/sweep_st4.jsonl > gpurun_out/g20_sweep.log 2>&1
tail -n 3 gpurun_out/g20_tests.log
