mkdir -p gpurun_out
timeout 900 python -m pytest -q tests/test_gpu_multi.py tests/test_gpu_blas1.py > gpurun_out/g6_tests.log 2>&1
timeout 600 python tools/exp/multi_cmp3.py > gpurun_out/g6_multi_cmp3.jsonl 2> gpurun_out/g6_multi_cmp3.err
timeout 600 python bench.py --workload multi > gpurun_out/g6_bench_multi.json 2> gpurun_out/g6_bench_multi.err
timeout 600 python bench.py --workload blas1 > gpurun_out/g6_bench_blas1.json 2> gpurun_out/g6_bench_blas1.err
tail -n 3 gpurun_out/g6_tests.log
