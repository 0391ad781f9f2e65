mkdir -p gpurun_out
timeout 900 python -m pytest -q tests/test_gpu_multi.py > gpurun_out/g7_tests.log 2>&1
timeout 900 python tools/exp/multi_cmp3.py > gpurun_out/g7_multi_cmp3.jsonl 2> gpurun_out/g7_multi_cmp3.err
timeout 600 python bench.py --workload multi > gpurun_out/g7_bench_multi.json 2> gpurun_out/g7_bench_multi.err
tail -n 3 gpurun_out/g7_tests.log
