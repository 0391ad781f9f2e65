mkdir -p gpurun_out
timeout 1500 python -m pytest -q -m gpu tests > gpurun_out/g5_gpu.log 2>&1
timeout 600 python bench.py --workload blas1 > gpurun_out/g5_bench_blas1.json 2> gpurun_out/g5_bench_blas1.err
timeout 600 python bench.py > gpurun_out/g5_bench.json 2> gpurun_out/g5_bench.err
timeout 600 python tools/exp/multi_cmp2.py > gpurun_out/g5_multi_cmp2.jsonl 2> gpurun_out/g5_multi_cmp2.err
tail -n 3 gpurun_out/g5_gpu.log
