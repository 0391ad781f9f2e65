mkdir -p gpurun_out
timeout 1500 python -m pytest -q -m gpu tests > gpurun_out/g18_gpu.log 2>&1
export PYTORCH_NO_CUDA_MEMORY_CACHING=1
K="not 256MiB and not large_grid and not paper_sizes and not config1 and not config2 and not config3 and not config4 and not single_vector_lengths and not device_generator"
timeout 1500 compute-sanitizer --tool memcheck --leak-check no --print-limit 10 \
    python -m pytest -q -m gpu tests/test_gpu_parity.py -k "$K" > gpurun_out/g18_memcheck_parity.log 2>&1
unset PYTORCH_NO_CUDA_MEMORY_CACHING
rm -f gpurun_out/sweep_b1all.jsonl
timeout 1800 python tools/sweep.py --out gpurun_out/sweep_b1all.jsonl --ops b1all --elems 22,26 \
   --extra 1x1024,1x4096,1x16384,1x65536,1x262144,1x1048576,1x4194304,1x16777216,1x67108864,1x268435456 > gpurun_out/g18_sweep.log 2>&1
timeout 600 python bench.py --workload config0 > gpurun_out/g18_bench_config0.json 2> gpurun_out/g18_bench_config0.err
tail -n 2 gpurun_out/g18_gpu.log gpurun_out/g18_memcheck_parity.log gpurun_out/g18_sweep.log
