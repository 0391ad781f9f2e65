mkdir -p gpurun_out
export PYTORCH_NO_CUDA_MEMORY_CACHING=1
timeout 2400 compute-sanitizer --tool memcheck --leak-check no --print-limit 20 \
  python -m pytest -q -m gpu tests -k "not 256MiB and not large_grid and not paper_sizes and not config1 and not config2 and not config3 and not config4 and not single_vector_lengths and not device_generator" \
  > gpurun_out/g15_memcheck.log 2>&1
tail -n 5 gpurun_out/g15_memcheck.log
