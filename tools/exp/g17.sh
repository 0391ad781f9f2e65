mkdir -p gpurun_out
export PYTORCH_NO_CUDA_MEMORY_CACHING=1
K="not 256MiB and not large_grid and not paper_sizes and not config1 and not config2 and not config3 and not config4 and not single_vector_lengths and not device_generator"
for f in mis multi mv_tile stencil parity blas1 bicgstab; do
  timeout 1500 compute-sanitizer --tool memcheck --leak-check no --print-limit 10 \
    python -m pytest -q -m gpu tests/test_gpu_$f.py -k "$K" > gpurun_out/g17_memcheck_$f.log 2>&1
  echo "$f: $(grep -c 'Invalid' gpurun_out/g17_memcheck_$f.log) invalid; $(tail -n 1 gpurun_out/g17_memcheck_$f.log)" >> gpurun_out/g17_summary.txt
done
cat gpurun_out/g17_summary.txt
