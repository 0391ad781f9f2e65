mkdir -p gpurun_out
timeout 900 python -m pytest -q tests/test_gpu_multi.py tests/test_gpu_stencil.py > gpurun_out/g8_tests.log 2>&1
timeout 900 python tools/exp/multi_cmp3.py > gpurun_out/g8_multi_cmp3.jsonl 2> gpurun_out/g8_multi_cmp3.err
timeout 600 python bench.py --workload multi > gpurun_out/g8_bench_multi.json 2> gpurun_out/g8_bench_multi.err
rm -f gpurun_out/sweep_st3.jsonl
timeout 900 python tools/sweep_stencil.py --elems 24,26 --out gpurun_out/sweep_st3.jsonl > gpurun_out/g8_sweep.log 2>&1
tail -n 3 gpurun_out/g8_tests.log
