mkdir -p gpurun_out
timeout 900 python -m pytest -q tests/test_gpu_stencil.py tests/test_gpu_multi.py > gpurun_out/g3_tests.log 2>&1
timeout 600 python tools/exp/multi_cmp.py > gpurun_out/g3_multi_cmp.jsonl 2> gpurun_out/g3_multi_cmp.err
rm -f gpurun_out/sweep_st2.jsonl
timeout 900 python tools/sweep_stencil.py --out gpurun_out/sweep_st2.jsonl > gpurun_out/g3_sweep.log 2>&1
timeout 600 python bench.py --workload stencil > gpurun_out/g3_bench_stencil.json 2> gpurun_out/g3_bench_stencil.err
timeout 600 python bench.py --workload multi > gpurun_out/g3_bench_multi.json 2> gpurun_out/g3_bench_multi.err
tail -n 3 gpurun_out/g3_tests.log
