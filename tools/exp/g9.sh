mkdir -p gpurun_out
timeout 900 python -m pytest -q tests/test_gpu_multi.py tests/test_gpu_stencil.py > gpurun_out/g9_tests.log 2>&1
timeout 600 python bench.py --workload multi > gpurun_out/g9_bench_multi.json 2> gpurun_out/g9_bench_multi.err
timeout 900 bash tools/profile_workload.sh multi 8 r1d > gpurun_out/g9_prof.log 2>&1
MULTI_AUTO_ONLY=1 timeout 600 python tools/exp/multi_cmp3.py > gpurun_out/g9_multi_cmp3.jsonl 2> gpurun_out/g9_multi_cmp3.err
tail -n 3 gpurun_out/g9_tests.log
