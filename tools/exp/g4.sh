mkdir -p gpurun_out
timeout 900 python -m pytest -q tests/test_gpu_stencil.py tests/test_gpu_multi.py > gpurun_out/g4_tests.log 2>&1
timeout 600 python tools/exp/multi_cmp.py > gpurun_out/g4_multi_cmp.jsonl 2> gpurun_out/g4_multi_cmp.err
timeout 600 python bench.py --workload stencil > gpurun_out/g4_bench_stencil.json 2> gpurun_out/g4_bench_stencil.err
timeout 600 python bench.py --workload multi > gpurun_out/g4_bench_multi.json 2> gpurun_out/g4_bench_multi.err
timeout 900 bash tools/profile_workload.sh stencil 11 r1c > gpurun_out/g4_prof1.log 2>&1
timeout 900 bash tools/profile_workload.sh multi 8 r1c > gpurun_out/g4_prof2.log 2>&1
tail -n 3 gpurun_out/g4_tests.log
