mkdir -p gpurun_out
timeout 600 python tools/exp/mv1_tile.py > gpurun_out/g10_mv1.jsonl 2> gpurun_out/g10_mv1.err
timeout 900 python -m pytest -q tests/test_gpu_multi.py > gpurun_out/g10_tests.log 2>&1
tail -n 2 gpurun_out/g10_tests.log
