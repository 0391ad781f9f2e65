set -x
mkdir -p gpurun_out/r2v
timeout 900 python -m pytest tests/test_gpu_multi.py -x -q > gpurun_out/r2v/pytest.log 2>&1; echo pytest $? >> gpurun_out/r2v/pytest.log
timeout 400 python bench.py --workload multi --detail gpurun_out/r2v/multi.detail.jsonl > gpurun_out/r2v/multi.json 2> gpurun_out/r2v/multi.err
