set -x
mkdir -p gpurun_out/r2q
timeout 900 python -m pytest tests/test_gpu_tshift.py tests/test_gpu_parity.py -x -q > gpurun_out/r2q/pytest.log 2>&1; echo pytest $? >> gpurun_out/r2q/pytest.log
timeout 400 python bench.py --workload offgrid --detail gpurun_out/r2q/offgrid.detail.jsonl > gpurun_out/r2q/offgrid.json 2> gpurun_out/r2q/offgrid.err
timeout 400 python bench.py --detail gpurun_out/r2q/sweep.detail.jsonl > gpurun_out/r2q/sweep.json 2> gpurun_out/r2q/sweep.err
timeout 400 python bench.py --workload multi --detail gpurun_out/r2q/multi.detail.jsonl > gpurun_out/r2q/multi.json 2> gpurun_out/r2q/multi.err
