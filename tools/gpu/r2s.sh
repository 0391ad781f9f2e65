set -x
mkdir -p gpurun_out/r2s
timeout 900 python -m pytest tests/test_gpu_rowtile.py tests/test_gpu_tshift.py tests/test_gpu_parity.py tests/test_gpu_mis.py -x -q > gpurun_out/r2s/pytest.log 2>&1; echo pytest $? >> gpurun_out/r2s/pytest.log
timeout 400 python bench.py --workload offgrid --detail gpurun_out/r2s/offgrid.detail.jsonl > gpurun_out/r2s/offgrid.json 2> gpurun_out/r2s/offgrid.err
timeout 400 python bench.py --detail gpurun_out/r2s/sweep.detail.jsonl > gpurun_out/r2s/sweep.json 2> gpurun_out/r2s/sweep.err
