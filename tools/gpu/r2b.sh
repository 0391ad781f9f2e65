set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/r2b_pytest_gpu.log 2>&1; echo pytest $? >> gpurun_out/r2b_pytest_gpu.log
tail -3 gpurun_out/r2b_pytest_gpu.log
timeout 300 python bench.py > gpurun_out/r2b_sweep.json 2> gpurun_out/r2b_sweep.err
timeout 300 python bench.py --workload offgrid --detail gpurun_out/r2b_offgrid.detail.jsonl > gpurun_out/r2b_offgrid.json 2> gpurun_out/r2b_offgrid.err
timeout 300 python bench.py --workload multi --detail gpurun_out/r2b_multi.detail.jsonl > gpurun_out/r2b_multi.json 2> gpurun_out/r2b_multi.err
timeout 300 python bench.py --workload small --detail gpurun_out/r2b_small.detail.jsonl > gpurun_out/r2b_small.json 2> gpurun_out/r2b_small.err
timeout 120 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2b_smoke.log 2>&1
