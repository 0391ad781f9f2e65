set -x
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/r2i_pytest_gpu.log 2>&1; echo pytest $? >> gpurun_out/r2i_pytest_gpu.log
tail -3 gpurun_out/r2i_pytest_gpu.log
timeout 300 python bench.py --workload offgrid --detail gpurun_out/r2i_offgrid.detail.jsonl > gpurun_out/r2i_offgrid.json 2> gpurun_out/r2i_offgrid.err
timeout 300 python bench.py --detail gpurun_out/r2i_sweep.detail.jsonl > gpurun_out/r2i_sweep.json 2> gpurun_out/r2i_sweep.err
timeout 120 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2i_smoke.log 2>&1
