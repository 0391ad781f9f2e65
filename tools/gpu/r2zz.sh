# last check at the final commit: the full GPU suite, smoke, the default bench line
set -x
mkdir -p gpurun_out/r2zz
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/r2zz/pytest_gpu.log 2>&1; echo pytest $? >> gpurun_out/r2zz/pytest_gpu.log
timeout 120 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2zz/smoke.log 2>&1
timeout 400 python bench.py > gpurun_out/r2zz/sweep.json 2> gpurun_out/r2zz/sweep.err
timeout 400 python bench.py --workload multi > gpurun_out/r2zz/multi.json 2> gpurun_out/r2zz/multi.err
