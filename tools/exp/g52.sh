#!/bin/bash
set -u
mkdir -p gpurun_out/memcheck
python -c "import __graft_entry__ as g; g.build(); g.smoke(); print('smoke ok')" > gpurun_out/r1p_smoke.log 2>&1; echo "smoke rc=$?"
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/r1p_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/r1p_pytest_gpu.log
export PYTORCH_NO_CUDA_MEMORY_CACHING=1
timeout 1800 compute-sanitizer --tool memcheck --error-exitcode 9 python -m pytest tests/test_gpu_mis.py -x -q > gpurun_out/memcheck/r1p_memcheck_mis.log 2>&1; echo "memcheck mis rc=$?"; tail -2 gpurun_out/memcheck/r1p_memcheck_mis.log
timeout 1800 compute-sanitizer --tool memcheck --error-exitcode 9 python -m pytest tests/test_gpu_rowtile.py -x -q > gpurun_out/memcheck/r1p_memcheck_rowtile.log 2>&1; echo "memcheck rowtile rc=$?"; tail -2 gpurun_out/memcheck/r1p_memcheck_rowtile.log
timeout 900 compute-sanitizer --tool racecheck --error-exitcode 9 python -m pytest tests/test_gpu_rowtile.py -x -q -k "tmv_rowtile_exact or deterministic" > gpurun_out/memcheck/r1p_racecheck_rowtile.log 2>&1; echo "racecheck rc=$?"; tail -2 gpurun_out/memcheck/r1p_racecheck_rowtile.log
