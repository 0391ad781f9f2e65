set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/g1_smi.txt
cat MEASURED_PEAKS.json > gpurun_out/g1_peaks.json 2>/dev/null
timeout 900 python -m pytest tests -q -m gpu -x tests/test_gpu_stencil.py > gpurun_out/g1_stencil.log 2>&1
timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/g1_gpu.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/g1_smoke.log 2>&1
timeout 600 python bench.py > gpurun_out/g1_bench.json 2> gpurun_out/g1_bench.err
tail -3 gpurun_out/g1_gpu.log gpurun_out/g1_stencil.log
