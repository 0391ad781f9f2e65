mkdir -p gpurun_out
rm -f gpurun_out/sweep_b1all.jsonl
timeout 1800 python tools/sweep.py --out gpurun_out/sweep_b1all.jsonl --ops b1all --elems 22,26 \
   --extra 1x1024,1x4096,1x16384,1x65536,1x262144,1x1048576,1x4194304,1x16777216,1x67108864,1x268435456 > gpurun_out/g16_sweep.log 2>&1
timeout 600 python -m pytest -q tests/test_gpu_stencil.py > gpurun_out/g16_tests.log 2>&1
tail -n 2 gpurun_out/g16_sweep.log gpurun_out/g16_tests.log
