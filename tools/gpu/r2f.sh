set -x
timeout 600 python -m pytest tests/test_gpu_chunk.py -x -q > gpurun_out/r2g_pytest_chunk.log 2>&1; echo pytest $? >> gpurun_out/r2g_pytest_chunk.log
tail -5 gpurun_out/r2g_pytest_chunk.log
timeout 900 python tools/exp/chunk_cmp.py 16x4194305,32x2097153,64x1048577,128x524289,256x262145,512x131073,1024x65537,2048x32769,4096x16385 > gpurun_out/r2g_chunk_cmp.jsonl 2> gpurun_out/r2g_chunk_cmp.err
tail -3 gpurun_out/r2g_chunk_cmp.err
