set -x
mkdir -p gpurun_out/r2p
timeout 900 python -m pytest tests/test_gpu_tshift.py -x -q > gpurun_out/r2p/pytest.log 2>&1; echo pytest $? >> gpurun_out/r2p/pytest.log
timeout 900 python tools/exp/cand_cmp.py tmv 1025x65536,2049x32768,4097x16384,8193x8192,16385x4096,32769x2048,65537x1024,131073x512 "TMV_SPLITK:32,0,0,8,7" "TMV_SPLITK:16,0,0,8,7" "TMV_SPLITK:64,0,0,8,7" "TMV_SPLITK:32,0,2,8,7" > gpurun_out/r2p/cmp.jsonl 2> gpurun_out/r2p/cmp.err
timeout 400 python bench.py --workload offgrid --detail gpurun_out/r2p/offgrid.detail.jsonl > gpurun_out/r2p/offgrid.json 2> gpurun_out/r2p/offgrid.err
