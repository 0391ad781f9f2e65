mkdir -p gpurun_out
timeout 300 compute-sanitizer --tool memcheck python tools/exp/st_dbg.py > gpurun_out/g12_san.log 2>&1
timeout 300 python tools/exp/st_dbg.py > gpurun_out/g12_plain.log 2>&1
tail -n 30 gpurun_out/g12_san.log
