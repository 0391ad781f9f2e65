mkdir -p gpurun_out
timeout 1500 python -m pytest -q -m gpu tests > gpurun_out/g14_gpu.log 2>&1
rm -f gpurun_out/val_tile.jsonl
timeout 900 python tools/sweep.py --out gpurun_out/val_tile.jsonl --ops mv --elems 22,24,26 --auto-only > /dev/null 2>&1
timeout 900 python tools/sweep.py --out gpurun_out/val_tile.jsonl --ops mv --elems 26 --auto-only --dtype i32 > /dev/null 2>&1
timeout 600 python bench.py > gpurun_out/g14_bench.json 2> gpurun_out/g14_bench.err
timeout 600 python bench.py --workload stencil > gpurun_out/g14_bench_stencil.json 2> gpurun_out/g14_bench_stencil.err
tail -n 3 gpurun_out/g14_gpu.log
