mkdir -p gpurun_out
timeout 900 python -m pytest -q tests/test_gpu_blas1.py > gpurun_out/g19_tests.log 2>&1
timeout 600 python bench.py --workload blas1 > gpurun_out/g19_bench_blas1.json 2> gpurun_out/g19_bench_blas1.err
rm -f gpurun_out/val_b1all.jsonl
timeout 900 python tools/sweep.py --out gpurun_out/val_b1all.jsonl --ops b1all --elems 22,26 --auto-only > /dev/null 2>&1
timeout 1500 bash tools/profile_bench.sh r1e > gpurun_out/g19_prof.log 2>&1
tail -n 2 gpurun_out/g19_tests.log gpurun_out/g19_prof.log
