mkdir -p gpurun_out
timeout 600 python -m pytest -q tests/test_gpu_stencil.py > gpurun_out/g2_stencil.log 2>&1
timeout 600 python bench.py --workload stencil > gpurun_out/g2_bench_stencil.json 2> gpurun_out/g2_bench_stencil.err
timeout 900 python tools/sweep_stencil.py --out gpurun_out/sweep_st.jsonl > gpurun_out/g2_sweep.log 2>&1
timeout 900 bash tools/profile_workload.sh stencil 11 r1 > gpurun_out/g2_prof.log 2>&1
tail -n 3 gpurun_out/g2_stencil.log
