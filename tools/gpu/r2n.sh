set -x
mkdir -p gpurun_out/r2n
timeout 900 python -m pytest tests/test_gpu_rowtile.py tests/test_gpu_parity.py -x -q > gpurun_out/r2n/pytest.log 2>&1; echo pytest $? >> gpurun_out/r2n/pytest.log
timeout 1800 python tools/sweep.py --out gpurun_out/r2n/sweep_r2_offtmv_full.jsonl --elems 26 --ops tmv --perturb-only 2> gpurun_out/r2n/sweep.err
tail -2 gpurun_out/r2n/sweep.err
