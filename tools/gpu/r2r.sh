set -x
mkdir -p gpurun_out/r2r
timeout 1800 python tools/sweep.py --out gpurun_out/r2r/sweep_r2_offtmv_full2.jsonl --elems 26 --ops tmv --perturb-only 2> gpurun_out/r2r/sweep.err
