set -x
timeout 600 python -m pytest tests/test_gpu_chunk.py -x -q > gpurun_out/r2h_pytest_chunk.log 2>&1; echo pytest $? >> gpurun_out/r2h_pytest_chunk.log
timeout 1500 python tools/sweep.py --out gpurun_out/sweep_r2_offmv_full.jsonl --elems 26 --ops mv --perturb-only 2> gpurun_out/sweep_offmv.err
timeout 600 python tools/sweep.py --out gpurun_out/sweep_r2_chunk_A.jsonl --elems 26 --kmin 99 --ops mv --chunk-only --extra 391x397085,11047x16191,92x2754178,9808x18131,26x8071465,708x239445,7650x34307,701x210869,22294x10607,437x289085,72x3536510 2> gpurun_out/sweep_chunkA.err
timeout 600 python tools/sweep.py --out gpurun_out/val_r2_chunk_B.jsonl --elems 26 --kmin 99 --ops mv --chunk-only --extra 8460x20903,40x2789073,17x7176425,23417x10181,105x1673907,37x5016695,8348x29273,6671x34845,17896x11501,13x13644223,31x2540883,190x1399425 2> gpurun_out/sweep_chunkB.err
tail -2 gpurun_out/*.err
