set -x
timeout 900 python -m pytest tests/test_gpu_rowtile.py tests/test_gpu_parity.py -x -q > gpurun_out/r2j_pytest.log 2>&1; echo pytest $? >> gpurun_out/r2j_pytest.log
tail -3 gpurun_out/r2j_pytest.log
timeout 900 python tools/exp/tgroup_cmp.py 9x8388608,17x4194304,33x2097152,65x1048576,129x524288,257x262144,513x131072,1025x65536 > gpurun_out/r2j_cmp.jsonl 2> gpurun_out/r2j_cmp.err
timeout 300 python bench.py --workload offgrid --detail gpurun_out/r2j_offgrid.detail.jsonl > gpurun_out/r2j_offgrid.json 2> gpurun_out/r2j_offgrid.err
