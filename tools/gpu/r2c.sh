set -x
timeout 600 python -m pytest tests/test_gpu_tgroup.py -x -q > gpurun_out/r2e_pytest_tgroup.log 2>&1; echo pytest $? >> gpurun_out/r2e_pytest_tgroup.log
tail -5 gpurun_out/r2e_pytest_tgroup.log
timeout 900 python tools/exp/tgroup_cmp.py 9x8388608,33x2097152,129x524288,257x262144,513x131072,1025x65536,2049x32768 > gpurun_out/r2e_tgroup_cmp.jsonl 2> gpurun_out/r2e_tgroup_cmp.err
tail -3 gpurun_out/r2e_tgroup_cmp.err
