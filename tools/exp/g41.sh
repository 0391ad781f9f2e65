#!/bin/bash
set -u
mkdir -p gpurun_out
out=gpurun_out/g42_times.txt; : > $out
for flags in "" "-DTRT_CPASYNC=1"; do
  rm -f build/adaptic/k_rowtile.o
  ADAPTIC_NVCC_EXTRA="$flags" python -c "from paper_conf_pldi_samadihmlm12_b200 import build_ext; build_ext.build()" > /dev/null 2>&1 || echo build-failed
  for a in "tmv 9 8388608 TMV_REGTILE --params 0,0,0,0,4,512,44" "tmv 9 8388608 TMV_REGTILE --params 0,0,0,0,4,512,0" "tmv 513 131072 TMV_REGTILE --params 0,0,0,0,4,1024,28" "tmv 129 524288 TMV_REGTILE --params 0,0,0,0,4,512,0" "tmv 257 262144 TMV_REGTILE --params 0,0,0,0,4,512,0" "tmv 9 8388608 TMV_REGTILE --params 0,0,0,0,4,256,0"; do
    echo "[$flags] $a $(timeout 60 python tools/run_one.py $a --reps 20 2>&1 | tail -1 | cut -c1-50)" >> $out
  done
done
cat $out
rm -f build/adaptic/k_rowtile.o; ADAPTIC_NVCC_EXTRA="-DTRT_CPASYNC=1" python -c "from paper_conf_pldi_samadihmlm12_b200 import build_ext; build_ext.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_rowtile.py -q -x -k tmv > gpurun_out/g42_pytest.log 2>&1; echo "cpasync pytest rc=$?"; tail -1 gpurun_out/g42_pytest.log
