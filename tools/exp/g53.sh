#!/bin/bash
set -u
mkdir -p gpurun_out
out=gpurun_out/g53_times.txt; : > $out
for flags in "" "-DTMVMIS_L1=1"; do
  rm -f build/adaptic/k_tmv_mis_f32.o build/adaptic/k_tmv_mis_i32.o
  ADAPTIC_NVCC_EXTRA="$flags" python -c "from paper_conf_pldi_samadihmlm12_b200 import build_ext; build_ext.build()" > /dev/null 2>&1 || echo build-failed
  for a in "tmv 1025 65536 AUTO" "tmv 2049 32768 AUTO" "tmv 65537 1024 AUTO" "tmv 8388609 8 AUTO" "tmv 262145 256 AUTO"; do
    echo "[$flags] $a $(timeout 60 python tools/run_one.py $a --reps 30 2>&1 | tail -1 | cut -c1-50)" >> $out
  done
done
cat $out
