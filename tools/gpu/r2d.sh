set -x
for cfg in "129 524288 TMV_SPLITK --params 0,0,0,0,12,512,1,0,0" "129 524288 TMV_SPLITK --params 0,0,0,0,12,1024,1,0,0" "129 524288 AUTO" "513 131072 TMV_SPLITK --params 0,0,0,0,12,288,2,0,0" "513 131072 AUTO"; do
  python tools/run_one.py tmv $cfg --reps 10 >> gpurun_out/r2d_runone.txt 2>&1
done
ncu --set full --clock-control none -k regex:"tmv_" -c 5 -o /tmp/r2d_full -f python tools/run_one.py tmv 129 524288 TMV_SPLITK --params 0,0,0,0,12,512,1,0,0 --reps 1 > /dev/null 2>&1
ncu -i /tmp/r2d_full.ncu-rep --page raw --csv > gpurun_out/r2d_full_raw.csv 2>/dev/null
ncu -i /tmp/r2d_full.ncu-rep --page details --csv > gpurun_out/r2d_full_details.csv 2>/dev/null
ncu --set full --clock-control none -k regex:"tmv_" -c 5 -o /tmp/r2d_full2 -f python tools/run_one.py tmv 129 524288 AUTO --reps 1 > /dev/null 2>&1
ncu -i /tmp/r2d_full2.ncu-rep --page details --csv > gpurun_out/r2d_full2_details.csv 2>/dev/null
