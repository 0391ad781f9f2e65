# Round-2 final evidence at the last kernel commit: every workload's bench line (N = 1), the
# oracle arm, ncu launch lists + full captures of the default and offgrid steps, and the
# selector's AUTO picks on held-out sets B / Bs with the current table.
set -x
mkdir -p gpurun_out/r2k
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv
timeout 600 python -m pytest tests/test_gpu_mv_tile.py tests/test_gpu_chunk.py -x -q > gpurun_out/r2k/pytest_tile.log 2>&1; echo pytest $? >> gpurun_out/r2k/pytest_tile.log
for w in sweep offgrid multi dot rowshard splitk config0 blas1 bicgstab stencil small; do
  timeout 400 python bench.py --workload $w --detail gpurun_out/r2k/$w.detail.jsonl > gpurun_out/r2k/$w.json 2> gpurun_out/r2k/$w.err
done
timeout 300 python bench.py --workload dot --dtype i32 --detail gpurun_out/r2k/dot_i32.detail.jsonl > gpurun_out/r2k/dot_i32.json 2> gpurun_out/r2k/dot_i32.err
timeout 400 python bench.py --impl reference > gpurun_out/r2k/reference.json 2> gpurun_out/r2k/reference.err
timeout 120 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2k/smoke.log 2>&1
timeout 900 python tools/sweep.py --out gpurun_out/r2k/val_r2_valB3_auto.jsonl --elems 26 --kmin 99 --ops mv,tmv,dot --auto-only --extra 6x27262976,26x6291456,12x6815744,52x1572864,24x6815744,104x1572864,48x1703936,208x393216,96x1703936,416x393216,192x425984,832x98304,384x425984,1664x98304,768x106496,3328x24576,1536x106496,6656x24576,3072x26624,13312x6144,6144x26624,26624x6144,12288x6656,53248x1536,24576x6656,106496x1536,49152x1664,212992x384,98304x1664,425984x384,196608x416,851968x96,393216x416,1703936x96,786432x104,3407872x24,1572864x104,6815744x24,1151813x93,402589x599,8460x20903,40x2789073,17x7176425,23417x10181,105x1673907,2870578x40,507478x488,37x5016695,3085902x61,678999x358,8348x29273,30x8314064,6671x34845,17896x11501,429231x450,2872808x63,13x13644223,156445x1590,31x2540883,147352x1083,190x1399425,5677x29996 2> gpurun_out/r2k/valB3.err
timeout 600 python tools/sweep.py --out gpurun_out/r2k/val_r2_valBs3_auto.jsonl --elems 26 --kmin 99 --ops mv,tmv,dot --auto-only --graph-below 1e12 --extra 6x425984,26x98304,12x851968,52x196608,24x53248,104x12288,48x53248,208x12288,96x106496,416x24576,192x6656,832x1536,384x6656,1664x1536,768x13312,3328x3072,1536x832,6656x192,3072x832,13312x192,6144x1664,26624x384,12288x104,53248x24,24576x104,106496x24,49152x208,212992x48,8256x1964,603392x7,4601x1140,11x292338,41441x137,15581x341,331x6914,15610x299,21x351931,169014x8,5479x2100,418x33170 2> gpurun_out/r2k/valBs3.err
timeout 900 bash tools/profile_bench.sh r2k > gpurun_out/r2k/profile_bench.log 2>&1
timeout 900 bash tools/profile_workload.sh offgrid 42 r2k > gpurun_out/r2k/profile_offgrid.log 2>&1
ls -la gpurun_out
