#!/bin/sh
# Round-2 selector refit (reproducible): round 1's fit input (tools/merge_sweeps.py, exactly
# the merge that produced the round-1 table -- checked: identical entries), plus
#   sweep_r2_trainA   held-out set A (tools/heldout_shapes.py A), measured against the round-1
#                     table (101 / 186 gated shapes passing) and then used for TRAINING
#   sweep_r2_dotA     set A's DOT shapes re-swept with b 256-byte aligned (the first sweep put b
#                     right after a: misaligned DOT rows fell back to scalar loads)
#   sweep_r2_small    the 4-64 MiB diagonals, AUTO and every candidate in one run
#   sweep_r2_tshift_* the constant-shift TMV kernel on the R+1 shapes and set A's R % 4 != 0 shapes
#   sweep_r2_misx_*   the misaligned-MV x-funnel / residue-class kernels on the C+1 shapes and set A
#   sweep_r2_rtc_*    the long-row staged MV kernel (MV_CPR, XSMEM 11) on the C+1 shapes and set A
#   sweep_r2_dot1     Sdot N = 1, L = 2^10 .. 2^24 (graph-timed, like sweep_r2_small)
#   sweep_r2_trainAs  small training shapes (tools/heldout_shapes.py As, 4-64 MiB, graph-timed)
#   sweep_r2_offmv_full  the offgrid bench's 21 MV C + 1 shapes, EVERY candidate (incl. the
#                     column-chunk staged kernel, XSMEM 13) in one run: replaces all earlier runs
#   sweep_r2_chunk_A  the column-chunk candidates on set A's misaligned long-row MV shapes
#   sweep_r2_offtmv_full  the offgrid bench's 21 TMV R + 1 shapes, every candidate (incl. 544-thread
#                     staged tiles) in one run: replaces all earlier runs of those shapes
#   sweep_r2_offtmv_full2 the same shapes re-swept after the constant-shift TMV change (2 accumulators,
#                     3 CTAs below R = 4096) and the 544-thread CTA count rule: replaces _full's runs
# DOT cells with rows of 64..1023 values (>= 256 MiB) prefer a staged row-tile candidate within 3 %.
# Set B (tools/heldout_shapes.py B / Bs) is NEVER fitted: profiles/val_r2_* only.
# Fit: bench.py's own shapes protected (pick within 1 % of the best on each), adjacent cells'
# shapes scoring with weight 0.5 (generalisation), tie -> fewer CTAs.
set -e
OUT=${1:-/tmp/r2_all.jsonl}
P=profiles
python tools/merge_sweeps.py "$OUT" \
  $P/sweep_r1_main_fit.jsonl.gz $P/sweep_r1_mv_tile.jsonl.gz +$P/sweep_r1f_offgrid.jsonl.gz \
  $P/sweep_r1f_tmvrt.jsonl.gz +$P/sweep_r1g_tmvmis.jsonl.gz $P/sweep_r1k_shift_restricted.jsonl.gz \
  $P/sweep_r1o_rowtile_vec_restricted.jsonl.gz $P/sweep_r1l_tmvrt.jsonl.gz +$P/sweep_r1s_offgrid_full.jsonl.gz \
  +$P/sweep_r2_trainA.jsonl.gz +$P/sweep_r2_dotA.jsonl.gz +$P/sweep_r2_small.jsonl.gz +$P/sweep_r2_trainAs.jsonl.gz \
  $P/sweep_r2_tshift_fit.jsonl.gz $P/sweep_r2_tshift_A.jsonl.gz $P/sweep_r2_misx_fit.jsonl.gz $P/sweep_r2_misx_A.jsonl.gz $P/sweep_r2_rtc_fit.jsonl.gz $P/sweep_r2_rtc_A.jsonl.gz $(ls $P/sweep_r2_dot1.jsonl.gz 2>/dev/null | sed 's/^/+/') \
  $(ls $P/sweep_r2_offmv_full.jsonl.gz 2>/dev/null | sed 's/^/+/') $(ls $P/sweep_r2_chunk_A.jsonl.gz 2>/dev/null) \
  $(ls $P/sweep_r2_offtmv_full.jsonl.gz 2>/dev/null | sed 's/^/+/') $(ls $P/sweep_r2_offtmv_full2.jsonl.gz 2>/dev/null | sed 's/^/+/')
python tools/fit_thresholds.py "$OUT" --ops mv,tmv,dot --protect-bench --neighbor-weight 0.5 --prefer-staged-dot 0.03 \
  --out paper_conf_pldi_samadihmlm12_b200/csrc/table_data.inc --json $P/selector_table_r2.json > /dev/null
