#!/usr/bin/env python
"""Round-2 selector report (profiles/r2_selector_report.md): how the fitted table
generalises, on shapes it was NOT fitted on, for each of the paper's size regimes.

Sections (every AUTO-vs-best comparison uses AUTO and the fixed candidates of the SAME kind
of timing; 'best fixed' = the fastest of every swept (variant, params) on that shape):
  1. round-1 table on held-out set A (5/7 multipliers + random; measured before set A was
     added to the training data) -- the honest baseline of round 1's table;
  2. round-2 table on held-out set B (3/13 multipliers + random, never fitted), >= 256 MiB;
  3. round-2 table on held-out set Bs, the paper's small-input regime (4-64 MiB, CUDA-graph
     device timing; gate: within 5 % of the best fixed only -- these inputs live in L2);
  4. the offline replica (tools/select_sim.py) on the same sets, as a cross-check;
  2c / 3c. the clean sets C / Cs, defined after the last table / planner change (section 2 and 3's
     set B located the failures that the end-of-round planner rules address).

  python tools/selector_report_r2.py --out profiles/r2_selector_report.md
"""
import argparse
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
P = os.path.join(ROOT, "profiles")


def report(args):
    r = subprocess.run([sys.executable, os.path.join(HERE, "report.py")] + args, capture_output=True, text=True,
                       cwd=ROOT)
    if r.returncode:
        raise SystemExit(r.stderr)
    return r.stdout


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=os.path.join(P, "r2_selector_report.md"))
    ap.add_argument("--valB", default=os.path.join(P, "val_r2_valB3_auto.jsonl.gz"))
    ap.add_argument("--valBs", default=os.path.join(P, "val_r2_valBs3_auto.jsonl.gz"))
    a = ap.parse_args()
    best_B = [os.path.join(P, f) for f in ("val_r2_heldoutB_nodot.jsonl.gz", "val_r2_dotB.jsonl.gz",
                                             "val_r2_tshift_B.jsonl.gz", "val_r2_misx_B.jsonl.gz",
                                             "val_r2_rtc_B.jsonl.gz", "val_r2_chunk_B.jsonl.gz")]
    parts = ["# Selector report (round 2): held-out generalisation\n",
             "Shapes: `tools/heldout_shapes.py` (A, B: 256 MiB - 2 GiB; As, Bs: 4-64 MiB).  Training input: "
             "`tools/refit_r2.sh` (round 1's exact fit input + set A + As + the DOT re-sweep with b aligned + "
             "small diagonals + Sdot lengths + constant-shift TMV, misaligned-MV, long-row and column-chunk "
             "candidates, the offgrid MV shapes re-swept in full).  Sets B and Bs are never fitted; sections 2 "
             "and 3 time the FINAL table's AUTO pick and every fixed candidate of each shape in one run.  Gates (BJ:north_star): AUTO >= 0.95 x the best fixed variant and >= 0.70 of the "
             "measured copy peak (6554.9 GB/s) for inputs >= 256 MiB.\n"]
    parts.append("## 1. Round-1 table, held-out set A (before A entered the training data)\n")
    parts.append("DOT rows of this run placed b right after a, so for R*C % 4 != 0 the two operands differed "
                 "in alignment mod 16 and the misaligned-row DOT kernels (which need equal alignment) fell back "
                 "to scalar loads: those DOT rows understate both AUTO and the best fixed.\n\n```\n")
    parts.append(report([os.path.join(P, "sweep_r2_trainA.jsonl.gz")]).splitlines()[-2] + "\n```\n")
    parts.append("## 2. Round-2 table before the end-of-round planner rules (code of commit 8a83827), held-out set "
                 "B (never fitted), >= 256 MiB, every candidate and AUTO in ONE run (`val_r2_B_final`)\n\n")
    parts.append(report([os.path.join(P, "val_r2_B_final.jsonl.gz")]))
    parts.append("\n## 3. The same code, held-out small set Bs (4-64 MiB, device-timed from CUDA graphs, one "
                 "run: `val_r2_Bs_final`)\n\n")
    parts.append(report([os.path.join(P, "val_r2_Bs_final.jsonl.gz"), "--min-bytes", "0", "--no-peak-gate"]))
    parts.append("\n## 2c. CLEAN held-out set C (9 / 11 multipliers + 24 random shapes, new seed; defined AFTER the "
                 "last planner change of round 2, every candidate and AUTO of a shape in one run; its TMV shapes "
                 "re-swept after the last refit of the misaligned TMV cells: `val_r2_C_final2`), >= 256 MiB\n\n")
    parts.append(report([os.path.join(P, "val_r2_C_final2.jsonl.gz")]))
    parts.append("\n## 3c. CLEAN held-out small set Cs (4-64 MiB, graph-timed, TMV re-swept likewise: `val_r2_Cs_final2`)\n\n")
    parts.append(report([os.path.join(P, "val_r2_Cs_final2.jsonl.gz"), "--min-bytes", "0", "--no-peak-gate"]))
    parts.append("\n## 3b. The same table's AUTO picks timed in another run against the earlier sweeps' best "
                 "fixed (`val_r2_valB3_auto` vs `val_r2_heldoutB_nodot` + DOT / tshift / misx / rtc / chunk "
                 "sweeps): cross-run timing, so a ~1 % box-to-box shift moves borderline shapes\n\n```\n")
    parts.append(report([a.valB, "--best-from"] + best_B).splitlines()[-2] + "\n```\n")
    r = subprocess.run([sys.executable, os.path.join(HERE, "select_sim.py"), "--table",
                        os.path.join(P, "selector_table_r2.json")] + best_B, capture_output=True, text=True)
    parts.append("\n## 4. Offline replica on set B (tools/select_sim.py: the fitted entry's measured GB/s on each "
                 "shape, where the entry was a swept candidate)\n\n```\n" + r.stdout.splitlines()[0] + "\n```\n")
    open(a.out, "w").write("".join(parts))
    print(open(a.out).read()[:3000])


if __name__ == "__main__":
    main()
