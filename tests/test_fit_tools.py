"""Host-side selector-fitting tools (tools/fit_thresholds.py, tools/merge_sweeps.py): the
table is what AUTO runs, so its construction is tested like any other host logic.  CPU only."""
import gzip
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(ROOT, "tools"))

import fit_thresholds as ft  # noqa: E402


def run(op, R, C, variant, params, gbps, grid=100, vec=False, mis=True, req=None):
    return {"op": op, "dtype": "f32", "R": R, "C": C, "variant": variant, "req": req or variant,
            "params": params, "us": 4 * R * C / gbps / 1e3, "GBps": gbps,
            "plan": {"vec_shape": vec, "mis": mis, "grid": [grid, grid]}}


def test_staged_tile_height_becomes_a_size():
    # 47 rows of 257 words = 47.2 KB -> -48 KB (whole KB, rounded up); DOT stages two operands
    assert ft.norm_params(run("mv", 262144, 257, "MV_SUBWARP", [16, 0, 0, 0, 4, 256, 47], 1))[6] == -48
    assert ft.norm_params(run("dot", 262144, 257, "MV_SUBWARP", [16, 0, 0, 0, 4, 256, 47], 1))[6] == -95
    # TMV: rows of B plus their x value
    assert ft.norm_params(run("tmv", 9, 8388608, "TMV_REGTILE", [0, 0, 0, 0, 4, 512, 1364], 1))[6] == -54
    # other plans keep their parameters
    assert ft.norm_params(run("mv", 8192, 8192, "MV_CPR", [256, 0, 0, 4, 1], 1))[:5] == [256, 0, 0, 4, 1]


def test_fit_scores_fractions_not_raw_times():
    """A cell holding a small and a large shape: the large shape's winner must not lose just
    because the small shape's runs are faster in microseconds."""
    rows = [run("mv", 2097152, 17, "MV_TPR", [256, 0, 0, 2], 6100),        # small shape: TPR best
            run("mv", 2097152, 17, "MV_SUBWARP", [1, 0, 0, 1, 2], 6000),
            run("mv", 3145728, 22, "MV_TPR", [256, 0, 0, 2], 3000),        # large shape: TPR poor
            run("mv", 3145728, 22, "MV_SUBWARP", [1, 0, 0, 1, 2], 6500)]
    t = ft.fit(rows)
    assert len(t) == 1 and t[0]["variant"] == "MV_SUBWARP", t
    assert t[0]["shapes"] == 2


def test_fit_tie_break_prefers_fewer_ctas_and_uses_mis_grid():
    rows = [run("dot", 1048576, 65, "MV_TPR", [128, 0, 1, 4], 6854, grid=148),
            run("dot", 1048576, 65, "MV_SUBWARP", [16, 0, 0, 0, 4, 512, 94], 6805, grid=296)]
    assert ft.fit(rows)[0]["variant"] == "MV_TPR"


def test_merge_later_runs_win_and_full_resweeps_replace_shapes(tmp_path):
    a = [run("mv", 64, 65, "MV_TPR", [128, 0, 0, 4], 1000), run("mv", 64, 65, "MV_WPR", [0, 0, 0, 1], 900),
         run("mv", 8, 9, "MV_TPR", [128, 0, 0, 4], 100)]
    b = [run("mv", 64, 65, "MV_TPR", [128, 0, 0, 4], 2000)]          # same key: replaces
    c = [run("mv", 8, 9, "MV_WPR", [0, 0, 0, 1], 50)]                # "+": drops every earlier 8x9 run
    paths = []
    for name, rows in (("a.jsonl.gz", a), ("b.jsonl", b), ("c.jsonl", c)):
        p = tmp_path / name
        op = gzip.open if name.endswith(".gz") else open
        with op(p, "wt") as f:
            for r in rows:
                f.write(json.dumps(r) + "\n")
        paths.append(str(p))
    out = tmp_path / "m.jsonl"
    subprocess.check_call([sys.executable, os.path.join(ROOT, "tools", "merge_sweeps.py"), str(out),
                           paths[0], paths[1], "+" + paths[2]], stderr=subprocess.DEVNULL)
    m = [json.loads(l) for l in open(out)]
    got = {(r["R"], r["variant"]): r["GBps"] for r in m}
    assert got == {(64, "MV_TPR"): 2000, (64, "MV_WPR"): 900, (8, "MV_WPR"): 50}


def test_prefer_staged_dot_only_for_big_short_row_dot_cells():
    """--prefer-staged-dot: in a DOT cell of rows with 64..1023 values and >= 2^25 elements, a
    staged row-tile candidate (XSMEM 4) within the margin of the top score wins; outside that
    range (MV, long rows, small cells, beyond the margin) the plain fit decides."""
    def cell(op, R, C, direct, staged):
        return [run(op, R, C, "MV_SUBWARP", [8, 0, 0, 4, 0], direct, vec=True, mis=False),
                run(op, R, C, "MV_SUBWARP", [8, 0, 0, 0, 4, 256, 47], staged, vec=True, mis=False)]
    t = ft.fit(cell("dot", 1048576, 64, 6800, 6700), prefer_staged_dot=0.03)
    assert t[0]["xsmem"] == 4, t
    assert ft.fit(cell("dot", 1048576, 64, 6800, 6700))[0]["xsmem"] == 0                    # off by default
    assert ft.fit(cell("dot", 1048576, 64, 7100, 6700), prefer_staged_dot=0.03)[0]["xsmem"] == 0   # 5.6 % apart
    assert ft.fit(cell("mv", 1048576, 64, 6800, 6700), prefer_staged_dot=0.03)[0]["xsmem"] == 0    # not DOT
    assert ft.fit(cell("dot", 8192, 512, 6800, 6700), prefer_staged_dot=0.03)[0]["xsmem"] == 0     # 2^22 elements
