"""Host-side planner rules added for the stencil, the x-tile stream-K MV kernel and the
multi-vector TMA/TMV choices.  No GPU needed: plans are built and
described, nothing is launched (no device: occupancy takes its documented fallback)."""
import pytest

import paper_conf_pldi_samadihmlm12_b200 as adaptic


def d(op, R, C, dtype="f32", variant="AUTO", params=None, nvec=1):
    return adaptic.plan(op, R, C, dtype, variant=variant, params=params, nvec=nvec).describe()


def test_stencil_selector_and_orders():
    assert d("stencil5", 8192, 8192)["variant"] == "ST_DIRECT"
    assert d("stencil5", 8192, 8192)["xmode"] == 0                 # rows < 2 MB: row-major sweep
    assert d("stencil5", 8, 1 << 23)["xmode"] == 1                 # 32 MB rows: L2 strips
    assert d("stencil5", 64, 4096, variant="ST_DIRECT", params=[0, 0, 0, 0, 0, 0, 0, 2])["xmode"] == 1
    col = d("stencil5", 64, 4096, variant="ST_DIRECT", params=[0, 0, 0, 0, 0, 0, 16, 3])
    assert col["xmode"] == 2 and col["rows_per_group"] == 16
    assert d("stencil5", 100, 101)["vec_shape"] is False           # odd width: scalar direct kernel
    t = d("stencil5", 4096, 16384, variant="ST_TILE")               # the paper's reuse-metric super tile
    assert t["variant"] == "ST_TILE" and t["smem"] > 0
    with pytest.raises(adaptic.AdapticError):
        d("stencil5", 64, 64, "i32")


def test_tile_kernel_cells_fp32_and_int32():
    for dt in ("f32", "i32"):
        p = d("mv", 4096, 16384, dt)
        assert p["variant"] == "MV_SPLIT" and p["xmode"] == 4, p
        assert p["lanes"] == 16384 and p["path_ok"][1]
    p = d("mv", 300, 50000, variant="MV_SPLIT", params=[1024, 0, 0, 0, 3, 0, 2])
    assert p["xmode"] == 4 and p["lanes"] == 1024 and p["rows_per_group"] == 2
    assert p["splits"] == -(-50000 // 1024) and p["workspace_bytes"] > 0
    # one chunk: no merge, no workspace
    assert d("mv", 300, 1024, variant="MV_SPLIT", params=[0, 0, 0, 0, 3])["workspace_bytes"] == 0
    # rows off the 16-byte grid never take the tile kernel
    assert d("mv", 300, 1027, variant="MV_SPLIT", params=[0, 0, 0, 0, 3])["xmode"] != 4


def test_multi_vector_rules():
    assert d("mv", 16384, 4096, nvec=4)["xmode"] == 4              # x-tile stream-K (C < 8192)
    assert d("mv", 8192, 8192, nvec=4)["xmode"] == 6               # long rows: the matrix via the TMA ring
    assert d("mv", 64, 1 << 20, nvec=8)["xmode"] == 6
    assert d("mv", 8, 1 << 23, nvec=4)["xmode"] == 6                # (round 1: interleaved splits)
    assert d("mv", 1 << 20, 64, nvec=4)["variant"] == "MV_SUBWARP"  # short rows: x in registers
    few = d("tmv", 64, 1 << 20, nvec=4)
    assert few["xmode"] == 5 and few["lanes"] == 16                 # one contiguous TMA tile
    huge = d("tmv", 262144, 256, nvec=2)
    assert huge["xmode"] == 5 and huge["lanes"] == 256 and huge["splits"] == 1
    assert d("tmv", 262144, 256, nvec=4)["xmode"] == 8                # row groups of 4 (measured +2 %)
    mid = d("tmv", 8192, 8192, nvec=4)
    assert mid["xmode"] == 8 and mid["variant"] == "TMV_SPLITK"     # rows in groups of 4, x as float4
    assert d("tmv", 1 << 20, 64, nvec=4)["xmode"] == 8
    assert d("tmv", 1 << 21, 32, nvec=4)["variant"] == "TMV_COL"
    assert d("tmv", 8192, 8190, nvec=4)["xmode"] != 8               # C % 4 != 0: register-fed tiles
    forced = d("tmv", 8192, 8192, variant="TMV_SPLITK", params=[128, 9, 0, 0, 3], nvec=8)
    assert forced["xmode"] == 5 and forced["splits"] == 9


@pytest.mark.parametrize("K", [2, 4, 8])
def test_multi_plans_respect_the_error_bound(K):
    for op in ("mv", "tmv"):
        for k in range(3, 24, 2):
            p = d(op, 1 << k, 1 << (26 - k), nvec=K)
            w = 1 if p["vec_shape"] else 0
            assert p["path_ok"][w], (op, k, p)


def test_staged_row_tiles_mv_dot():
    """XSMEM 4 on MV_SUBWARP / MV_WPR: the staged row-tile kernel (rowtile_kernel.cuh)."""
    p = d("mv", 262144, 257, variant="MV_WPR", params=[0, 0, 0, 0, 4])
    assert p["xmode"] == 4 and p["lanes"] == 32 and p["stages"] >= 2 and p["mis"]
    assert p["rows_per_group"] % 8 == 0                               # whole warps of rows (256/32 groups)
    assert p["chain"][1] == 5 and p["path_ok"][1]                      # ceil(ceil(257/32)/2)
    # ROWS = -n: an ~n KB tile (the fitted tables' portable form); DOT stages b too
    assert d("mv", 100000, 100, variant="MV_SUBWARP", params=[4, 0, 0, 0, 4, 256, -12])["rows_per_group"] == 30
    assert d("dot", 100000, 100, variant="MV_SUBWARP", params=[4, 0, 0, 0, 4, 256, -12])["rows_per_group"] == 15
    # an explicit height too tall for two stages is capped, not refused
    capped = d("mv", 3145728, 22, variant="MV_SUBWARP", params=[1, 0, 0, 0, 4, 256, 722])
    assert capped["rows_per_group"] < 722 and capped["stages"] == 2
    # x must fit the registers: C <= 32 * G
    with pytest.raises(adaptic.AdapticError):
        d("mv", 1000, 300, variant="MV_SUBWARP", params=[8, 0, 0, 0, 4])
    # the fitted table takes the staged kernel on the off-grid short-row shapes
    for op, R, C in (("mv", 262144, 257), ("mv", 8388608, 9), ("dot", 524288, 129)):
        assert d(op, R, C)["xmode"] == 4, (op, R, C)


def test_staged_tmv_tiles():
    """XSMEM 4 on TMV_REGTILE: tiles of B + x chunks (tmv_rowtile_kernel.cuh), R <= 1024."""
    p = d("tmv", 9, 8388608, variant="TMV_REGTILE", params=[0, 0, 0, 0, 4])
    assert p["xmode"] == 4 and p["block"] == 256 and p["rows_per_group"] % 4 == 0 and p["stages"] >= 3
    assert p["workspace_bytes"] > 0 and p["path_ok"][1]
    assert d("tmv", 513, 131072, variant="TMV_REGTILE", params=[0, 0, 0, 0, 4])["block"] == 1024
    two = d("tmv", 300, 1000, variant="TMV_REGTILE", params=[0, 0, 0, 0, 4, 256])
    assert two["block"] == 256 and two["unroll"] == 2                  # two outputs per thread
    with pytest.raises(adaptic.AdapticError):                          # more than 2 outputs per thread
        d("tmv", 600, 1000, variant="TMV_REGTILE", params=[0, 0, 0, 0, 4, 256])
    four = d("tmv", 4000, 1000, variant="TMV_REGTILE", params=[0, 0, 0, 0, 4])
    assert four["block"] == 1024 and four["unroll"] == 4               # four outputs per thread
    with pytest.raises(adaptic.AdapticError):                          # R > 4096
        d("tmv", 4097, 1000, variant="TMV_REGTILE", params=[0, 0, 0, 0, 4])
    with pytest.raises(adaptic.AdapticError):                          # tile height not a multiple of 4
        d("tmv", 9, 1000, variant="TMV_REGTILE", params=[0, 0, 0, 0, 4, 256, 6])
    for R, C in ((9, 8388608), (129, 524288), (14, 5162220)):
        assert d("tmv", R, C)["xmode"] == 4, (R, C)


def _p(p):
    return (list(p) + [0] * 9)[:9]


def test_chunk_plan_geometry():
    """XSMEM 13 (staged column chunks): nch = ceil(C / (NT MX)) chunks, k <= 4 row segments per
    ~64 KB tile, >= 2 ring stages, partials nch x R (+ counter) only when nch > 1; the selector
    takes it for the offgrid bench's long C + 1 rows (profiles/sweep_r2_offmv_full)."""
    for R, C, MX, NT in ((512, 131073, 16, 512), (16, 4194305, 36, 512), (3, 5000, 8, 256), (1000, 8193, 36, 256)):
        p = d("mv", R, C, variant="MV_SPLIT", params=_p([MX, 0, 0, 0, 13, NT]))
        nch = -(-C // (NT * MX))
        assert p["xmode"] == 13 and p["splits"] == nch and p["lanes"] == MX and p["block"] == NT, p
        assert 1 <= p["rows_per_group"] <= min(4, R) and p["stages"] >= 2 and p["path_ok"][1]
        W = -(-C // nch)
        assert p["smem"] == p["stages"] * p["rows_per_group"] * ((W + 9) // 4 * 4) * 4
        if nch > 1:
            assert p["workspace_bytes"] >= nch * R * 4 + 4
    for MX in (4, 12, 64):
        with pytest.raises(adaptic.AdapticError):
            d("mv", 100, 100000, variant="MV_SPLIT", params=_p([MX, 0, 0, 0, 13]))
    for R in (32, 128, 512, 1024):
        a = d("mv", R, (1 << 26) // R + 1)
        assert a["xmode"] == 13, (R, a)


def test_group_plan_geometry():
    """XSMEM 12 (TMV on groups of four rows): KG = NT div R sub-groups with the fewest idle
    threads for R <= 1024, S = 2..4 slots per thread above, R in [4, 2560]; two-level merge
    workspace (G + ceil(G / 16)) x R partials."""
    for R in (5, 17, 129, 513, 1023):
        p = d("tmv", R, 100003, variant="TMV_SPLITK", params=_p([0, 0, 0, 0, 12]))
        assert p["xmode"] == 12 and p["rows_per_group"] == 1 and p["block"] >= R and p["block"] % 32 == 0, p
        assert (p["block"] // R) * R / p["block"] >= 0.75
    for R, S in ((1025, 2), (1537, 3), (2049, 4), (2559, 4)):
        p = d("tmv", R, 9999, variant="TMV_REGTILE", params=_p([0, 0, 0, 0, 12]))
        assert p["rows_per_group"] == S and p["block"] * S >= R and p["block"] <= 640, (R, p)
        G = p["grid"][1]
        assert p["workspace_bytes"] >= (G + -(-G // 16)) * R * 4
    for R in (3, 2561):
        with pytest.raises(adaptic.AdapticError):
            d("tmv", R, 1000, variant="TMV_SPLITK", params=_p([0, 0, 0, 0, 12]))
    # interleaved order and forced slots
    assert d("tmv", 129, 5000, variant="TMV_SPLITK", params=_p([0, 0, 0, 0, 12, 0, 2, 2]))["rows_per_group"] == 2


def test_staged_tile_floor_and_lane_group_bump():
    """Staged MV / DOT row tiles from the table or the default: >= ~40 KB per tile when the
    matrix still gives every SM two tiles (training sweeps: smaller tiles 0.71-0.93 of the big
    ones); a fitted lane group too small for this C grows to the smallest that holds it (the
    cell spans a factor 2 in C); a FORCED size stays exact."""
    for R, C in ((2872808, 63), (3085902, 61)):
        p = d("dot", R, C)
        assert p["xmode"] == 4 and p["rows_per_group"] * C * 8 >= 40 * 1024, p
    p = d("dot", 393216, 416)                 # cell entry G = 8 fitted on C = 256 (G * 32 < 416)
    assert p["xmode"] == 4 and p["lanes"] == 16, p
    assert d("mv", 100000, 100, variant="MV_SUBWARP", params=[4, 0, 0, 0, 4, 256, -12])["rows_per_group"] == 30
    with pytest.raises(adaptic.AdapticError):  # forced G too small: still an error
        d("dot", 393216, 416, variant="MV_SUBWARP", params=[8, 0, 0, 0, 4, 256])


def test_misaligned_tmv_funnel_cells_run_the_constant_shift_kernel():
    """Rows off the 16-byte grid with 1024 <= R <= 2^17 and >= 2^24 elements: a table cell that
    kept the funnel kernel (XSMEM 0) runs the constant-shift kernel (XSMEM 7) instead (training
    sweeps: 1.03-1.19x, 15 of 15); small problems and aligned rows keep their fitted entry."""
    for R, C in ((27215, 2924), (1950, 44236), (16385, 4096)):
        p = d("tmv", R, C)
        assert p["variant"] == "TMV_SPLITK" and p["xmode"] == 7, (R, C, p)
    assert d("tmv", 1025, 1024)["xmode"] != 7              # 1 Mi elements: the fitted small-cell entry
    assert d("tmv", 4772, 50180)["xmode"] != 7             # R % 4 == 0: the 128-bit path
