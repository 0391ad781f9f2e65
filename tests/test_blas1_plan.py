"""Host-side planner for the BLAS-1 reductions (ASUM/NRM2/IAMAX/IAMIN, SURVEY 8(f)
rank 1): op/variant/dtype rules, the ASUM error bound, workspace sizing and the
x-unused run contract.  No GPU needed (no compute calls)."""
import re
import os

import pytest

from paper_conf_pldi_samadihmlm12_b200 import _lib as L
import paper_conf_pldi_samadihmlm12_b200 as adaptic

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OPS = ("asum", "nrm2", "iamax", "iamin")
SHAPES = [(1, 1 << k) for k in range(10, 31, 2)] + [(1 << k, 1 << (26 - k)) for k in range(0, 24, 3)] + \
         [(3, 5), (1, 1), (1000, 1000), (7, 100003)]


def test_op_enums_match_header():
    src = open(os.path.join(ROOT, "include", "adaptic.h")).read()
    for name, val in [("ASUM", L.OP_ASUM), ("NRM2", L.OP_NRM2), ("IAMAX", L.OP_IAMAX), ("IAMIN", L.OP_IAMIN)]:
        assert re.search(rf"ADAPTIC_OP_{name}\s*=\s*{val}\b", src), name


@pytest.mark.parametrize("op", OPS)
def test_auto_plans_are_b1_variants_and_bounded(op):
    for R, C in SHAPES:
        p = adaptic.plan(op, R, C)
        d = p.describe()
        assert d["op"] == op.upper()
        assert d["variant"] in L.B1_VARIANTS, d
        w = 1 if d["vec_shape"] else 0
        assert d["path_ok"][w]
        if op == "asum":
            assert d["chain"][w] + d["depth"][w] <= 1677, d     # gamma_m <= 1e-4 (Higham 4.4)
        else:
            assert d["chain"][w] == 0                            # fp64 / exact: no fp32 chain
        assert (p.workspace_bytes > 0) == (d["splits"] > 1)
        if d["splits"] > 1:
            assert p.workspace_bytes >= R * d["splits"] * 8 + R * 4


def test_regimes_follow_the_paper():
    """Fig. 1 / P:116: few long rows -> split rows; many short rows -> lane groups."""
    assert adaptic.plan("asum", 1, 1 << 26).variant == "MV_SPLIT"
    assert adaptic.plan("asum", 1 << 22, 16).variant == "MV_SUBWARP"
    assert adaptic.plan("nrm2", 1 << 16, 1024).variant == "MV_WPR"
    assert adaptic.plan("iamax", 4096, 16384).variant == "MV_CPR"


@pytest.mark.parametrize("op", OPS)
def test_unsupported_combinations(op):
    for v in ("MV_TPR", "TMV_COL", "TMV_SPLITK", "TMV_REGTILE"):
        with pytest.raises(adaptic.AdapticError) as e:
            adaptic.plan(op, 8, 64, variant=v)
        assert e.value.status == L.ERR_UNSUPPORTED
    with pytest.raises(adaptic.AdapticError) as e:
        adaptic.plan(op, 8, 64, "i32")
    assert e.value.status == L.ERR_UNSUPPORTED


def test_iamax_length_limit():
    with pytest.raises(adaptic.AdapticError) as e:
        adaptic.plan("iamax", 1, 1 << 31)
    assert e.value.status == L.ERR_UNSUPPORTED
    adaptic.plan("iamax", 1, (1 << 31) - 1)
    adaptic.plan("asum", 1, 1 << 31)


def test_forced_split_count_and_lanes():
    d = adaptic.plan("asum", 5, 1 << 20, variant="MV_SPLIT", params=[0, 7]).describe()
    assert d["splits"] == 7 and d["ilv"] == 1
    d = adaptic.plan("iamin", 1 << 16, 64, variant="MV_SUBWARP", params=[8, 0, 0, 0, 0, 0, 1]).describe()
    assert (d["lanes"], d["rows_per_group"], d["unroll"]) == (8, 1, 8)
    with pytest.raises(adaptic.AdapticError):
        adaptic.plan("iamin", 64, 64, variant="MV_SUBWARP", params=[3])
    with pytest.raises(adaptic.AdapticError):
        adaptic.plan("iamin", 64, 64, variant="MV_WPR", params=[0, 0, 0, 0, 0, 0, 2])


def test_asum_split_raised_for_the_bound():
    """A single CTA per row on a 2^34 row would chain > 1677 fp32 roundings: CPR is
    refused, SPLIT raises its split count until the bound holds."""
    with pytest.raises(adaptic.AdapticError) as e:
        adaptic.plan("asum", 1, 1 << 34, variant="MV_CPR")
    assert e.value.status == L.ERR_UNSUPPORTED
    d = adaptic.plan("asum", 1, 1 << 34, variant="MV_SPLIT", params=[0, 4]).describe()
    assert d["path_ok"][1]
    adaptic.plan("nrm2", 1, 1 << 30, variant="MV_CPR")     # fp64: no bound to violate


def test_run_contract_x_unused():
    p = adaptic.plan("asum", 16, 16)
    A = 0x10000000
    assert p.run_ptrs(A, 0, A + 64) == L.ERR_ALIAS             # y inside A
    assert p.run_ptrs(A + 2, 0, 0x30000000) == L.ERR_MISALIGNED
    assert p.run_ptrs(0, 0, 0x30000000) == L.ERR_INVALID_ARG   # A required
    q = adaptic.plan("nrm2", 4, 1 << 22, variant="MV_SPLIT")
    assert q.run_ptrs(A, 0, 0x30000000) == L.ERR_NO_WORKSPACE
    assert adaptic.plan("iamax", 0, 5).run_ptrs(0, 0, 0) == L.OK


def test_b1all_plan_and_contract():
    """B1ALL (horizontal actor integration): four N-vectors in y, 32-byte
    partials, the asum chain bound with one accumulator per row."""
    src = open(os.path.join(ROOT, "include", "adaptic.h")).read()
    assert re.search(r"ADAPTIC_OP_B1ALL\s*=\s*7\b", src)
    for R, C in SHAPES:
        d = adaptic.plan("b1all", R, C).describe()
        w = 1 if d["vec_shape"] else 0
        assert d["path_ok"][w] and d["chain"][w] + d["depth"][w] <= 1677, d
    p = adaptic.plan("b1all", 4, 1 << 22, variant="MV_SPLIT")
    d = p.describe()
    assert p.workspace_bytes >= 4 * d["splits"] * 32 + 4 * 4
    A = 0x10000000
    assert p.run_ptrs(A, 0, A + 4 * (1 << 22) * 4 - 8) == L.ERR_ALIAS      # y spans 16*N bytes
    with pytest.raises(adaptic.AdapticError):
        adaptic.plan("b1all", 1, 1 << 31)


def test_multi_vector_plans():
    """adaptic_plan_multi (K vectors, one pass): K in {1,2,4,8}, fp32, MV/TMV only."""
    for op, R, C in (("mv", 1 << 16, 1024), ("mv", 1 << 20, 64), ("mv", 64, 1 << 20), ("tmv", 8192, 8192),
                     ("tmv", 8, 1 << 23), ("mv", 100, 1001), ("tmv", 1001, 100)):
        for K in (2, 4, 8):
            d = adaptic.plan(op, R, C, nvec=K).describe()
            w = 1 if d["vec_shape"] else 0
            assert d["nvec"] == K and d["path_ok"][w] and d["chain"][w] + d["depth"][w] <= 1677, d
    for bad in ((3, L.ERR_UNSUPPORTED), (0, L.ERR_INVALID_ARG), (16, L.ERR_UNSUPPORTED)):
        with pytest.raises(adaptic.AdapticError) as e:
            adaptic.plan("mv", 64, 64, nvec=bad[0])
        assert e.value.status == bad[1]
    for op, dt in (("dot", "f32"), ("asum", "f32"), ("mv", "i32")):
        with pytest.raises(adaptic.AdapticError) as e:
            adaptic.plan(op, 64, 64, dt, nvec=4)
        assert e.value.status == L.ERR_UNSUPPORTED
    p = adaptic.plan("mv", 16, 64, nvec=4)
    A, X = 0x10000000, 0x20000000
    assert p.run_ptrs(A, X, X + 4 * 64 * 4 - 4) == L.ERR_ALIAS      # X spans K*C elements
