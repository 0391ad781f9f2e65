"""C-ABI library: loads, exports every symbol include/adaptic.h declares, and the
host-only planner (adaptic_plan is O(1) host logic, no device work) behaves.
Runs without a GPU (no compute calls)."""
import ctypes
import os
import re

import pytest

from paper_conf_pldi_samadihmlm12_b200 import _lib as L
import paper_conf_pldi_samadihmlm12_b200 as adaptic

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "adaptic.h")


def _declared_symbols():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(adaptic_[a-z_]+)\s*\(", src)))


def test_library_exports_every_declared_symbol():
    lib = ctypes.CDLL(L.LIB_PATH)
    declared = _declared_symbols()
    assert len(declared) >= 12
    for name in declared:
        assert hasattr(lib, name), name
    assert sorted(L.SYMBOLS) == declared
    assert L.lib().adaptic_abi_version() == 6


def test_enums_match_header():
    src = open(HEADER).read()
    for i, name in enumerate(L.VARIANTS):
        assert re.search(rf"ADAPTIC_V_{name}\s*=\s*{i}\b", src), name
        assert L.lib().adaptic_variant_name(i).decode() == name
    for name, val in [("ADAPTIC_OP_MV", 0), ("ADAPTIC_OP_TMV", 1), ("ADAPTIC_OP_DOT", 2),
                      ("ADAPTIC_F32", 0), ("ADAPTIC_I32", 1), ("ADAPTIC_ERR_CUDA", 6)]:
        assert re.search(rf"{name}\s*=\s*{val}\b", src), name
    assert L.lib().adaptic_status_string(4).decode() == "ADAPTIC_ERR_ALIAS"


SWEEP = [(1 << k, 1 << (26 - k)) for k in range(3, 24)]


@pytest.mark.parametrize("op", ["mv", "tmv", "dot"])
@pytest.mark.parametrize("dt", ["f32", "i32"])
def test_selector_covers_sweep_and_bound_holds(op, dt):
    for R, C in SWEEP + [(256, 256), (131072, 32768), (1024, 1 << 24), (1, 1 << 30), (3, 5), (1, 1)]:
        p = adaptic.plan(op, R, C, dt)
        d = p.describe()
        v = d["variant"]
        assert (v in adaptic.TMV_VARIANTS) == (op == "tmv")
        w = 1 if (d["vec_shape"] or d["mis"]) else 0      # index 1: the 128-bit-body kernels
        assert d["path_ok"][w], d
        assert d["chain"][w] + d["depth"][w] <= 1677 or dt == "i32", d
        assert d["grid"][w] >= 1
        if d["splits"] > 1 or d["flat"]:                   # cross-CTA merge: partials + ticket
            assert p.workspace_bytes > 0
        else:
            assert p.workspace_bytes == 0


@pytest.mark.parametrize("variant", adaptic.MV_VARIANTS)
def test_forced_mv_variants_sweep(variant):
    for R, C in SWEEP:
        try:
            p = adaptic.plan("mv", R, C, "f32", variant=variant)
        except adaptic.AdapticError as e:
            assert e.status == L.ERR_UNSUPPORTED
            continue
        d = p.describe()
        assert d["variant"] == variant and d["source"] == "forced"
        assert d["path_ok"][1]


@pytest.mark.parametrize("variant", adaptic.TMV_VARIANTS)
def test_forced_tmv_variants_sweep(variant):
    ok = 0
    for R, C in SWEEP:
        try:
            p = adaptic.plan("tmv", R, C, "f32", variant=variant)
        except adaptic.AdapticError as e:
            assert e.status == L.ERR_UNSUPPORTED
            continue
        ok += 1
        assert p.describe()["path_ok"][1]
    assert ok > 0


def test_variant_op_mismatch_is_unsupported():
    with pytest.raises(adaptic.AdapticError) as e:
        adaptic.plan("mv", 64, 64, variant="TMV_COL")
    assert e.value.status == L.ERR_UNSUPPORTED
    with pytest.raises(adaptic.AdapticError) as e:
        adaptic.plan("tmv", 64, 64, variant="MV_WPR")
    assert e.value.status == L.ERR_UNSUPPORTED
    with pytest.raises(adaptic.AdapticError) as e:
        adaptic.plan("dot", 64, 64, variant="TMV_SPLITK")
    assert e.value.status == L.ERR_UNSUPPORTED


def test_invalid_args():
    lib = L.lib()
    h = ctypes.c_void_p()
    assert lib.adaptic_plan(0, -1, 5, 0, ctypes.byref(h)) == L.ERR_INVALID_ARG
    assert lib.adaptic_plan(0, 5, -1, 0, ctypes.byref(h)) == L.ERR_INVALID_ARG
    assert lib.adaptic_plan(9, 5, 5, 0, ctypes.byref(h)) == L.ERR_INVALID_ARG
    assert lib.adaptic_plan(0, 5, 5, 9, ctypes.byref(h)) == L.ERR_INVALID_ARG
    assert lib.adaptic_plan(0, 1 << 40, 1 << 40, 0, ctypes.byref(h)) == L.ERR_INVALID_ARG  # byte overflow
    assert lib.adaptic_plan(0, 5, 5, 0, None) == L.ERR_INVALID_ARG
    assert lib.adaptic_plan_forced(0, 5, 5, 0, 42, None, ctypes.byref(h)) == L.ERR_INVALID_ARG
    bad = (ctypes.c_int32 * 4)(3, 0, 0, 0)     # SUBWARP lanes must be a power of two
    assert lib.adaptic_plan_forced(0, 64, 64, 0, L.V["MV_SUBWARP"], bad, ctypes.byref(h)) == L.ERR_INVALID_ARG
    assert lib.adaptic_run(None, None, None, None, None) == L.ERR_INVALID_ARG
    assert lib.adaptic_plan_describe(None, None, 0) == -1
    assert lib.adaptic_plan_workspace_bytes(None) == 0


def test_degenerate_plans_and_run_without_device():
    p = adaptic.plan("mv", 0, 10)
    assert p.run_ptrs(0, 0, 0) == L.OK            # R == 0: nothing launched
    p = adaptic.plan("tmv", 5, 0)
    assert p.run_ptrs(0, 0, 0) == L.ERR_INVALID_ARG   # y required
    assert p.run_ptrs(0, 0, 0x1002) == L.ERR_MISALIGNED


def test_alias_and_alignment_checks_are_host_side():
    p = adaptic.plan("mv", 16, 16)
    A, x = 0x10000000, 0x20000000
    assert p.run_ptrs(A, x, A + 64) == L.ERR_ALIAS            # y inside A
    assert p.run_ptrs(A, x, x) == L.ERR_ALIAS                 # y == x
    assert p.run_ptrs(A + 2, x, 0x30000000) == L.ERR_MISALIGNED
    pd = adaptic.plan("dot", 4, 8)
    assert pd.run_ptrs(A, x, x + 4 * 8 * 4 - 4) == L.ERR_ALIAS  # DOT's b spans N*L elements


def test_workspace_contract():
    p = adaptic.plan("mv", 8, 1 << 23, variant="MV_SPLIT")
    n = p.workspace_bytes
    assert n > 0
    assert p.run_ptrs(0x10000000, 0x20000000, 0x30000000) == L.ERR_NO_WORKSPACE
    with pytest.raises(adaptic.AdapticError):
        p.set_workspace(0x40000000, n - 4)
    with pytest.raises(adaptic.AdapticError):
        p.set_workspace(0x40000004, n)                        # 16-byte alignment
    p.set_workspace(0x40000000, n)
    p.set_workspace(0, 0)


def test_forced_params_are_honoured():
    p = adaptic.plan("tmv", 8192, 8192, variant="TMV_SPLITK", params=[32, 16, 2, 8])
    d = p.describe()
    assert (d["lanes"], d["splits"], d["ctas_per_sm"], d["unroll"]) == (32, 16, 2, 8)
    p = adaptic.plan("mv", 1 << 20, 64, variant="MV_SUBWARP", params=[4, 0, 0, 2])
    d = p.describe()
    assert (d["lanes"], d["unroll"], d["rows_per_group"]) == (4, 2, 4)


def test_plan_is_o1_host_only():
    """P:236 (selection adds no visible time): repeated plans cost one memo lookup + a
    struct copy.  tools/plan_latency.c times adaptic_plan + destroy in C over the 93 shapes
    of the bench workloads (no device needed); the binding's own overhead is ctypes."""
    import json
    import subprocess
    exe = os.path.join(ROOT, "tools", "plan_latency")
    src = exe + ".c"
    subprocess.check_call(["gcc", "-O2", "-I" + os.path.join(ROOT, "include"), src,
                           "-L" + os.path.dirname(L.LIB_PATH), "-ladaptic",
                           "-Wl,-rpath," + os.path.dirname(L.LIB_PATH), "-o", exe])
    r = json.loads(subprocess.check_output([exe, "500"], text=True))
    assert r["shapes"] == 93
    assert r["plan_ns_median"] < 1000 and r["plan_ns_max"] < 5000, r
    import time
    t = time.perf_counter()
    for _ in range(2000):
        adaptic.plan("tmv", 8192, 8192)
    dt = (time.perf_counter() - t) / 2000
    assert dt < 2e-4, dt


def test_run_batch_host_checks():
    lib = L.lib()
    VP = ctypes.c_void_p
    one = (VP * 1)(VP(None))
    assert lib.adaptic_run_batch(0, None, None, None, None, 1, None) == L.OK
    assert lib.adaptic_run_batch(-1, one, one, one, one, 1, None) == L.ERR_INVALID_ARG
    assert lib.adaptic_run_batch(1, one, one, one, one, 0, None) == L.ERR_INVALID_ARG
    assert lib.adaptic_run_batch(1, one, one, one, one, 9, None) == L.ERR_INVALID_ARG
    assert lib.adaptic_run_batch(1, one, one, one, one, 2, None) == L.ERR_INVALID_ARG   # NULL plan
    p = adaptic.plan("mv", 16, 16)
    b = L.Batch([(p, 0x10000000, 0x20000000, 0x10000040)])                          # y inside A
    with pytest.raises(adaptic.AdapticError) as e:
        b.run(2)
    assert e.value.status == L.ERR_ALIAS
