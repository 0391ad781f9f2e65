"""Lane groups on TMA-staged row tiles (csrc/rowtile_kernel.cuh; MV_SUBWARP / MV_WPR
with [ADAPTIC_P_XSMEM] = 4) against the oracle -- needs a GPU.

fp32 within 1e-4 * S_r (north_star), int32 bit-exact, P5 (integer-valued fp32) exact.
Covers every lane-group width, tiles of 1 .. many rows, ragged last tiles, a matrix
whose word count is not a multiple of 4 (the last tile's remainder copied by the
threads), rows at every 16-byte phase (C % 4 = 1, 2, 3 and 0), 256/512-thread CTAs,
2..8 ring stages, DOT, and base pointers that are not 16-byte aligned (those run the
variant's direct kernel)."""
import itertools

import numpy as np
import pytest
import torch

import oracle
import synth

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    import paper_conf_pldi_samadihmlm12_b200 as adaptic
    from paper_conf_pldi_samadihmlm12_b200 import _lib as L

DEV = "cuda:0"
TOL = 1e-4


def check(y, ref, dt, what):
    if dt == "i32":
        assert np.array_equal(y, ref), f"{what}: int32 mismatch at {np.nonzero(y != ref)[0][:8]}"
    else:
        yr, S = ref
        err = np.abs(y.astype(np.float64) - yr)
        bad = ~(err <= TOL * S)
        assert not bad.any(), f"{what}: {bad.sum()} out of tolerance, worst {np.max(err - TOL * S)}"


def _collect(cases):
    fails = []
    for what, fn in cases:
        try:
            fn()
        except Exception as e:  # noqa: BLE001 -- report every failing case at once
            fails.append(f"{what}: {type(e).__name__}: {str(e)[:200]}")
    assert not fails, f"{len(fails)} failures:\n" + "\n".join(fails[:40])


def rt_params(g, nt=0, k=0, stages=0, cps=0):
    """[lanes, splits, ctas_per_sm, unroll(stages), xsmem=4, block, rows]"""
    return [g, 0, cps, stages, 4, nt, k]


SHAPES = [(1, 5), (3, 17), (7, 9), (33, 19), (64, 31), (65, 127), (130, 257), (257, 66), (1000, 21),
          (999, 513), (4097, 33), (12345, 9), (100003, 7), (5, 1024), (300, 100), (2, 1), (17, 2), (31, 3)]
PLANS = [("MV_SUBWARP", rt_params(g, nt, k, st)) for g in (1, 2, 4, 8, 16) for nt, k, st in
         ((0, 0, 0), (512, 0, 2), (256, 1, 4), (256, 37, 8))] + \
        [("MV_WPR", rt_params(32, nt, k, st)) for nt, k, st in ((0, 0, 0), (512, 3, 3), (256, 64, 2))]


@pytest.mark.parametrize("op", ["mv", "dot"])
@pytest.mark.parametrize("dt", ["f32", "i32"])
def test_rowtile_every_width_and_tile(op, dt):
    npdt = np.float32 if dt == "f32" else np.int32

    def case(R, C, v, p):
        A = synth.matrix(R, C, "mv", npdt, "uniform", synth.seed(21, "A") + R + C)
        X = (synth.matrix(R, C, "mv", npdt, "uniform", synth.seed(21, "b") + R) if op == "dot"
             else synth.vector(C, npdt, "uniform", synth.seed(21, "x") + C))
        try:
            plan = adaptic.plan(op, R, C, dt, variant=v, params=p)
        except adaptic.AdapticError as e:
            assert e.status == L.ERR_UNSUPPORTED, str(e)
            # auto tile height always fits; a forced one may leave < 2 stages of ring
            assert C > 32 * p[0] or p[6] > 0, f"unexpected UNSUPPORTED {R}x{C} {p}"
            return
        d = plan.describe()
        assert d["xmode"] == 4 and d["stages"] >= 2, d
        fn = adaptic.mv if op == "mv" else adaptic.dot
        y = fn(torch.from_numpy(A).to(DEV), torch.from_numpy(X).to(DEV), variant=v, params=p).cpu().numpy()
        ref = oracle.mv(A, X) if op == "mv" else oracle.dot(A, X)
        check(y, ref, dt, f"{op} {dt} {R}x{C} {v} {p}")
    _collect([(f"{R}x{C} {v} {p}", lambda R=R, C=C, v=v, p=p: case(R, C, v, p))
              for (R, C), (v, p) in itertools.product(SHAPES, PLANS)])


def test_rowtile_exact_on_integer_valued_fp32():
    """P5: every partial sum exact, so the staged kernel equals the oracle bit for bit."""
    for R, C, g in [(4099, 257, 16), (100003, 9, 1), (2049, 1023, 32), (777, 130, 8)]:
        A = synth.matrix(R, C, "mv", np.float32, "smallint", 41 + C)
        x = synth.vector(C, np.float32, "smallint", 42 + C)
        v = "MV_WPR" if g == 32 else "MV_SUBWARP"
        y = adaptic.mv(torch.from_numpy(A).to(DEV), torch.from_numpy(x).to(DEV), variant=v,
                       params=rt_params(g)).cpu().numpy()
        assert np.array_equal(y.astype(np.float64), oracle.mv(A, x)[0]), f"P5 {R}x{C} g{g}"


def test_rowtile_deterministic_scaling_and_negation():
    """P7: the same plan on 2^k x and -x gives exactly 2^k y and -y (fixed order)."""
    R, C = 5000, 171
    A = torch.from_numpy(synth.matrix(R, C, "mv", np.float32, "uniform", 51)).to(DEV)
    x = torch.from_numpy(synth.vector(C, np.float32, "uniform", 52)).to(DEV)
    p = rt_params(8)
    y = adaptic.mv(A, x, variant="MV_SUBWARP", params=p)
    assert torch.equal(adaptic.mv(A, x * 8, variant="MV_SUBWARP", params=p), y * 8)
    assert torch.equal(adaptic.mv(A, -x, variant="MV_SUBWARP", params=p), -y)
    assert torch.equal(adaptic.mv(A, x, variant="MV_SUBWARP", params=p), y)


def test_rowtile_unaligned_bases_fall_back():
    """A (or DOT's b) not 16-byte aligned: the variant's direct kernel, same results."""
    for R, C, off in [(31, 37, 1), (640, 101, 2), (9, 500, 3), (1000, 16, 1)]:
        A = synth.matrix(R, C, "mv", np.float32, "uniform", 5 + C)
        x = synth.vector(C, np.float32, "uniform", 6 + C)
        big = torch.zeros(R * C + 8, dtype=torch.float32, device=DEV)
        big[off:off + R * C] = torch.from_numpy(A.reshape(-1)).to(DEV)
        Ad = big[off:off + R * C].view(R, C)
        for v, g in (("MV_SUBWARP", 4), ("MV_WPR", 32)):
            p = rt_params(g)
            try:
                adaptic.plan("mv", R, C, "f32", variant=v, params=p)
            except adaptic.AdapticError:
                continue
            y = adaptic.mv(Ad, torch.from_numpy(x).to(DEV), variant=v, params=p).cpu().numpy()
            check(y, oracle.mv(A, x), "f32", f"off {off} {R}x{C} {v}")
    R, C = 333, 129
    a = synth.matrix(R, C, "mv", np.int32, "uniform", 71)
    b = synth.matrix(R, C, "mv", np.int32, "uniform", 72)
    bb = torch.zeros(R * C + 4, dtype=torch.int32, device=DEV)
    bb[1:1 + R * C] = torch.from_numpy(b.reshape(-1)).to(DEV)
    y = adaptic.dot(torch.from_numpy(a).to(DEV), bb[1:1 + R * C].view(R, C), variant="MV_SUBWARP",
                    params=rt_params(8)).cpu().numpy()
    check(y, oracle.dot(a, b), "i32", "dot b off by 4 bytes")


def test_rowtile_large_held_out_shape_sampled():
    """A 256 MiB held-out shape at full size in the bench's configuration (AUTO and the
    forced staged plan): sampled rows against the oracle row by row."""
    R, C = 262144, 257
    A = torch.empty(R * C, dtype=torch.float32, device=DEV)
    synth.device_matrix(A, R, C, "mv", "uniform", 61)
    x = torch.empty(C, dtype=torch.float32, device=DEV)
    synth.device_vector(x, "uniform", 62)
    xs = x.cpu().numpy()
    rows = np.unique(np.concatenate([np.arange(0, 64), np.arange(R - 64, R),
                                     np.random.default_rng(3).integers(0, R, 256)]))
    for v, p in (("AUTO", None), ("MV_WPR", rt_params(32)), ("MV_SUBWARP", rt_params(16, 512))):
        y = adaptic.mv(A.view(R, C), x, variant=v, params=p).cpu().numpy()
        Arows = A.view(R, C)[torch.from_numpy(rows).to(DEV)].cpu().numpy()
        yr, S = oracle.mv(Arows, xs)
        err = np.abs(y[rows].astype(np.float64) - yr)
        assert np.all(err <= TOL * S), f"{v} {p}"


# ---------------------------------------------------------------- long rows, CTA-wide (XSMEM 11)
def rtc_params(nt=0, k=0, stages=0, cps=0):
    """MV_CPR [lanes, splits, ctas_per_sm, unroll(stages), xsmem=11, block, rows]"""
    return [0, 0, cps, stages, 11, nt, k]


RTC_SHAPES = [(1, 1), (1, 4097), (2, 1025), (7, 3), (8, 999), (9, 1025), (33, 2049), (100, 77), (257, 1026),
              (1000, 1027), (3, 5000), (17, 8193), (5, 16385), (4096, 1028), (12345, 129), (3, 20903), (2, 40001)]
RTC_PLANS = [rtc_params()] + [rtc_params(nt, k, st, cps) for nt, k, st, cps in
                              ((512, 0, 0, 0), (256, 1, 2, 0), (256, 8, 3, 2), (512, 3, 8, 1), (256, 5, 0, 2))]


@pytest.mark.parametrize("dt", ["f32", "i32"])
def test_rowtile_cta_long_rows(dt):
    """mv_rowtile_cta_kernel: k <= 8 whole rows per bulk copy reduced by the whole CTA, x in
    registers (4..36 values per thread), the transposing butterfly; every C % 4 phase, tiles of 1..8 rows, ragged last tiles, the matrix's
    last < 4 words copied by the threads, 256/512 threads, 2..8 stages."""
    npdt = np.float32 if dt == "f32" else np.int32

    def case(R, C, p):
        A = synth.matrix(R, C, "mv", npdt, "uniform", synth.seed(23, "A") + R + C)
        x = synth.vector(C, npdt, "uniform", synth.seed(23, "x") + C)
        d = adaptic.plan("mv", R, C, dt, variant="MV_CPR", params=p).describe()
        if C > 36 * (p[5] or 512):
            # x lives in registers (C <= 36 columns per thread): longer rows take the direct
            # CTA-per-row kernel, 256 lanes x 2 vectors (shifted x copies when C % 4 != 0)
            assert d["xmode"] != 11 and d["lanes"] == 256 and d["unroll"] == 2, d
        else:
            assert d["xmode"] == 11 and d["stages"] >= 2 and 1 <= d["rows_per_group"] <= 8, d
        y = adaptic.mv(torch.from_numpy(A).to(DEV), torch.from_numpy(x).to(DEV), variant="MV_CPR", params=p)
        check(y.cpu().numpy(), oracle.mv(A, x), dt, f"mv {dt} {R}x{C} {p}")
    _collect([(f"{R}x{C} {p}", lambda R=R, C=C, p=p: case(R, C, p))
              for (R, C), p in itertools.product(RTC_SHAPES, RTC_PLANS)])


def test_rowtile_cta_exact_deterministic_and_unaligned():
    """P5 exact on integer-valued fp32; P7 scaling / negation / rerun identity; an A that is
    not 16-byte aligned takes MV_CPR's direct kernel with the same results."""
    for R, C in [(4099, 1025), (333, 4097), (65, 8193)]:
        A = synth.matrix(R, C, "mv", np.float32, "smallint", 91 + C)
        x = synth.vector(C, np.float32, "smallint", 92 + C)
        y = adaptic.mv(torch.from_numpy(A).to(DEV), torch.from_numpy(x).to(DEV), variant="MV_CPR",
                       params=rtc_params()).cpu().numpy()
        assert np.array_equal(y.astype(np.float64), oracle.mv(A, x)[0]), f"P5 {R}x{C}"
    R, C = 3001, 1025
    A = torch.from_numpy(synth.matrix(R, C, "mv", np.float32, "uniform", 93)).to(DEV)
    x = torch.from_numpy(synth.vector(C, np.float32, "uniform", 94)).to(DEV)
    p = rtc_params()
    y = adaptic.mv(A, x, variant="MV_CPR", params=p)
    assert torch.equal(adaptic.mv(A, x * 8, variant="MV_CPR", params=p), y * 8)
    assert torch.equal(adaptic.mv(A, -x, variant="MV_CPR", params=p), -y)
    assert torch.equal(adaptic.mv(A, x, variant="MV_CPR", params=p), y)
    An = A.cpu().numpy()
    for off in (1, 2, 3):
        big = torch.zeros(R * C + 8, dtype=torch.float32, device=DEV)
        big[off:off + R * C] = A.reshape(-1)
        yo = adaptic.mv(big[off:off + R * C].view(R, C), x, variant="MV_CPR", params=p).cpu().numpy()
        check(yo, oracle.mv(An, x.cpu().numpy()), "f32", f"A off by {4 * off} bytes")


def test_rowtile_cta_full_size_sampled():
    """The offgrid bench shapes at 256 MiB in the bench's configuration: sampled rows."""
    for R, C in [(65536, 1025), (16384, 4097)]:
        A = torch.empty(R * C, dtype=torch.float32, device=DEV)
        synth.device_matrix(A, R, C, "mv", "uniform", 95)
        x = torch.empty(C, dtype=torch.float32, device=DEV)
        synth.device_vector(x, "uniform", 96)
        rows = np.unique(np.concatenate([np.arange(0, 32), np.arange(R - 32, R),
                                         np.random.default_rng(5).integers(0, R, 128)]))
        y = adaptic.mv(A.view(R, C), x, variant="MV_CPR", params=rtc_params()).cpu().numpy()
        Arows = A.view(R, C)[torch.from_numpy(rows).to(DEV)].cpu().numpy()
        yr, S = oracle.mv(Arows, x.cpu().numpy())
        assert np.all(np.abs(y[rows].astype(np.float64) - yr) <= TOL * S), f"{R}x{C}"


# ---------------------------------------------------------------- TMV on staged tiles of B
def trt_params(nt=0, k=0, stages=0, cps=0):
    """TMV_REGTILE [lanes, splits, ctas_per_sm, unroll(stages), xsmem=4, block, rows]"""
    return [0, 0, cps, stages, 4, nt, k]


TMV_SHAPES = [(1, 1), (1, 1000), (2, 77), (3, 100003), (5, 7), (9, 4099), (13, 1000), (63, 257), (64, 333),
              (129, 4099), (255, 100), (256, 17), (257, 999), (513, 1001), (1023, 65), (1024, 9), (4, 3), (30, 7),
              (1025, 333), (2049, 65), (4095, 17), (3000, 1001)]
TMV_PLANS = [trt_params()] + [trt_params(nt, k, st) for nt, k, st in
                              ((256, 4, 0), (512, 8, 2), (1024, 0, 3), (1024, 4, 8), (256, 64, 2), (512, 0, 0),
                               (544, 0, 0), (544, 8, 2))]


@pytest.mark.parametrize("dt", ["f32", "i32"])
def test_tmv_rowtile_shapes_and_tiles(dt):
    npdt = np.float32 if dt == "f32" else np.int32

    def case(R, C, p):
        B = synth.matrix(R, C, "tmv", npdt, "uniform", synth.seed(22, "A") + R + C)
        x = synth.vector(C, npdt, "uniform", synth.seed(22, "x") + C)
        try:
            plan = adaptic.plan("tmv", R, C, dt, variant="TMV_REGTILE", params=p)
        except adaptic.AdapticError as e:
            assert e.status in (L.ERR_UNSUPPORTED, L.ERR_INVALID_ARG), str(e)
            # forced shapes may exceed the CTA (R > threads), the ring budget (< 2 stages) or
            # the error bound (slice sums of 1024 threads for R = 1); the default plan may not
            assert p != trt_params() or R > 4096, f"unexpected {e} for {R}x{C} {p}"
            return
        assert plan.describe()["xmode"] == 4
        y = adaptic.tmv(torch.from_numpy(B).to(DEV), torch.from_numpy(x).to(DEV), variant="TMV_REGTILE", params=p)
        check(y.cpu().numpy(), oracle.tmv(B, x), dt, f"tmv {dt} {R}x{C} {p}")
    _collect([(f"{R}x{C} {p}", lambda R=R, C=C, p=p: case(R, C, p))
              for (R, C), p in itertools.product(TMV_SHAPES, TMV_PLANS)])


def test_tmv_rowtile_exact_and_deterministic():
    """P5 exact at 2^22 elements with R off the 16-byte grid; P7 scaling/negation."""
    for R in (9, 129, 513):
        C = (1 << 22) // R
        B = synth.matrix(R, C, "tmv", np.float32, "smallint", 81 + R)
        x = synth.vector(C, np.float32, "smallint", 82 + R)
        Bd, xd = torch.from_numpy(B).to(DEV), torch.from_numpy(x).to(DEV)
        y = adaptic.tmv(Bd, xd, variant="TMV_REGTILE", params=trt_params())
        assert np.array_equal(y.cpu().numpy().astype(np.float64), oracle.tmv(B, x)[0]), f"P5 {R}x{C}"
        Bu = torch.from_numpy(synth.matrix(R, C, "tmv", np.float32, "uniform", 83 + R)).to(DEV)
        yu = adaptic.tmv(Bu, xd, variant="TMV_REGTILE", params=trt_params())
        assert torch.equal(adaptic.tmv(Bu, xd * 4, variant="TMV_REGTILE", params=trt_params()), yu * 4)
        assert torch.equal(adaptic.tmv(Bu, -xd, variant="TMV_REGTILE", params=trt_params()), -yu)


def test_tmv_rowtile_unaligned_bases_fall_back():
    for R, C in [(9, 1000), (61, 333), (517, 64)]:
        B = synth.matrix(R, C, "tmv", np.float32, "uniform", 91 + R)
        x = synth.vector(C, np.float32, "uniform", 92 + C)
        for off in (1, 2, 3):
            big = torch.zeros(R * C + 8, dtype=torch.float32, device=DEV)
            big[off:off + R * C] = torch.from_numpy(B.reshape(-1)).to(DEV)
            xb = torch.zeros(C + 8, dtype=torch.float32, device=DEV)
            xb[off:off + C] = torch.from_numpy(x).to(DEV)
            for Bv, xv in ((big[off:off + R * C].view(C, R), torch.from_numpy(x).to(DEV)),
                           (torch.from_numpy(B).to(DEV), xb[off:off + C])):
                y = adaptic.tmv(Bv, xv, variant="TMV_REGTILE", params=trt_params())
                check(y.cpu().numpy(), oracle.tmv(B, x), "f32", f"tmv off {off} {R}x{C}")


def test_batch_with_exclusive_staged_plans():
    """adaptic_run_batch with staged-tile plans (>= 64 KB of dynamic shared memory per CTA;
    run alone between the other lanes' work when ADAPTIC_EXCLUSIVE=1, interleaved by default):
    results equal single runs bit for bit on 1..3 streams, staged and direct plans mixed."""
    dev = torch.device(DEV)
    stream = torch.cuda.current_stream().cuda_stream
    cases = [("mv", 20000, 257, "MV_WPR", rt_params(32)), ("mv", 512, 3000, "AUTO", None),
             ("tmv", 9, 300001, "TMV_REGTILE", trt_params()), ("dot", 7, 50000, "AUTO", None),
             ("dot", 30000, 129, "MV_SUBWARP", rt_params(16)), ("tmv", 1000, 999, "AUTO", None)]
    items, refs = [], []
    for op, R, C, v, p in cases:
        M = synth.matrix(R, C, "tmv" if op == "tmv" else "mv", np.float32, "uniform", 71 + R)
        X = (synth.matrix(R, C, "mv", np.float32, "uniform", 72 + R) if op == "dot"
             else synth.vector(C, np.float32, "uniform", 73 + C))
        Md, Xd = torch.from_numpy(M).to(dev), torch.from_numpy(X).to(dev)
        plan = adaptic.get_plan({"mv": L.OP_MV, "tmv": L.OP_TMV, "dot": L.OP_DOT}[op], R, C, L.F32, dev, v, p, stream)
        y = torch.empty(R, device=dev)
        items.append((plan, Md.data_ptr(), Xd.data_ptr(), y.data_ptr(), Md, Xd, y))
        plan.run(Md.data_ptr(), Xd.data_ptr(), y.data_ptr(), stream)
        refs.append(y.clone())
    assert any(it[0].describe()["smem"] >= 64 * 1024 for it in items)
    for k in (1, 2, 3):
        for it in items:
            it[6].fill_(float("nan"))
        L.Batch([it[:4] for it in items]).run(k, stream)
        for it, ref in zip(items, refs):
            assert torch.equal(it[6], ref), k
