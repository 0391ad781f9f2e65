"""Parity of the CUDA path (through the C ABI) against the CPU oracle -- needs a GPU.

fp32: |y_gpu - y_oracle| <= 1e-4 * S_r, S_r = sum_c |a(r,c) x_c| (north_star);
int32 and integer-valued fp32 data (P5): bit-exact.
"""
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

SIZES = [1, 2, 3, 4, 5, 7, 8, 9, 15, 16, 17, 31, 32, 33, 63, 64, 65, 127, 128, 129,
         255, 256, 257, 1023, 1024, 1025]
SIZES_SMALL = [1, 3, 4, 5, 8, 17, 32, 33, 64, 129, 256, 257, 1025]
OPS = ("mv", "tmv", "dot")
NPDT = {"f32": np.float32, "i32": np.int32}


def variants_for(op):
    return ("AUTO",) + (adaptic.TMV_VARIANTS if op == "tmv" else adaptic.MV_VARIANTS)


def make_inputs(op, R, C, dt, kind="uniform", xkind=None, cfg=0):
    """Host arrays (numpy, from synth) in the op's layout."""
    np_dt = NPDT[dt]
    xkind = xkind or (kind if kind in synth.VECTOR_KINDS else "uniform")
    if op == "dot":
        a = synth.matrix(R, C, "mv", np_dt, kind, synth.seed(cfg, "A"))
        b = synth.matrix(R, C, "mv", np_dt, xkind if xkind in synth.KINDS else "uniform", synth.seed(cfg, "b"))
        return a, b
    M = synth.matrix(R, C, "tmv" if op == "tmv" else "mv", np_dt, kind, synth.seed(cfg, "A"))
    x = synth.vector(C, np_dt, xkind, synth.seed(cfg, "x"))
    return M, x


def run_oracle(op, M, X):
    return {"mv": oracle.mv, "tmv": oracle.tmv, "dot": oracle.dot}[op](M, X)


def run_gpu(op, M, X, variant="AUTO", params=None):
    Md = torch.from_numpy(np.ascontiguousarray(M)).to(DEV)
    Xd = torch.from_numpy(np.ascontiguousarray(X)).to(DEV)
    fn = {"mv": adaptic.mv, "tmv": adaptic.tmv, "dot": adaptic.dot}[op]
    y = fn(Md, Xd, variant=variant, params=params)
    return y.cpu().numpy()


def check(y, ref, dt, what=""):
    if dt == "i32":
        assert np.array_equal(y, ref), f"{what}: int32 mismatch at {np.nonzero(y != ref)[0][:8]}"
    else:
        yr, S = ref
        err = np.abs(y.astype(np.float64) - yr)
        bad = ~(err <= TOL * S)
        assert not bad.any(), f"{what}: {bad.sum()} outputs out of tolerance, worst {np.max(err - TOL * S)}"


def try_plan_ok(op, R, C, dt, v):
    try:
        adaptic.plan(op, R, C, dt, variant=v)
        return True
    except adaptic.AdapticError as e:
        assert e.status == L.ERR_UNSUPPORTED
        return False


# ------------------------------------------------------------------------ generator twin
@pytest.mark.parametrize("kind", synth.KINDS)
@pytest.mark.parametrize("layout", ["mv", "tmv"])
def test_device_generator_matches_numpy(kind, layout):
    for dt in ("f32", "i32"):
        if kind == "rowscale" and dt == "i32":
            continue
        R, C = 37, 129
        ref = synth.matrix(R, C, layout, NPDT[dt], kind, 12345, rows=(3, 30), cols=(5, 120))
        t = torch.empty(ref.size, dtype=torch.float32 if dt == "f32" else torch.int32, device=DEV)
        synth.device_matrix(t, R, C, layout, kind, 12345, rows=(3, 30), cols=(5, 120))
        assert np.array_equal(t.cpu().numpy().reshape(ref.shape), ref)
        if kind in synth.VECTOR_KINDS:
            v = synth.vector(1000, NPDT[dt], kind, 999, start=77)
            tv = torch.empty(1000, dtype=t.dtype, device=DEV)
            synth.device_vector(tv, kind, 999, start=77)
            assert np.array_equal(tv.cpu().numpy(), v)


# ------------------------------------------------------------------------ brute force (P11)
def _collect(cases):
    """Run every case, report all failures at once (a GPU call is precious)."""
    fails = []
    for what, fn in cases:
        try:
            fn()
        except (AssertionError, Exception) as e:  # noqa: B014
            fails.append(f"{what}: {type(e).__name__}: {str(e)[:200]}")
    assert not fails, f"{len(fails)} failures:\n" + "\n".join(fails[:40])


@pytest.mark.parametrize("op", OPS)
@pytest.mark.parametrize("dt", ["f32", "i32"])
def test_bruteforce_auto_all_sizes(op, dt):
    def case(R, C):
        M, X = make_inputs(op, R, C, dt)
        check(run_gpu(op, M, X), run_oracle(op, M, X), dt, f"{op} {dt} {R}x{C} AUTO")
    _collect([(f"{R}x{C}", lambda R=R, C=C: case(R, C)) for R, C in itertools.product(SIZES, SIZES)])


@pytest.mark.parametrize("op", OPS)
@pytest.mark.parametrize("dt", ["f32", "i32"])
def test_bruteforce_every_forced_variant(op, dt):
    def case(v, R, C):
        M, X = make_inputs(op, R, C, dt)
        check(run_gpu(op, M, X, v), run_oracle(op, M, X), dt, f"{op} {dt} {R}x{C} {v}")
    _collect([(f"{v} {R}x{C}", lambda v=v, R=R, C=C: case(v, R, C))
              for v in variants_for(op)[1:] for R, C in itertools.product(SIZES_SMALL, SIZES_SMALL)
              if try_plan_ok(op, R, C, dt, v)])


@pytest.mark.parametrize("op", ["mv", "tmv"])
def test_variant_parameter_grid(op):
    """Every compiled lane/unroll instance on ragged shapes (several tiles + tail)."""
    dt = "f32"
    shapes = [(1000, 333), (77, 4100), (4099, 36)]
    if op == "mv":
        grid = [("MV_SUBWARP", [g, 0, 0, u]) for g in (1, 2, 4, 8, 16) for u in (1, 2, 4, 8)]
        grid += [("MV_WPR", [0, 0, 0, u]) for u in (1, 2, 4, 8)]
        rbu = [(1, 2), (1, 4), (1, 8), (2, 2), (2, 4), (4, 2)]
        grid += [("MV_CPR", [nt, 0, 0, u, xs, 0, rb, 0, pp]) for nt in (256, 1024) for rb, u in rbu
                 for xs in (1, 2) for pp in (1, 2)]
        grid += [("MV_SPLIT", [nt, s, 0, u, 0, 0, rb, order, pp]) for nt in (256, 1024) for s in (2, 7)
                 for rb, u in rbu for order in (1, 2) for pp in (1, 2)]
        grid += [("MV_TPR", [nt, 0, 0, st]) for nt in (128, 256) for st in (2, 3)]
    else:
        grid = [("TMV_SPLITK", [lr, s, 0, u, 0, nt]) for lr in (1, 2, 4, 8, 16, 32, 64, 128, 256)
                for s in (1, 5) for u in (2, 4, 8) for nt in (256, 1024)]
    cache = {}

    def case(R, C, v, params, dti):
        if (R, C, dti) not in cache:
            M, X = make_inputs(op, R, C, dti)
            cache[(R, C, dti)] = (M, X, run_oracle(op, M, X))
        M, X, ref = cache[(R, C, dti)]
        check(run_gpu(op, M, X, v, params), ref, dti, f"{op} {R}x{C} {v} {params}")

    cases = []
    for (R, C), (v, params) in itertools.product(shapes, grid):
        for dti in ("f32", "i32"):
            try:
                adaptic.plan(op, R, C, dti, variant=v, params=params)
            except adaptic.AdapticError:
                continue
            cases.append((f"{v} {params} {R}x{C} {dti}", lambda a=(R, C, v, params, dti): case(*a)))
    _collect(cases)


# ------------------------------------------------------------------------ closed forms
@pytest.mark.parametrize("op", OPS)
def test_P1_ones_bit_exact(op):
    for R, C in [(1, 1 << 24), (3, 1 << 20), (1 << 16, 64), (257, 4097)]:
        for v in variants_for(op):
            if not try_plan_ok(op, R, C, "f32", v):
                continue
            for dt in ("f32", "i32"):
                M, X = make_inputs(op, R, C, dt, kind="ones")
                y = run_gpu(op, M, X, v)
                assert np.all(y == C), (op, R, C, v, dt)


@pytest.mark.parametrize("op", ["mv", "tmv"])
def test_P2_identity_and_perm(op):
    for n in (1, 5, 64, 1000):
        x = synth.vector(n, np.float32, "uniform", 3)
        for kind, expect in (("identity", x), ("perm", x[::-1])):
            M = synth.matrix(n, n, op, np.float32, kind, 0)
            for v in variants_for(op):
                if try_plan_ok(op, n, n, "f32", v):
                    assert np.array_equal(run_gpu(op, M, x, v), expect), (op, n, kind, v)


def test_P3_diagonal_single_rounding():
    n = 777
    D = synth.matrix(n, n, "mv", np.float32, "diag", 5)
    x = synth.vector(n, np.float32, "uniform", 6)
    expect = (np.diag(D).astype(np.float64) * x.astype(np.float64)).astype(np.float32)
    for op in ("mv", "tmv"):
        M = D if op == "mv" else np.ascontiguousarray(D.T)
        for v in variants_for(op):
            if try_plan_ok(op, n, n, "f32", v):
                assert np.array_equal(run_gpu(op, M, x, v), expect), (op, v)


@pytest.mark.parametrize("op", OPS)
@pytest.mark.parametrize("kind", ["smallint", "smallint4"])
def test_P5_integer_valued_fp32_exact_every_variant(op, kind):
    for R, C in [(3, 100000), (1000, 1000), (20000, 12)]:
        M, X = make_inputs(op, R, C, "f32", kind=kind)
        yref, _ = run_oracle(op, M, X)
        for v in variants_for(op):
            if try_plan_ok(op, R, C, "f32", v):
                assert np.array_equal(run_gpu(op, M, X, v).astype(np.float64), yref), (op, R, C, v)


def test_P6_tmv_equals_mv_of_transpose():
    for R, C in [(100, 300), (4096, 64), (16, 50000)]:
        for dt in ("f32", "i32"):
            A, x = make_inputs("mv", R, C, dt)
            B = np.ascontiguousarray(A.T)
            ym, yt = run_gpu("mv", A, x), run_gpu("tmv", B, x)
            if dt == "i32":
                assert np.array_equal(ym, yt)
            else:
                ref = oracle.mv(A, x)
                check(ym, ref, dt)
                check(yt, ref, dt)
            ks, _ = make_inputs("mv", R, C, "f32", kind="smallint")
            xs = synth.vector(C, np.float32, "smallint", 9)
            assert np.array_equal(run_gpu("mv", ks, xs), run_gpu("tmv", np.ascontiguousarray(ks.T), xs))


@pytest.mark.parametrize("op", OPS)
def test_P7_scaling_and_negation_same_plan(op):
    R, C = 300, 5000
    M, X = make_inputs(op, R, C, "f32")
    for v in variants_for(op):
        if not try_plan_ok(op, R, C, "f32", v):
            continue
        y = run_gpu(op, M, X, v)
        assert np.array_equal(run_gpu(op, M, (X * np.float32(8)).astype(np.float32), v), y * np.float32(8))
        assert np.array_equal(run_gpu(op, M, -X, v), -y)
        assert np.array_equal(run_gpu(op, M, X, v), y)          # deterministic across runs


def test_P8_P9_linearity_and_column_split_int32():
    R, C, k = 500, 3000, 1234
    A, x = make_inputs("mv", R, C, "i32")
    z = synth.vector(C, np.int32, "uniform", 77)
    y = run_gpu("mv", A, x).astype(np.uint32)
    yz = run_gpu("mv", A, z).astype(np.uint32)
    w = (3 * x.astype(np.int64) - 5 * z.astype(np.int64)).astype(np.int32)
    assert np.array_equal(run_gpu("mv", A, w).astype(np.uint32), (np.uint32(3) * y - np.uint32(5) * yz))
    left = run_gpu("mv", np.ascontiguousarray(A[:, :k]), x[:k]).astype(np.uint32)
    right = run_gpu("mv", np.ascontiguousarray(A[:, k:]), x[k:]).astype(np.uint32)
    assert np.array_equal(left + right, y)


def test_rowscale_relative_tolerance():
    for op in ("mv", "tmv"):
        R, C = 410, 2048
        M = synth.matrix(R, C, op, np.float32, "rowscale", 4)
        x = synth.vector(C, np.float32, "uniform", 5)
        for v in variants_for(op):
            if try_plan_ok(op, R, C, "f32", v):
                check(run_gpu(op, M, x, v), run_oracle(op, M, x), "f32", f"rowscale {op} {v}")


def test_positive_data_long_rows_tolerance():
    """P14 stress: U[0,1) data, where a long serial fp32 chain would fail."""
    for op, R, C in (("mv", 2, 1 << 22), ("tmv", 8, 1 << 21), ("dot", 1, 1 << 23)):
        M, X = make_inputs(op, R, C, "f32", kind="positive")
        for v in variants_for(op):
            if try_plan_ok(op, R, C, "f32", v):
                check(run_gpu(op, M, X, v), run_oracle(op, M, X), "f32", f"positive {op} {v}")


# ------------------------------------------------------------------------ edge cases
def test_nan_propagates_to_its_row_only():
    for op in ("mv", "tmv"):
        R, C = 64, 700
        M, x = make_inputs(op, R, C, "f32")
        if op == "mv":
            M[10, 33] = np.nan
        else:
            M[33, 10] = np.nan
        for v in variants_for(op):
            if try_plan_ok(op, R, C, "f32", v):
                y = run_gpu(op, M, x, v)
                assert np.isnan(y[10]) and not np.isnan(np.delete(y, 10)).any(), (op, v)


def test_degenerate_shapes():
    for op in OPS:
        M, X = make_inputs(op, 0, 7, "f32")
        assert run_gpu(op, M, X).shape == (0,)
    y = adaptic.mv(torch.zeros(5, 0, device=DEV), torch.zeros(0, device=DEV))
    assert torch.equal(y.cpu(), torch.zeros(5))
    y = adaptic.tmv(torch.zeros(0, 6, device=DEV, dtype=torch.int32), torch.zeros(0, device=DEV, dtype=torch.int32))
    assert torch.equal(y.cpu(), torch.zeros(6, dtype=torch.int32))


def test_misaligned_pointers_take_scalar_path():
    R, C = 300, 512
    A, x = make_inputs("mv", R, C, "f32")
    ref = oracle.mv(A, x)
    big = torch.zeros(R * C + 1, device=DEV)
    big[1:] = torch.from_numpy(A.ravel()).to(DEV)
    Ad = big[1:].view(R, C)                                     # 4-byte aligned, not 16
    assert Ad.data_ptr() % 16 != 0
    xd = torch.from_numpy(x).to(DEV)
    for v in variants_for("mv"):
        if try_plan_ok("mv", R, C, "f32", v):
            check(adaptic.mv(Ad, xd, variant=v).cpu().numpy(), ref, "f32", f"misaligned {v}")
    B = np.ascontiguousarray(A.T)
    bigB = torch.zeros(R * C + 1, device=DEV)
    bigB[1:] = torch.from_numpy(B.ravel()).to(DEV)
    for v in variants_for("tmv"):
        if try_plan_ok("tmv", R, C, "f32", v):
            check(adaptic.tmv(bigB[1:].view(C, R), xd, variant=v).cpu().numpy(), ref, "f32", f"misaligned {v}")


def test_error_statuses_on_device():
    A = torch.zeros(64, 64, device=DEV)
    x = torch.zeros(64, device=DEV)
    p = adaptic.plan("mv", 64, 64)
    assert p.run_ptrs(A.data_ptr(), x.data_ptr(), A.data_ptr() + 256) == L.ERR_ALIAS
    assert p.run_ptrs(A.data_ptr() + 2, x.data_ptr(), torch.empty(64, device=DEV).data_ptr()) == L.ERR_MISALIGNED
    with pytest.raises(ValueError):
        adaptic.mv(A.cpu(), x.cpu())                            # no CPU path
    with pytest.raises(TypeError):
        adaptic.mv(A.double(), x.double())


def test_workspace_stays_zero_and_reruns_are_identical():
    R, C = 16, 1 << 20
    A, x = make_inputs("mv", R, C, "f32")
    Ad, xd = torch.from_numpy(A).to(DEV), torch.from_numpy(x).to(DEV)
    stream = torch.cuda.current_stream().cuda_stream
    plan = adaptic.get_plan(L.OP_MV, R, C, L.F32, torch.device(DEV), "MV_SPLIT", None, stream)
    assert plan.workspace_bytes > 0
    ys = [adaptic.mv(Ad, xd, variant="MV_SPLIT").cpu().numpy() for _ in range(20)]
    for y in ys[1:]:
        assert np.array_equal(y, ys[0])
    check(ys[0], oracle.mv(A, x), "f32")
    ws = adaptic.ops._cache[(L.OP_MV, R, C, L.F32, "MV_SPLIT", None, 0, stream, 1)][1]
    cnt_off = plan.describe()["workspace_bytes"] - R * 4
    assert int(ws[cnt_off:].sum().item()) == 0                  # tickets re-armed


def test_run_host_end_to_end():
    for op, R, C in (("mv", 1000, 513), ("tmv", 1000, 513), ("dot", 7, 10000)):
        M, X = make_inputs(op, R, C, "f32")
        Mh = torch.from_numpy(M).pin_memory()
        Xh = torch.from_numpy(X).pin_memory()
        yh = torch.empty(R, dtype=torch.float32).pin_memory()
        dM, dX = torch.empty_like(Mh, device=DEV), torch.empty_like(Xh, device=DEV)
        dy = torch.empty(R, device=DEV)
        adaptic.run_host(op, Mh, Xh, yh, dM, dX, dy)
        torch.cuda.synchronize()
        check(yh.numpy(), run_oracle(op, M, X), "f32", f"run_host {op}")


# ------------------------------------------------------------------------ BASELINE configs
def test_config0_tmv_256():
    M, x = make_inputs("tmv", 256, 256, "f32", cfg=0)
    check(run_gpu("tmv", M, x), oracle.tmv(M, x), "f32", "config0")
    for kind in ("ones", "identity"):
        M, x = make_inputs("tmv", 256, 256, "f32", kind=kind, cfg=0)
        assert np.array_equal(run_gpu("tmv", M, x).astype(np.float64), oracle.tmv(M, x)[0])


def _device_problem(op, R, C, dt, kind="uniform", cfg=1):
    tdt = torch.float32 if dt == "f32" else torch.int32
    M = torch.empty(R * C, dtype=tdt, device=DEV)
    synth.device_matrix(M, R, C, "tmv" if op == "tmv" else "mv", kind, synth.seed(cfg, "A"))
    x = torch.empty(C, dtype=tdt, device=DEV)
    synth.device_vector(x, kind if kind in synth.VECTOR_KINDS else "uniform", synth.seed(cfg, "x"))
    return M, x


def _sample_rows(R, n=48):
    rng = np.random.default_rng(R)
    idx = set(rng.integers(0, R, size=min(n, R)).tolist()) | {0, R - 1, R // 2}
    return np.array(sorted(idx), dtype=np.int64)


@pytest.mark.parametrize("k", range(3, 24))
@pytest.mark.parametrize("op", ["mv", "tmv"])
def test_config1_sweep_256MiB_auto_and_fixed(op, k):
    R, C = 1 << k, 1 << (26 - k)
    M, x = _device_problem(op, R, C, "f32")
    idx = _sample_rows(R)
    xh = x.cpu().numpy()
    if op == "mv":
        sub = M.view(R, C)[torch.from_numpy(idx).to(DEV)].cpu().numpy()
    else:
        sub = M.view(C, R)[:, torch.from_numpy(idx).to(DEV)].t().contiguous().cpu().numpy()
    ref = oracle.mv(sub, xh)
    fn = adaptic.mv if op == "mv" else adaptic.tmv
    Mv = M.view(R, C) if op == "mv" else M.view(C, R)
    for v in variants_for(op):
        if not try_plan_ok(op, R, C, "f32", v):
            continue
        y = fn(Mv, x, variant=v)
        check(y[torch.from_numpy(idx).to(DEV)].cpu().numpy(), ref, "f32", f"config1 {op} {R}x{C} {v}")
    del M


def test_config1_sweep_int32_smallint_exact():
    for op in ("mv", "tmv"):
        for k in (3, 13, 23):
            R, C = 1 << k, 1 << (26 - k)
            M, x = _device_problem(op, R, C, "i32", kind="smallint4")
            fn = adaptic.mv if op == "mv" else adaptic.tmv
            Mv = M.view(R, C) if op == "mv" else M.view(C, R)
            y = fn(Mv, x).cpu().numpy()
            idx = _sample_rows(R)
            if op == "mv":
                sub = Mv[torch.from_numpy(idx).to(DEV)].cpu().numpy()
            else:
                sub = Mv[:, torch.from_numpy(idx).to(DEV)].t().contiguous().cpu().numpy()
            assert np.array_equal(y[idx], oracle.mv(sub, x.cpu().numpy()))


@pytest.mark.parametrize("dt", ["f32", "i32"])
def test_config2_scalar_product_lengths(dt):
    tdt = torch.float32 if dt == "f32" else torch.int32
    for k in (10, 13, 17, 20, 24, 28):
        L_ = 1 << k
        a = torch.empty(L_, dtype=tdt, device=DEV)
        b = torch.empty(L_, dtype=tdt, device=DEV)
        synth.device_matrix(a, 1, L_, "mv", "uniform", synth.seed(2, "A"))
        synth.device_matrix(b, 1, L_, "mv", "uniform", synth.seed(2, "b"))
        y = adaptic.dot(a, b).cpu().numpy()
        ref = oracle.dot(a.cpu().numpy()[None, :], b.cpu().numpy()[None, :])
        check(y, ref, dt, f"dot L=2^{k}")


@pytest.mark.parametrize("k", [29, 30])
def test_config2_fp32_longest_lengths(k):
    """configs[2]'s two longest fp32 lengths (2 and 4 GiB per operand), the ones the bench
    times beyond 2^28: every term through the plan's split/fold tree, tolerance 1e-4 * S."""
    L_ = 1 << k
    a = torch.empty(L_, dtype=torch.float32, device=DEV)
    b = torch.empty(L_, dtype=torch.float32, device=DEV)
    synth.device_matrix(a, 1, L_, "mv", "uniform", synth.seed(2, "A"))
    synth.device_matrix(b, 1, L_, "mv", "uniform", synth.seed(2, "b"))
    y = adaptic.dot(a, b).cpu().numpy()
    ah, bh = a.cpu().numpy(), b.cpu().numpy()
    del a, b
    check(y, oracle.dot(ah[None, :], bh[None, :]), "f32", f"dot L=2^{k}")


def test_config2_int32_wrap_at_2pow30():
    L_ = 1 << 30
    a = torch.empty(L_, dtype=torch.int32, device=DEV)
    b = torch.empty(L_, dtype=torch.int32, device=DEV)
    synth.device_matrix(a, 1, L_, "mv", "uniform", synth.seed(2, "A"))
    synth.device_matrix(b, 1, L_, "mv", "uniform", synth.seed(2, "b"))
    y = adaptic.dot(a, b).cpu().numpy()
    ah, bh = a.cpu().numpy(), b.cpu().numpy()
    del a, b
    assert np.array_equal(y, oracle.dot(ah[None, :], bh[None, :]))


def test_config3_mv_131072x32768_sampled():
    R, C = 131072, 32768
    M, x = _device_problem("mv", R, C, "f32", cfg=3)
    y = adaptic.mv(M.view(R, C), x)
    idx = np.array(sorted(set(_sample_rows(R, 64).tolist()) | {R // 2 - 1, R // 2, R // 4, 3 * R // 4}))
    sub = M.view(R, C)[torch.from_numpy(idx).to(DEV)].cpu().numpy()
    check(y[torch.from_numpy(idx).to(DEV)].cpu().numpy(), oracle.mv(sub, x.cpu().numpy()), "f32", "config3")


def test_config4_tmv_1024x16M_sampled():
    R, C = 1024, 1 << 24
    M, x = _device_problem("tmv", R, C, "f32", cfg=4)
    y = adaptic.tmv(M.view(C, R), x)
    idx = _sample_rows(R, 12)
    sub = M.view(C, R)[:, torch.from_numpy(idx).to(DEV)].t().contiguous().cpu().numpy()
    check(y[torch.from_numpy(idx).to(DEV)].cpu().numpy(), oracle.mv(sub, x.cpu().numpy()), "f32", "config4")


def test_run_batch_equals_single_runs():
    """adaptic_run_batch: independent problems on 1..4 concurrent streams give exactly the
    single-call results (same plans, same kernels); a plan with a workspace repeated in a
    batch stays on one stream; validation is all-or-nothing."""
    dev = torch.device(DEV)
    stream = torch.cuda.current_stream().cuda_stream
    shapes = [("mv", 8, 1 << 20), ("tmv", 1 << 16, 64), ("mv", 4096, 1001), ("tmv", 9, 100000), ("dot", 3, 1 << 18)]
    items, refs = [], []
    for op, R, C in shapes:
        M, X = make_inputs(op, R, C, "f32")
        Md, Xd = torch.from_numpy(M).to(dev), torch.from_numpy(X).to(dev)
        plan = adaptic.get_plan({"mv": L.OP_MV, "tmv": L.OP_TMV, "dot": L.OP_DOT}[op], R, C, L.F32, dev, "AUTO", None, stream)
        y = torch.full((R,), float("nan"), device=dev)
        items.append((plan, Md.data_ptr(), Xd.data_ptr(), y.data_ptr(), Md, Xd, y))
        refs.append(run_gpu(op, M, X))
    # the same split plan twice (workspace): second copy with its own output
    p0 = items[0]
    y2 = torch.full_like(p0[6], float("nan"))
    items.append((p0[0], p0[1], p0[2], y2.data_ptr(), p0[4], p0[5], y2))
    refs.append(refs[0])
    for k in (1, 2, 3, 4):
        for it in items:
            it[6].fill_(float("nan"))
        L.Batch([it[:4] for it in items]).run(k, stream)
        for it, ref in zip(items, refs):
            assert np.array_equal(it[6].cpu().numpy(), ref), k
    bad = list(items[:2]) + [(items[2][0], items[2][1], items[2][2], items[2][1])]     # y aliases A
    items[0][6].fill_(7.0)
    with pytest.raises(adaptic.AdapticError) as e:
        L.Batch([it[:4] for it in bad]).run(2, stream)
    assert e.value.status == L.ERR_ALIAS
    torch.cuda.synchronize()
    assert (items[0][6] == 7.0).all()                    # nothing was issued


def test_run_host_validates_every_buffer():
    """adaptic_run_host copies R*C, C and R elements blindly, so the binding must
    reject short, mistyped or misplaced buffers before calling it."""
    R, C = 300, 257
    M = torch.ones(R, C, dtype=torch.float32).pin_memory()
    X = torch.ones(C, dtype=torch.float32).pin_memory()
    y = torch.empty(R, dtype=torch.float32).pin_memory()
    dM = torch.empty(R * C, device=DEV)
    dX = torch.empty(C, device=DEV)
    dy = torch.empty(R, device=DEV)
    adaptic.run_host("mv", M, X, y, dM, dX, dy)
    torch.cuda.synchronize()
    assert (y == C).all()                         # P1
    bad = [
        dict(y=torch.empty(R - 1)), dict(X=torch.ones(C - 1)), dict(dy=torch.empty(R - 1, device=DEV)),
        dict(dM=torch.empty(R * C - 1, device=DEV)), dict(dX=torch.empty(C + 1, device=DEV)),
        dict(X=torch.ones(C, dtype=torch.float64)), dict(dy=torch.empty(R, dtype=torch.int32, device=DEV)),
    ]
    for over in bad:
        args = dict(M=M, X=X, y=y, dM=dM, dX=dX, dy=dy)
        args.update(over)
        with pytest.raises((ValueError, TypeError)):
            adaptic.run_host("mv", args["M"], args["X"], args["y"], args["dM"], args["dX"], args["dy"])
