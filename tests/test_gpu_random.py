"""Randomised parity sweep (seeded, reproducible) over every op of the C ABI -- needs a GPU.

300 cases drawn from a fixed-seed generator: op, shape (log-uniform, ragged, up to ~2M
elements), dtype, forced variant or AUTO, and a base-pointer offset of 0..3 elements
(misaligned starts).  Each result is compared with the oracle exactly as the dedicated
parity tests do: int32 and integer-valued results bit-exact, fp32 within 1e-4 S_r (MV/TMV/
DOT/ASUM), one ulp (NRM2), 1e-6 S (stencil).  A forced variant may answer UNSUPPORTED or
MISALIGNED (its documented contract); AUTO must always succeed."""
import random

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
OPS = ["mv", "tmv", "dot", "asum", "nrm2", "iamax", "iamin", "stencil5"]


def on_device(a: np.ndarray, off: int) -> torch.Tensor:
    """Copy into a device buffer starting `off` elements past a 256-byte-aligned base."""
    flat = torch.zeros(a.size + off + 4, dtype=torch.from_numpy(a).dtype, device=DEV)
    flat[off:off + a.size] = torch.from_numpy(np.ascontiguousarray(a).reshape(-1)).to(DEV)
    return flat[off:off + a.size].view(a.shape)


def draw(rng: random.Random):
    op = rng.choice(OPS)
    n = 2 ** rng.uniform(0, 21)
    R = max(1, int(2 ** rng.uniform(0, np.log2(max(2, n)))))
    C = max(1, int(n / R))
    if rng.random() < 0.5:
        C += rng.randint(0, 5)
    dt = rng.choice(["f32", "i32"]) if op in ("mv", "tmv", "dot") else "f32"
    if op in ("mv", "tmv", "dot"):
        vs = ["AUTO"] + list(L.TMV_VARIANTS if op == "tmv" else L.MV_VARIANTS)
    elif op == "stencil5":
        vs = ["AUTO", "ST_DIRECT", "ST_TILE"]
    else:
        vs = ["AUTO"] + list(L.B1_VARIANTS)
    v = rng.choice(vs)
    off = rng.choice([0, 0, 0, 1, 2, 3])
    return op, R, C, dt, v, off


def run_case(op, R, C, dt, v, off, seed):
    npdt = np.int32 if dt == "i32" else np.float32
    A = synth.matrix(R, C, "tmv" if op == "tmv" else "mv", npdt, "uniform", seed)
    Ad = on_device(A, off)
    if op in ("mv", "tmv"):
        x = synth.vector(C, npdt, "uniform", seed + 1)
        y = (adaptic.mv if op == "mv" else adaptic.tmv)(Ad, on_device(x, off), variant=v).cpu().numpy()
        ref = oracle.mv(A, x) if op == "mv" else oracle.tmv(A, x)
    elif op == "dot":
        b = synth.matrix(R, C, "mv", npdt, "uniform", seed + 2)
        y = adaptic.dot(Ad, on_device(b, off), variant=v).cpu().numpy()
        ref = oracle.dot(A, b)
    elif op == "stencil5":
        y = adaptic.stencil5(Ad, 0.6, 0.1, variant=v).cpu().numpy()
        vr, S = oracle.stencil5(A, 0.6, 0.1)
        assert (np.abs(y.astype(np.float64) - vr) <= 1e-6 * S).all()
        return
    else:
        y = getattr(adaptic, op)(Ad, variant=v).cpu().numpy()
        ref = getattr(oracle, op)(A)
    if dt == "i32" or op in ("iamax", "iamin"):
        exp = ref if not isinstance(ref, tuple) else ref[0]
        assert np.array_equal(y, np.asarray(exp).astype(y.dtype)), "not bit-exact"
    elif op == "nrm2":
        r = np.asarray(ref[0], dtype=np.float64)
        assert (np.abs(y.astype(np.float64) - r) <= 2.0 ** -23 * r + 1e-45).all()
    elif op == "asum":
        r = np.asarray(ref, dtype=np.float64)
        assert (np.abs(y.astype(np.float64) - r) <= 1e-4 * r).all()
    else:
        yr, S = ref
        assert (np.abs(y.astype(np.float64) - yr) <= 1e-4 * S).all()


def test_random_parity_300_cases():
    rng = random.Random(20120611)
    fails, ran = [], 0
    for i in range(300):
        op, R, C, dt, v, off = draw(rng)
        what = f"#{i} {op} {dt} {R}x{C} {v} off={off}"
        try:
            run_case(op, R, C, dt, v, off, 1000 + i)
            ran += 1
        except adaptic.AdapticError as e:
            if v == "AUTO" or e.status not in (L.ERR_UNSUPPORTED, L.ERR_MISALIGNED):
                fails.append(f"{what}: {e}")
        except Exception as e:  # noqa: BLE001 -- report every failing case at once
            fails.append(f"{what}: {type(e).__name__}: {str(e)[:150]}")
    assert not fails, f"{len(fails)} failures:\n" + "\n".join(fails[:30])
    assert ran >= 200, ran
