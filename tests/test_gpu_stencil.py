"""Five-point stencil (the paper's neighbouring-access actor with input-adaptive super
tiles, Sec. 4.1.2; reading R19) against the oracle -- needs a GPU.

|v - v_ref| <= 1e-6 * S per point (S = |c u| + |n| sum |neighbours|; the kernel does five
fp32 roundings, gamma_5 < 3.1e-7); edge points are copies, compared exactly."""
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
C0, N0 = 0.6, 0.1


def check(v, u, c, n, what):
    ref, S = oracle.stencil5(u, c, n)
    err = np.abs(v.astype(np.float64) - ref)
    bad = ~(err <= 1e-6 * S)
    assert not bad.any(), f"{what}: {bad.sum()} points out of tolerance, first {np.argwhere(bad)[:3].tolist()}"
    edge = np.zeros(u.shape, bool)
    edge[0, :] = edge[-1, :] = True
    edge[:, 0] = edge[:, -1] = True
    assert np.array_equal(v[edge], u[edge]), f"{what}: edge not copied"


def _collect(cases):
    fails = []
    for what, fn in cases:
        try:
            fn()
        except Exception as e:  # noqa: BLE001 -- report every failing case at once
            fails.append(f"{what}: {type(e).__name__}: {str(e)[:200]}")
    assert not fails, f"{len(fails)} failures:\n" + "\n".join(fails[:40])


SHAPES = [(1, 4), (2, 8), (3, 3), (5, 12), (33, 100), (64, 256), (65, 260), (129, 1000), (300, 516), (1000, 64),
          (7, 4096), (2049, 132), (5, 8200), (9, 16384), (1, 8192)]
FORCED = [("AUTO", None), ("ST_DIRECT", None), ("ST_DIRECT", [0, 0, 0, 0, 0, 0, 0, 1]),
          ("ST_DIRECT", [0, 0, 0, 0, 0, 0, 0, 2]), ("ST_DIRECT", [0, 0, 0, 0, 0, 0, 0, 3]),
          ("ST_DIRECT", [0, 0, 0, 0, 0, 0, 3, 3]), ("ST_DIRECT", [0, 0, 0, 0, 0, 0, 9, 3]),
          ("ST_DIRECT", [0, 0, 0, 0, 0, 0, 0, 4])] + \
         [("ST_TILE", [tw, 0, 0, 0, 0, 0, th]) for th in (4, 8, 16, 32) for tw in (128, 256, 512)]


def test_every_variant_and_tile():
    def case(H, W, v, p):
        u = synth.matrix(H, W, "mv", np.float32, "uniform", 41 + H + W)
        try:
            out = adaptic.stencil5(torch.from_numpy(u).to(DEV), C0, N0, variant=v, params=p)
        except adaptic.AdapticError as e:
            assert e.status == L.ERR_UNSUPPORTED, str(e)
            return
        check(out.cpu().numpy(), u, C0, N0, f"{H}x{W} {v} {p}")
    _collect([(f"{H}x{W} {v} {p}", lambda H=H, W=W, v=v, p=p: case(H, W, v, p))
              for (H, W), (v, p) in itertools.product(SHAPES, FORCED)])


def test_odd_widths_and_misaligned_pointers_take_the_direct_kernel():
    for H, W in [(17, 33), (100, 101), (3, 7)]:
        u = synth.matrix(H, W, "mv", np.float32, "uniform", 7 + W)
        check(adaptic.stencil5(torch.from_numpy(u).to(DEV), -1.5, 0.25).cpu().numpy(), u, -1.5, 0.25, f"{H}x{W}")
    H, W = 64, 512
    u = synth.matrix(H, W, "mv", np.float32, "uniform", 9)
    big = torch.zeros(H * W + 4, device=DEV)
    big[1:1 + H * W] = torch.from_numpy(u.reshape(-1)).to(DEV)
    for v in ("AUTO", "ST_TILE", "ST_DIRECT"):
        out = adaptic.stencil5(big[1:1 + H * W].view(H, W), C0, N0, variant=v)
        check(out.cpu().numpy(), u, C0, N0, f"misaligned {v}")


def test_harmonic_field_is_reproduced():
    """c + 4n = 1 and u = i + 2j (discrete harmonic): v == u at every point (exact on
    integer-valued data: every partial sum is an exact fp32 integer)."""
    H, W = 200, 640
    i, j = np.meshgrid(np.arange(H), np.arange(W), indexing="ij")
    u = (i + 2 * j).astype(np.float32)
    for v, p in (("ST_DIRECT", None), ("ST_TILE", None), ("ST_DIRECT", [0, 0, 0, 0, 0, 0, 0, 2]),
                 ("ST_DIRECT", [0, 0, 0, 0, 0, 0, 0, 3])):
        out = adaptic.stencil5(torch.from_numpy(u).to(DEV), 0.5, 0.125, variant=v, params=p).cpu().numpy()
        assert np.array_equal(out, u), (v, p)


def test_large_grid_device_generated():
    H, W = 4096, 16384                                   # 256 MiB
    t = torch.empty(H * W, device=DEV)
    synth.device_matrix(t, H, W, "mv", "uniform", synth.seed(30, "A"))
    out = adaptic.stencil5(t.view(H, W), C0, N0)
    u = t.cpu().numpy().reshape(H, W)
    o = out.cpu().numpy()
    ref, S = oracle.stencil5(u[:64], C0, N0)
    err = np.abs(o[:64].astype(np.float64) - ref)
    assert (err[:-1] <= 1e-6 * S[:-1]).all()              # row 63 is an edge only in the slice
    ref, S = oracle.stencil5(u[-64:], C0, N0)
    err = np.abs(o[-64:].astype(np.float64) - ref)
    assert (err[1:] <= 1e-6 * S[1:]).all()                # row 0 of the slice is an edge only in the slice
    mid, S = oracle.stencil5(u[2000:2100], C0, N0)           # a band in the middle (interior rows 1..98)
    err = np.abs(o[2001:2099].astype(np.float64) - mid[1:-1])
    assert (err <= 1e-6 * S[1:-1]).all()


def test_run_host_end_to_end():
    """Host buffers through the C ABI (adaptic_run_host: H2D of u and {c, n}, kernel, D2H of v)."""
    H, W = 300, 1028
    u = synth.matrix(H, W, "mv", np.float32, "uniform", 77)
    uh = torch.from_numpy(u).pin_memory()
    ch = torch.tensor([C0, N0], dtype=torch.float32).pin_memory()
    vh = torch.empty(H, W, dtype=torch.float32).pin_memory()
    du, dc, dv = torch.empty(H, W, device=DEV), torch.empty(2, device=DEV), torch.empty(H, W, device=DEV)
    adaptic.run_host("stencil5", uh, ch, vh, du, dc, dv)
    torch.cuda.synchronize()
    check(vh.numpy(), u, C0, N0, "run_host")
