"""BiCGSTAB on the adaptive MV against the fp64
oracle (oracle/bicgstab.py) -- needs a GPU.

The GPU solver runs in fp32 (the paper's Sgemv/Sdot), the oracle in fp64, so the
iterates drift apart by rounding; what must agree:
  * the first iteration's scalars rho, alpha, omega (relative 1e-4);
  * the converged solution: ||x_gpu - x*|| / ||x*|| <= 1e-4 (x* = LAPACK solve; the
    synthetic systems are strictly diagonally dominant, kappa ~ 1);
  * the true residual ||b - A x_gpu|| / ||b|| within 10x the requested tolerance;
  * the iteration count within 2 of the oracle's at the same tolerance.
"""
import numpy as np
import pytest
import torch

import synth
from oracle.bicgstab import bicgstab as oracle_bicgstab

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    import paper_conf_pldi_samadihmlm12_b200 as adaptic
    from paper_conf_pldi_samadihmlm12_b200 import _lib as L

DEV = "cuda:0"


def system(n, cfg=20):
    A = synth.matrix(n, n, "mv", np.float32, "diagdom", synth.seed(cfg, "A"))
    b = synth.vector(n, np.float32, "uniform", synth.seed(cfg, "b"))
    return A, b


@pytest.mark.parametrize("n", [1, 2, 7, 64, 300, 512, 1023, 2048])
def test_solution_and_iterations_match_oracle(n):
    A, b = system(n)
    tol = 1e-5
    x, it, rel = adaptic.bicgstab(torch.from_numpy(A).to(DEV), torch.from_numpy(b).to(DEV), tol=tol, max_iters=200)
    x = x.cpu().numpy().astype(np.float64)
    A64, b64 = A.astype(np.float64), b.astype(np.float64)
    xs = np.linalg.solve(A64, b64)
    xo, ito, _ = oracle_bicgstab(A64, b64, tol=tol, max_iters=200)
    assert np.linalg.norm(x - xs) <= 1e-4 * np.linalg.norm(xs), (n, it, rel)
    assert np.linalg.norm(b64 - A64 @ x) / np.linalg.norm(b64) <= 10 * tol
    assert abs(it - ito) <= 2, (it, ito)
    assert rel < tol


def test_first_iteration_scalars():
    """One iteration on the device vs steps 1-11 of the oracle: rho, alpha, omega."""
    n = 1024
    A, b = system(n, cfg=21)
    A += np.diag(np.linspace(-200, 200, n).astype(np.float32))       # no convergence in one step
    Ad, bd = torch.from_numpy(A).to(DEV), torch.from_numpy(b).to(DEV)
    x = torch.empty(n, device=DEV)
    S = adaptic.bicgstab_solver(n, torch.device(DEV))
    stream = torch.cuda.current_stream().cuda_stream
    S.start(bd.data_ptr(), x.data_ptr(), stream)
    S.iterate(Ad.data_ptr(), x.data_ptr(), 1, 0.0, stream)
    it, rel, done = S.state(stream)
    xo, ito, hist = oracle_bicgstab(A.astype(np.float64), b.astype(np.float64), tol=0.0, max_iters=1)
    assert it == 1 and done == 0
    assert abs(rel - hist[0]["relres"]) <= 1e-4 * hist[0]["relres"]
    xg = x.cpu().numpy().astype(np.float64)
    assert np.linalg.norm(xg - xo) <= 1e-4 * np.linalg.norm(xo)


def test_identity_converges_in_one_step_and_freezes():
    """A = I: alpha = 1, s = 0 -> done at step 7 with x = b; further iterations leave x."""
    n = 777
    b = synth.vector(n, np.float32, "uniform", 5)
    Ad = torch.eye(n, device=DEV)
    bd = torch.from_numpy(b).to(DEV)
    x, it, rel = adaptic.bicgstab(Ad, bd, tol=1e-6, max_iters=10, check_every=5)
    assert it == 1 and rel == 0.0
    assert np.array_equal(x.cpu().numpy(), b)


def test_zero_rhs_and_errors():
    n = 64
    A, _ = system(n)
    x, it, rel = adaptic.bicgstab(torch.from_numpy(A).to(DEV), torch.zeros(n, device=DEV))
    assert it == 0 and torch.count_nonzero(x).item() == 0
    with pytest.raises(adaptic.AdapticError) as e:
        L.BiCGSTAB(0)
    assert e.value.status == L.ERR_INVALID_ARG
    with pytest.raises(adaptic.AdapticError) as e:
        L.BiCGSTAB(1 << 20)
    assert e.value.status == L.ERR_UNSUPPORTED


def test_paper_sizes_8192_device_generated():
    """Fig. 11's largest system, 8192 x 8192 (256 MiB), generated on the device."""
    n = 8192
    Ad = torch.empty(n * n, dtype=torch.float32, device=DEV)
    synth.device_matrix(Ad, n, n, "mv", "diagdom", synth.seed(22, "A"))
    b = synth.vector(n, np.float32, "uniform", synth.seed(22, "b"))
    x, it, rel = adaptic.bicgstab(Ad.view(n, n), torch.from_numpy(b).to(DEV), tol=1e-5, max_iters=100)
    A64 = Ad.view(n, n).cpu().numpy().astype(np.float64)
    xg = x.cpu().numpy().astype(np.float64)
    assert np.linalg.norm(b - A64 @ xg) / np.linalg.norm(b) <= 1e-4
    xo, ito, _ = oracle_bicgstab(A64, b.astype(np.float64), tol=1e-5, max_iters=100)
    assert abs(it - ito) <= 2 and np.linalg.norm(xg - xo) <= 1e-4 * np.linalg.norm(xo)


def convection_diffusion(m: int, beta: float) -> np.ndarray:
    """The classic nonsymmetric BiCGSTAB test system (van der Vorst 1992): -Δu + β ∂u/∂x on
    an m x m interior grid, 5-point Laplacian, central convection differences, Dirichlet
    boundary; n = m^2, scaled by h^2 (diagonal 4).  kappa ~ 10^3 at m = 64 (computed in the
    test), so the method needs tens to hundreds of iterations -- unlike the diagonally
    dominant `diagdom` systems above (kappa ~ 1, two iterations)."""
    n, h = m * m, 1.0 / (m + 1)
    A = np.zeros((n, n), dtype=np.float32)
    i, j = np.divmod(np.arange(n), m)
    k = np.arange(n)
    A[k, k] = 4.0
    for di, dj, w in ((1, 0, -1.0 + beta * h / 2), (-1, 0, -1.0 - beta * h / 2), (0, 1, -1.0), (0, -1, -1.0)):
        ii, jj = i + di, j + dj
        ok = (ii >= 0) & (ii < m) & (jj >= 0) & (jj < m)
        A[k[ok], (ii * m + jj)[ok]] = w
    return A


@pytest.mark.parametrize("m,beta,tol,count", [(64, 5.0, 1e-3, True), (64, 5.0, 1e-4, True), (64, 20.0, 1e-4, True),
                                              (64, 5.0, 1e-5, False), (64, 20.0, 1e-5, False)])
def test_ill_conditioned_nonsymmetric_system(m, beta, tol, count):
    """P:1252-1304 (nonsymmetric systems): a kappa ~ 10^3 system that needs >= 30 iterations.
    fp32 iterates vs the fp64 oracle (reading R18): convergence with the true residual within
    10 x tol, and the first 8 iterations' residual history within 1e-3 relative (step-by-step
    agreement before fp32 drift).  The iteration count must be within max(3, 15 %) of the
    oracle's only while tol is above fp32's attainable accuracy on this system (tol >= 1e-4):
    near kappa * u32 ~ 1e-5..1e-4 the fp32 recurrence is driven by rounding (measured: 103
    GPU vs 80 oracle iterations for 1e-5 at beta = 20), so there only convergence is checked."""
    A = convection_diffusion(m, beta)
    n = m * m
    b = synth.vector(n, np.float32, "uniform", synth.seed(23, "b"))
    A64, b64 = A.astype(np.float64), b.astype(np.float64)
    assert np.linalg.cond(A64) > 500 and not np.allclose(A64, A64.T)
    xo, ito, hist = oracle_bicgstab(A64, b64, tol=tol, max_iters=2000)
    assert ito >= 30
    Ad, bd = torch.from_numpy(A).to(DEV), torch.from_numpy(b).to(DEV)
    x, it, rel = adaptic.bicgstab(Ad, bd, tol=tol, max_iters=2000, check_every=4)
    xg = x.cpu().numpy().astype(np.float64)
    assert rel < tol
    assert np.linalg.norm(b64 - A64 @ xg) / np.linalg.norm(b64) <= 10 * tol
    if count:
        assert abs(it - ito) <= max(3, 0.15 * ito), (it, ito)
    # step-by-step: one iteration at a time, the recurrence residual after each
    xs = torch.empty(n, device=DEV)
    S = adaptic.bicgstab_solver(n, torch.device(DEV))
    stream = torch.cuda.current_stream().cuda_stream
    S.start(bd.data_ptr(), xs.data_ptr(), stream)
    for k in range(8):
        S.iterate(Ad.data_ptr(), xs.data_ptr(), 1, 0.0, stream)
        itk, relk, done = S.state(stream)
        assert itk == k + 1 and not done
        assert abs(relk - hist[k]["relres"]) <= 1e-3 * hist[k]["relres"], (k, relk, hist[k]["relres"])


def test_out_is_validated_and_solvers_are_per_stream():
    """`out` is checked (dtype, device, shape, no overlap with A or b), and two
    streams get two solvers (their vectors and state would race otherwise)."""
    n = 256
    A, b = system(n)
    Ad, bd = torch.from_numpy(A).to(DEV), torch.from_numpy(b).to(DEV)
    for out in (torch.empty(n, dtype=torch.float64, device=DEV), torch.empty(n + 1, device=DEV), bd,
                Ad.view(-1)[:n]):
        with pytest.raises(ValueError):
            adaptic.bicgstab(Ad, bd, out=out)
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    assert adaptic.bicgstab_solver(n, torch.device(DEV), s1.cuda_stream) is not \
        adaptic.bicgstab_solver(n, torch.device(DEV), s2.cuda_stream)
    xs = []
    for s in (s1, s2):
        with torch.cuda.stream(s):
            xs.append(adaptic.bicgstab(Ad, bd, tol=1e-6)[0])
    torch.cuda.synchronize()
    assert torch.equal(xs[0], xs[1])
