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
