"""GPU conjugate-gradient solve (tilespmv_cg) against the
oracle's CG (oracle.cg, pinned in test_oracle_cg.py)."""
import numpy as np
import pytest

from oracle import oracle as O
from synthetic import gen

pytestmark = pytest.mark.gpu


def _solve(A, b, tol, maxit, dev):
    import torch
    from paper_conf_ipps_niuldj0t21_b200 import TiledMatrix
    with TiledMatrix.from_host_csr(A, device=dev) as M:
        x, it, rel = M.cg(torch.from_numpy(b).to(dev), tol=tol, maxit=maxit)
        return x.cpu().numpy(), it, rel


@pytest.mark.parametrize("name", ["lap2d_64", "stencil27_21"])
def test_cg_matches_oracle(cuda_device, name):
    """SPD stencils (closed-form values 4/-1 and 26/-1): same iteration count
    up to the rounding at the stopping threshold, and the same solution to
    well within the stopping tolerance."""
    if name == "lap2d_64":
        A = gen.lap2d(64)
    else:
        A = gen.stencil27(21, values="stencil")
    b = gen.dense_x(A.n, 31)
    tol = 1e-11
    xo, ito, relo = O.cg(A, b, tol=tol, maxit=5000)
    xg, itg, relg = _solve(A, b, tol, 5000, cuda_device)
    assert abs(itg - ito) <= 2, (itg, ito)
    assert relg <= tol and relo <= tol
    # both iterates are within ~tol * cond(A) of the solution
    assert np.linalg.norm(xg - xo) <= 1e-7 * np.linalg.norm(xo)
    # the GPU's recursive residual agrees with a residual recomputed by the oracle
    r, _ = O.spmv(A, xg)
    true_rel = np.linalg.norm(b - r) / np.linalg.norm(b)
    assert true_rel <= 10 * tol


def test_cg_diagonal_closed_form(cuda_device):
    """3 distinct eigenvalues: converged after <= 4 steps to x = b / d."""
    n = 300
    d = np.array([1.0, 4.0, 9.0])[np.arange(n) % 3]
    A = gen.csr_from_coo(n, n, np.arange(n), np.arange(n), vals=d, name="diag3")
    b = gen.dense_x(n, 5)
    x, it, rel = _solve(A, b, 1e-12, 100, cuda_device)
    assert it <= 4 and np.allclose(x, b / d, rtol=0, atol=1e-12)


def test_cg_deterministic_and_args(cuda_device):
    import torch
    from paper_conf_ipps_niuldj0t21_b200 import TiledMatrix, TileSpMVError
    A = gen.lap2d(37, 29)
    b = torch.from_numpy(gen.dense_x(A.n, 7)).to(cuda_device)
    with TiledMatrix.from_host_csr(A, device=cuda_device) as M:
        x1, i1, _ = M.cg(b, tol=1e-9)
        x2, i2, _ = M.cg(b, tol=1e-9)
        assert i1 == i2 and torch.equal(x1, x2)
        _, i0, r0 = M.cg(b, tol=1e-9, maxit=0)
        assert i0 == 0
        with pytest.raises(TileSpMVError):
            M.cg(b, tol=-1.0)
    R = gen.random_sparse(17, 33, 0.3, seed=1)
    with TiledMatrix.from_host_csr(R, device=cuda_device) as M:
        with pytest.raises(TileSpMVError):
            M.cg(torch.zeros(33, dtype=torch.float64, device=cuda_device))


def test_cg_odd_n_and_misaligned_vectors(cuda_device):
    """Odd n (the vector kernels' pair loop plus the tail element) and b, x
    that are not 16-byte aligned (views at an odd element offset, staged
    internally): the oracle-matching solve, bitwise equal to the aligned
    call."""
    import torch
    from paper_conf_ipps_niuldj0t21_b200 import TiledMatrix
    A = gen.lap2d(37, 29)  # n = 1073
    assert A.n % 2 == 1
    b = gen.dense_x(A.n, 33)
    tol = 1e-11
    xo, ito, _ = O.cg(A, b, tol=tol, maxit=5000)
    with TiledMatrix.from_host_csr(A, device=cuda_device) as M:
        bd = torch.from_numpy(b).to(cuda_device)
        xa, ita, rela = M.cg(bd, tol=tol, maxit=5000)
        buf_b = torch.zeros(A.n + 1, dtype=torch.float64, device=cuda_device)
        buf_x = torch.zeros(A.n + 1, dtype=torch.float64, device=cuda_device)
        buf_b[1:].copy_(bd)
        xm, itm, relm = M.cg(buf_b[1:], x=buf_x[1:], tol=tol, maxit=5000)
        assert buf_b[1:].data_ptr() % 16 == 8
        xa, xm = xa.cpu().numpy(), xm.cpu().numpy()
    assert abs(ita - ito) <= 2 and relm <= tol
    assert ita == itm and np.array_equal(xa.view(np.uint64), xm.view(np.uint64))
    assert np.linalg.norm(xa - xo) <= 1e-7 * np.linalg.norm(xo)
    assert float(buf_x[0]) == 0.0  # nothing written outside the view
