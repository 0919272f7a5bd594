"""The oracle's conjugate-gradient solve (oracle.cg) pinned
to closed forms and to a library solve -- not to itself."""
import numpy as np

from oracle import oracle as O
from synthetic import gen


def test_cg_identity_one_iteration():
    """A = I: the first step is exact (alpha = 1), x = b after 1 iteration."""
    A = gen.identity(50)
    b = gen.dense_x(50, 3)
    x, it, rel = O.cg(A, b, tol=1e-14)
    assert it == 1 and np.array_equal(x, b) and rel == 0.0


def test_cg_distinct_eigenvalues_bound():
    """In exact arithmetic CG ends after at most as many steps as A has
    distinct eigenvalues: a diagonal matrix with 3 distinct values converges
    in 3 iterations (to rounding) and gives x_i = b_i / d_i."""
    n = 60
    d = np.array([1.0, 4.0, 9.0])[np.arange(n) % 3]
    A = gen.csr_from_coo(n, n, np.arange(n), np.arange(n), vals=d, name="diag3")
    b = gen.dense_x(n, 5)
    x, it, rel = O.cg(A, b, tol=1e-12)
    assert it <= 4, it
    assert np.allclose(x, b / d, rtol=0, atol=1e-12)


def test_cg_laplacian_matches_library_solve():
    """5-point Laplacian (SPD, C1 shape on a 20x20 grid): the CG solution
    agrees with numpy.linalg.solve of the dense matrix, and the reported
    relative residual is the true one."""
    A = gen.lap2d(20)
    b = gen.dense_x(A.n, 9)
    x, it, rel = O.cg(A, b, tol=1e-12, maxit=2000)
    Ad = np.zeros((A.m, A.n))
    for i in range(A.m):
        Ad[i, A.colidx[A.rowptr[i]:A.rowptr[i + 1]]] = A.val[A.rowptr[i]:A.rowptr[i + 1]]
    xs = np.linalg.solve(Ad, b)
    assert rel <= 1e-12
    assert np.linalg.norm(x - xs) <= 1e-9 * np.linalg.norm(xs)
    true_rel = np.linalg.norm(b - Ad @ x) / np.linalg.norm(b)
    assert true_rel <= 1e-11
    # CG's worst-case bound: iterations grow like sqrt(cond); for the 20x20
    # Laplacian cond ~ 178, so a few dozen to ~100 iterations
    assert 10 <= it <= 200, it


def test_cg_initial_guess_solution_returns_at_once():
    A = gen.lap2d(8)
    xs = gen.dense_x(A.n, 4)
    b, _ = O.spmv(A, xs)
    x, it, rel = O.cg(A, b, x0=xs, tol=1e-10)
    # r0 = b - A xs is zero up to the oracle's own rounding of b
    assert it <= 1 and np.allclose(x, xs, atol=1e-12)
