"""Pins for the oracle SpMV (Alg. 1) against things other
than itself: identities, closed-form stencil row sums, exact rational brute
force and integer arithmetic.  CPU only."""
from fractions import Fraction

import numpy as np
import pytest

from oracle import oracle as O
from synthetic import gen


def test_identity_exact():
    A = gen.identity(1000)
    x = gen.dense_x(1000, 5)
    y, ay = O.spmv(A, x)
    assert np.array_equal(y, x)
    assert np.array_equal(ay, np.abs(x))


def test_diagonal_exact():
    A = gen.diagonal(777)
    x = gen.dense_x(777, 6)
    y, _ = O.spmv(A, x)
    # one product per row: y_i = fl(d_i * x_i) exactly
    assert np.array_equal(y, A.val * x)


def test_permutation_exact():
    A, pi = gen.permutation(513)
    x = gen.dense_x(513, 7)
    y, _ = O.spmv(A, x)
    assert np.array_equal(y, x[pi])


@pytest.mark.parametrize("nx,ny", [(64, 64), (37, 29), (1, 5), (16, 1)])
def test_lap2d_rowsum_closed_form(nx, ny):
    """4 on the diagonal, -1 per grid neighbour, x = 1: y = 4 - degree."""
    A = gen.lap2d(nx, ny)
    y, _ = O.spmv(A, np.ones(A.n))
    i = np.arange(nx * ny)
    gx, gy = i % nx, i // nx
    deg = (gx > 0).astype(int) + (gx < nx - 1) + (gy > 0) + (gy < ny - 1)
    assert np.array_equal(y, 4.0 - deg)


@pytest.mark.parametrize("dims", [(7, 7, 7), (5, 6, 4), (16, 3, 2)])
def test_stencil27_rowsum_closed_form(dims):
    """26 on the diagonal, -1 per neighbour, x = 1: y = 27 - prod_d c_d with
    c_d = number of in-range positions among {p-1, p, p+1} along axis d."""
    nx, ny, nz = dims
    A = gen.stencil27(nx, values="stencil", ny=ny, nz=nz)
    y, _ = O.spmv(A, np.ones(A.n))
    i = np.arange(nx * ny * nz)
    gx, gy, gz = i % nx, (i // nx) % ny, i // (nx * ny)

    def c(p, N):
        return 1 + (p > 0).astype(int) + (p < N - 1)

    expect = 27.0 - c(gx, nx) * c(gy, ny) * c(gz, nz)
    assert np.array_equal(y, expect)
    # interior rows sum to 0, faces 9, edges 15, corners 19 on a cube
    if nx == ny == nz:
        assert set(np.unique(expect)) <= {0.0, 9.0, 15.0, 19.0}


def _exact_rows(A, x):
    out, outa = [], []
    for i in range(A.m):
        s = Fraction(0)
        sa = Fraction(0)
        for k in range(A.rowptr[i], A.rowptr[i + 1]):
            p = Fraction(float(A.val[k])) * Fraction(float(x[A.colidx[k]]))
            s += p
            sa += abs(p)
        out.append(s)
        outa.append(sa)
    return out, outa


@pytest.mark.parametrize("m,n,dens,seed", [(1, 1, 1.1, 1), (64, 64, 1.1, 2),
                                           (17, 33, 0.4, 3), (40, 7, 0.7, 4),
                                           (3, 64, 0.9, 5), (64, 2, 0.5, 6)])
def test_dense_bruteforce_exact_rational(m, n, dens, seed):
    """Brute force on <= 64 x 64: the exact rational sum of exact products,
    rounded once, must match within the oracle's own error bound
    (k+1) * 2^-63 * sum|a x| + half an ulp."""
    A = gen.random_sparse(m, n, dens, seed=seed)
    x = gen.dense_x(n, seed + 100)
    y, ay = O.spmv(A, x)
    ex, exa = _exact_rows(A, x)
    for i in range(m):
        k = A.rowptr[i + 1] - A.rowptr[i]
        bound = float(exa[i]) * (k + 1) * 2.0**-63 + abs(float(ex[i])) * 2.0**-53
        assert abs(y[i] - float(ex[i])) <= bound + 1e-300
        assert abs(ay[i] - float(exa[i])) <= float(exa[i]) * (k + 1) * 2.0**-62 + 1e-300
    # and against a dense matvec of the same matrix (library primitive)
    Ad = np.zeros((m, n))
    for i in range(m):
        Ad[i, A.colidx[A.rowptr[i]:A.rowptr[i + 1]]] = A.val[A.rowptr[i]:A.rowptr[i + 1]]
    assert np.allclose(y, Ad @ x, rtol=0, atol=1e-13 * max(1.0, np.abs(Ad).sum()))


def test_integer_valued_exact():
    """|a|, |x| <= 8: every partial sum is an integer far below 2^53, so the
    result is exact under any summation order."""
    A = gen.random_sparse(64, 64, 0.6, seed=9, values="int")
    x = gen.dense_x(64, 10, kind="int")
    y, _ = O.spmv(A, x)
    for i in range(A.m):
        s = 0
        for k in range(A.rowptr[i], A.rowptr[i + 1]):
            s += int(A.val[k]) * int(x[A.colidx[k]])
        assert y[i] == float(s)


def test_extended_accumulator_cancellation():
    """[1e16, 1, -1e16] . [1, 1, 1] = 1 exactly; a plain fp64 left-to-right sum
    gives 0.  Pins the extended-precision accumulator."""
    A = gen.csr_from_coo(1, 3, [0, 0, 0], [0, 1, 2], vals=[1e16, 1.0, -1e16])
    y, ay = O.spmv(A, np.ones(3))
    assert y[0] == 1.0
    assert ay[0] == 2e16 + 1.0 or abs(ay[0] - 2e16) <= 4.0


def test_empty_rows_and_row_subset():
    A = gen.random_sparse(50, 30, 0.3, seed=4, empty_rows=[0, 7, 49])
    x = gen.dense_x(30, 8)
    y, ay = O.spmv(A, x)
    assert y[0] == 0.0 and y[7] == 0.0 and y[49] == 0.0 and ay[7] == 0.0
    rows = np.array([49, 3, 3, 0, 17])
    ys, ays = O.spmv(A, x, rows)
    assert np.array_equal(ys, y[rows]) and np.array_equal(ays, ay[rows])


def test_zero_sized():
    A = gen.random_sparse(0, 5, 0.5)
    y, _ = O.spmv(A, np.ones(5))
    assert y.shape == (0,)
    A = gen.random_sparse(4, 0, 0.5)
    y, _ = O.spmv(A, np.zeros(0))
    assert np.array_equal(y, np.zeros(4))


def test_cpu_csr_omp_baseline_matches_oracle():
    """The multi-threaded CSR baseline bench.py reports as context (not the
    oracle) computes y = A x within the north-star tolerance of the oracle."""
    import numpy as np
    from oracle import oracle as O
    from synthetic import gen
    for name in ("mixed_small", "rmat12", "stencil27_21"):
        A, x = gen.make(name)
        y, threads = O.cpu_csr_omp(A, x)
        yr, absy = O.spmv(A, x)
        assert threads >= 1
        assert np.all(np.abs(y - yr) <= 1e-12 * absy + 1e-300), name


# ---------------------------------------------------------------------------
# oracle_spmv_f64: Alg. 1 as printed, in double (the CPU baseline of bench.py)
# ---------------------------------------------------------------------------

def test_f64_row_loop_identity_diagonal_permutation_exact():
    A = gen.identity(300)
    x = gen.dense_x(300, 5)
    assert np.array_equal(O.spmv_f64(A, x), x)
    D = gen.diagonal(257)
    assert np.array_equal(O.spmv_f64(D, gen.dense_x(257, 6)), D.val * gen.dense_x(257, 6))
    P, pi = gen.permutation(129)
    xp = gen.dense_x(129, 7)
    assert np.array_equal(O.spmv_f64(P, xp), O.spmv(P, xp)[0])


def test_f64_row_loop_sums_left_to_right_in_double():
    """y_i <- y_i + a_ij x_j in entry order, each step rounded to double
    (ulp(1e16) = 2, so 1e16 + 1 rounds back to 1e16): the three orders of
    {1e16, 1, -1e16} give 0, 0 and 1, where the extended-precision oracle
    gives 1 for all three."""
    rows = [0, 0, 0, 1, 1, 1, 2, 2, 2]
    cols = [0, 1, 2, 0, 1, 2, 0, 1, 2]
    vals = [1e16, 1.0, -1e16, 1.0, 1e16, -1e16, 1e16, -1e16, 1.0]
    A = gen.csr_from_coo(3, 3, rows, cols, vals=vals, name="order")
    y = O.spmv_f64(A, np.ones(3))
    assert y.tolist() == [0.0, 0.0, 1.0]
    assert O.spmv(A, np.ones(3))[0].tolist() == [1.0, 1.0, 1.0]


def test_f64_row_loop_integer_exact_and_within_bound():
    A = gen.stencil27(11, values="int", seed=3)
    x = gen.dense_x(A.n, 5, kind="int")
    assert np.array_equal(O.spmv_f64(A, x), O.spmv(A, x)[0])
    for name in ("rmat12", "mixed_small", "lap2d_37x29"):
        A, x = gen.make(name)
        y = O.spmv_f64(A, x)
        yref, absy = O.spmv(A, x)
        k = np.diff(A.rowptr.astype(np.int64))
        # sequential fp64 sum of k products: |err| <= (k + 1) u sum|a x| (u = 2^-53)
        assert np.all(np.abs(y - yref) <= (k + 1) * 2.0 ** -53 * absy * (1 + 1e-9))
