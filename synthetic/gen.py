"""Seeded synthetic inputs for the tiled fp64 SpMV path.

This module is the ONLY code shared by the oracle side (``oracle/``) and the
CUDA side (``paper_conf_ipps_niuldj0t21_b200``).  It holds none of the
method's arithmetic: it builds canonical CSR matrices (int32 rowptr, int32
column indices strictly increasing per row, fp64 values) and dense x vectors,
nothing else.  No tiling, no format selection, no SpMV.

Randomness is counter-based (splitmix64 of ``seed ^ index * golden``, all
arithmetic mod 2^64), so every value depends only on (seed, index) and never
on generation order.  The shapes mirror the paper's
workloads (SuiteSparse, Table II) as restated in
BASELINE.json ``configs`` and DESIGN.md "Input recipe":

  C1 ``lap2d(64)``          2D 5-point Laplacian, 4,096 rows, 20,224 nnz
  C2 ``fem(3904)``          cant-shaped banded block matrix, dense 16x16 tiles
  C3 ``rmat(20, 16)``       Graph500 R-MAT power-law graph (a,b,c)=(.57,.19,.19)
  C4 ``mixed(65536)``       dense blocks + dense rows/cols + CSR/ELL/HYB/COO scatter
  C5 ``stencil27(200)``     3D 27-point stencil, 8M rows, 213.8M nnz
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np

GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)
_TWO_M53 = 1.0 / 9007199254740992.0  # 2^-53


@dataclass
class CSR:
    """Canonical CSR: rowptr[m+1] int32, colidx[nnz] int32, val[nnz] float64."""

    m: int
    n: int
    rowptr: np.ndarray
    colidx: np.ndarray
    val: np.ndarray
    name: str = ""

    @property
    def nnz(self) -> int:
        return int(self.colidx.shape[0])

    def row_slice(self, r0: int, r1: int) -> "CSR":
        """Rows [r0, r1) with rowptr rebased; the column space stays n."""
        a, b = int(self.rowptr[r0]), int(self.rowptr[r1])
        rp = (self.rowptr[r0:r1 + 1] - a).astype(np.int32)
        return CSR(r1 - r0, self.n, rp, self.colidx[a:b], self.val[a:b],
                   f"{self.name}[{r0}:{r1}]")


# ----------------------------------------------------------------------------
# counter-based RNG
# ----------------------------------------------------------------------------

def splitmix64(z):
    """splitmix64 finaliser on uint64 arrays (wrapping arithmetic)."""
    z = np.asarray(z, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = z + GOLDEN
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
        z = z ^ (z >> np.uint64(31))
    return z


def hash_u64(seed: int, idx):
    """u = splitmix64(seed ^ (idx * golden)) for a uint64 index array."""
    idx = np.asarray(idx, dtype=np.uint64)
    with np.errstate(over="ignore"):
        return splitmix64(np.uint64(seed & 0xFFFFFFFFFFFFFFFF) ^ (idx * GOLDEN))


def uniform01(seed: int, idx):
    """U[0,1) with 53 random bits."""
    return (hash_u64(seed, idx) >> np.uint64(11)).astype(np.float64) * _TWO_M53


def uniform_pm1(seed: int, idx):
    """U[-1,1); an exact 0.0 (probability 2^-53) is replaced by 0.5 so that
    generated matrices never hold explicit zeros (reading R27)."""
    v = 2.0 * uniform01(seed, idx) - 1.0
    v[v == 0.0] = 0.5
    return v


def small_int(seed: int, idx, lim: int = 8):
    """Integers in [-lim, lim] without 0, as float64 (bitwise-exact tests)."""
    q = (hash_u64(seed, idx) % np.uint64(2 * lim)).astype(np.int64)
    v = q - lim
    v[v >= 0] += 1
    return v.astype(np.float64)


def values_for(seed: int, rows: np.ndarray, cols: np.ndarray, n: int,
               kind: str = "uniform") -> np.ndarray:
    """a_ij from the counter (seed, i*n + j)."""
    idx = rows.astype(np.uint64) * np.uint64(n) + cols.astype(np.uint64)
    if kind == "uniform":
        return uniform_pm1(seed, idx)
    if kind == "int":
        return small_int(seed, idx)
    raise ValueError(kind)


def dense_x(n: int, seed: int = 101, kind: str = "uniform") -> np.ndarray:
    """x_j from the counter (seed, j)."""
    j = np.arange(n, dtype=np.uint64)
    if kind == "uniform":
        return uniform_pm1(seed, j) if n else np.zeros(0)
    if kind == "int":
        return small_int(seed, j) if n else np.zeros(0)
    if kind == "ones":
        return np.ones(n)
    raise ValueError(kind)


# ----------------------------------------------------------------------------
# assembling CSR from row-sorted coordinates
# ----------------------------------------------------------------------------

def csr_from_sorted(m: int, n: int, rows: np.ndarray, cols: np.ndarray,
                    vals: np.ndarray, name: str) -> CSR:
    """rows/cols must already be sorted by (row, col) and unique."""
    counts = np.bincount(rows, minlength=m) if rows.size else np.zeros(m, np.int64)
    rowptr = np.zeros(m + 1, dtype=np.int64)
    np.cumsum(counts, out=rowptr[1:])
    assert rowptr[-1] < 2**31
    return CSR(m, n, rowptr.astype(np.int32), cols.astype(np.int32),
               np.ascontiguousarray(vals, dtype=np.float64), name)


def csr_from_coo(m: int, n: int, rows, cols, vals=None, seed: int = 1,
                 kind: str = "uniform", name: str = "coo") -> CSR:
    """Sort and de-duplicate (keep first occurrence) arbitrary coordinates."""
    rows = np.asarray(rows, dtype=np.int64)
    cols = np.asarray(cols, dtype=np.int64)
    key = rows * max(n, 1) + cols
    order = np.argsort(key, kind="stable")
    key = key[order]
    first = np.ones(key.shape[0], dtype=bool)
    first[1:] = key[1:] != key[:-1]
    sel = order[first]
    r, c = rows[sel], cols[sel]
    if vals is None:
        v = values_for(seed, r, c, n, kind)
    else:
        v = np.asarray(vals, dtype=np.float64)[sel]
    return csr_from_sorted(m, n, r, c, v, name)


# ----------------------------------------------------------------------------
# C1: 2D 5-point Laplacian  kron(I,T) + kron(T,I), T = tridiag(-1, 2, -1)
# ----------------------------------------------------------------------------

def lap2d(nx: int = 64, ny: int | None = None, values: str = "stencil",
          seed: int = 1) -> CSR:
    """Row i = x + nx*y; 4 on the diagonal, -1 for each grid neighbour
    (values='stencil'), or counter-random values ('uniform' / 'int')."""
    ny = nx if ny is None else ny
    m = nx * ny
    i = np.arange(m, dtype=np.int64)
    x, y = i % nx, i // nx
    # neighbour offsets in increasing column order: -nx, -1, 0, +1, +nx
    offs = [(-nx, y > 0), (-1, x > 0), (0, np.ones(m, bool)), (1, x < nx - 1),
            (nx, y < ny - 1)]
    cols = np.stack([i + o for o, _ in offs], axis=1)
    mask = np.stack([v for _, v in offs], axis=1)
    rows = np.broadcast_to(i[:, None], cols.shape)[mask]
    cols = cols[mask]
    if values == "stencil":
        vals = np.where(rows == cols, 4.0, -1.0)
    else:
        vals = values_for(seed, rows, cols, m, values)
    return csr_from_sorted(m, m, rows, cols, vals, f"lap2d_{nx}x{ny}")


# ----------------------------------------------------------------------------
# C5: 3D 27-point stencil, pattern of kron(kron(T,T),T) with T = tridiag(1,1,1)
# ----------------------------------------------------------------------------

def stencil27(nx: int = 200, values: str = "uniform", seed: int = 7,
              ny: int | None = None, nz: int | None = None,
              row_range: tuple[int, int] | None = None) -> CSR:
    """Row i = x + nx*y + nx*ny*z.  values='stencil' puts 26 on the diagonal
    and -1 on the 26 neighbours; 'uniform'/'int' use the counter RNG.
    row_range=(r0, r1) generates only rows [r0, r1) (rebased, n unchanged),
    identical to the same rows of the full matrix."""
    ny = nx if ny is None else ny
    nz = nx if nz is None else nz
    n = nx * ny * nz
    r0, r1 = (0, n) if row_range is None else row_range
    plane = nx * ny
    # column order is increasing in (dz, dy, dx) lexicographic order
    offsets = [(dz, dy, dx) for dz in (-1, 0, 1) for dy in (-1, 0, 1)
               for dx in (-1, 0, 1)]
    rows_out, cols_out, vals_out = [], [], []
    chunk = 1 << 22
    for c0 in range(r0, r1, chunk):
        c1 = min(r1, c0 + chunk)
        i = np.arange(c0, c1, dtype=np.int64)
        x = i % nx
        y = (i // nx) % ny
        z = i // plane
        cols = np.empty((i.shape[0], 27), dtype=np.int64)
        mask = np.empty((i.shape[0], 27), dtype=bool)
        for k, (dz, dy, dx) in enumerate(offsets):
            cols[:, k] = i + dz * plane + dy * nx + dx
            ok = np.ones(i.shape[0], dtype=bool)
            if dx:
                ok &= (x + dx >= 0) & (x + dx < nx)
            if dy:
                ok &= (y + dy >= 0) & (y + dy < ny)
            if dz:
                ok &= (z + dz >= 0) & (z + dz < nz)
            mask[:, k] = ok
        r = np.broadcast_to(i[:, None], cols.shape)[mask]
        c = cols[mask]
        if values == "stencil":
            v = np.where(r == c, 26.0, -1.0)
        else:
            v = values_for(seed, r, c, n, values)
        rows_out.append((r - r0).astype(np.int32))
        cols_out.append(c.astype(np.int32))
        vals_out.append(v)
    rows = np.concatenate(rows_out) if rows_out else np.zeros(0, np.int32)
    cols = np.concatenate(cols_out) if cols_out else np.zeros(0, np.int32)
    vals = np.concatenate(vals_out) if vals_out else np.zeros(0)
    del rows_out, cols_out, vals_out
    return csr_from_sorted(r1 - r0, n, rows, cols, vals, f"stencil27_{nx}x{ny}x{nz}")


# ----------------------------------------------------------------------------
# C2: FEM-like banded block matrix (cant-shaped, Table II)
# ----------------------------------------------------------------------------

def fem(tile_rows: int = 3904, seed: int = 2, values: str = "uniform") -> CSR:
    """Tile (I,J) exists for |J-I| <= 2.  |J-I| <= 1: fully dense 16x16;
    J = I-2: upper triangle (c >= r, 136 entries); J = I+2: lower triangle
    (c <= r, 136 entries).  m = n = 16 * tile_rows."""
    T = tile_rows
    m = 16 * T
    r = np.arange(16)
    per_row_rows, per_row_cols = [], []
    # pattern of one block row, relative column offsets (J - I) * 16 + c
    for dJ in (-2, -1, 0, 1, 2):
        for rr in range(16):
            for c in range(16):
                if dJ == -2 and not c >= rr:
                    continue
                if dJ == 2 and not c <= rr:
                    continue
                per_row_rows.append(rr)
                per_row_cols.append(dJ * 16 + c)
    pr = np.array(per_row_rows, dtype=np.int64)
    pc = np.array(per_row_cols, dtype=np.int64)
    # sort the block-row pattern by (row, col)
    o = np.lexsort((pc, pr))
    pr, pc = pr[o], pc[o]
    I = np.arange(T, dtype=np.int64)
    rows = (16 * I[:, None] + pr[None, :]).ravel()
    cols = (16 * I[:, None] + pc[None, :]).ravel()
    keep = (cols >= 0) & (cols < m)
    rows, cols = rows[keep], cols[keep]
    vals = values_for(seed, rows, cols, m, values)
    del r
    return csr_from_sorted(m, m, rows, cols, vals, f"fem_{T}")


# ----------------------------------------------------------------------------
# C3: Graph500 R-MAT
# ----------------------------------------------------------------------------

def rmat(scale: int = 20, edge_factor: int = 16, a: float = 0.57,
         b: float = 0.19, c: float = 0.19, seed: int = 3, vseed: int = 4,
         values: str = "uniform") -> CSR:
    """Directed R-MAT, no noise and no vertex scrambling (hubs at low ids).
    Edge e, level l draws u = U(seed, e*scale + l) and picks a quadrant with
    thresholds a, a+b, a+b+c; the MSB is set first.  Duplicates are merged."""
    N = 1 << scale
    E = edge_factor * N
    rows = np.zeros(E, dtype=np.int64)
    cols = np.zeros(E, dtype=np.int64)
    e = np.arange(E, dtype=np.uint64) * np.uint64(scale)
    ab, abc = a + b, a + b + c
    for lvl in range(scale):
        u = uniform01(seed, e + np.uint64(lvl))
        bit = np.int64(1) << np.int64(scale - 1 - lvl)
        rbit = u >= ab            # quadrants c, d -> lower half (row bit 1)
        cbit = ((u >= a) & (u < ab)) | (u >= abc)   # quadrants b, d
        rows += rbit.astype(np.int64) * bit
        cols += cbit.astype(np.int64) * bit
    key = rows * N + cols
    del rows, cols
    key.sort()
    keep = np.ones(key.shape[0], dtype=bool)
    keep[1:] = key[1:] != key[:-1]
    key = key[keep]
    r, cc = key // N, key % N
    vals = values_for(vseed, r, cc, N, values)
    return csr_from_sorted(N, N, r, cc, vals, f"rmat_s{scale}_ef{edge_factor}")


# ----------------------------------------------------------------------------
# C4: mixed structure exercising all seven tile formats
# ----------------------------------------------------------------------------

def _units_mod(k: int) -> np.ndarray:
    u = np.arange(1, max(k, 2), dtype=np.int64)
    return u[np.gcd(u, k) == 1] if k > 1 else np.array([1])


def mixed(tile_rows: int = 65536, seed: int = 5, vseed: int = 6,
          values: str = "uniform") -> CSR:
    """Per tile row I: tile J=I is fully dense (256); 15 further distinct tile
    columns J != I hold, in draw order: DnsRow (4 random full rows), DnsCol
    (4 random full columns), ELL (row r: columns (r+2k) mod 16, k<7), CSR
    (rows 0-7 length 4, rows 8-15 length 8), HYB (rows 0-1 length 15, rows
    2-15 length 1) and 10 very sparse tiles of 1..11 entries at random
    positions.  Requires tile_rows >= 16.  m = n = 16 * tile_rows."""
    T = tile_rows
    assert T >= 16
    m = 16 * T
    I = np.arange(T, dtype=np.int64)
    base = I.astype(np.uint64) * np.uint64(64)

    def draw(d):  # U[0,1) per tile row, draw index d < 64
        return uniform01(seed, base + np.uint64(d))

    def pick(d, k):  # integer in [0, k)
        return np.minimum((draw(d) * k).astype(np.int64), k - 1)

    # 15 distinct tile columns != I:  J = (I + 1 + ((o0 + i*s) mod (T-1))) mod T
    units = _units_mod(T - 1)
    o0 = pick(0, T - 1)
    s = units[pick(1, len(units))]
    Js = [(I + 1 + ((o0 + i * s) % (T - 1))) % T for i in range(15)]

    ents_r, ents_c = [], []   # per tile: arrays [T, k] of (local r, local c), and J

    def add(J, lr, lc):
        ents_r.append((16 * I[:, None] + lr))
        ents_c.append((16 * J[:, None] + lc))

    r16 = np.arange(16, dtype=np.int64)
    # Dns at J = I
    add(I, np.repeat(r16, 16)[None, :].repeat(T, 0), np.tile(r16, 16)[None, :].repeat(T, 0))

    def distinct16(d, k):  # k distinct values of [0,16): (a + i*odd) mod 16
        a = pick(d, 16)
        st = 2 * pick(d + 1, 8) + 1
        return (a[:, None] + np.arange(k)[None, :] * st[:, None]) % 16

    # DnsRow: 4 full rows
    fr = distinct16(2, 4)
    add(Js[0], np.repeat(fr, 16, axis=1), np.tile(r16, 4)[None, :].repeat(T, 0))
    # DnsCol: 4 full columns
    fc = distinct16(4, 4)
    add(Js[1], np.tile(r16, 4)[None, :].repeat(T, 0), np.repeat(fc, 16, axis=1))
    # ELL: row r has columns (r + 2k) mod 16, k < 7
    er = np.repeat(r16, 7)
    ec = (er + 2 * np.tile(np.arange(7), 16)) % 16
    add(Js[2], er[None, :].repeat(T, 0), ec[None, :].repeat(T, 0))
    # CSR: rows 0-7 length 4, rows 8-15 length 8 (distinct random columns)
    cr, cc = [], []
    for rr in range(16):
        k = 4 if rr < 8 else 8
        cr.append(np.full((T, k), rr))
        cc.append(distinct16(6 + 2 * rr, k))
    add(Js[3], np.concatenate(cr, 1), np.concatenate(cc, 1))
    # HYB: rows 0-1 length 15 (all but one column), rows 2-15 length 1
    hr, hc = [], []
    for rr in range(2):
        skip = pick(38 + rr, 16)
        cols15 = (skip[:, None] + 1 + np.arange(15)[None, :]) % 16
        hr.append(np.full((T, 15), rr))
        hc.append(cols15)
    for rr in range(2, 16):
        hr.append(np.full((T, 1), rr))
        hc.append(pick(40 + rr, 16)[:, None])
    add(Js[4], np.concatenate(hr, 1), np.concatenate(hc, 1))
    # 10 very sparse tiles: k in [1, 11] entries at distinct positions
    # p_i = (p0 + i * odd) mod 256
    coo_r, coo_c, coo_keep = [], [], []
    for t in range(10):
        Jt = Js[5 + t]
        k = 1 + (hash_u64(seed ^ 0x5151, base + np.uint64(t))
                 % np.uint64(11)).astype(np.int64)
        p0 = (hash_u64(seed ^ 0x7777, base + np.uint64(t)) % np.uint64(256)).astype(np.int64)
        st = 2 * (hash_u64(seed ^ 0x3333, base + np.uint64(t)) % np.uint64(128)).astype(np.int64) + 1
        pos = (p0[:, None] + np.arange(11)[None, :] * st[:, None]) % 256
        keep = np.arange(11)[None, :] < k[:, None]
        coo_r.append(16 * I[:, None] + pos // 16)
        coo_c.append(16 * Jt[:, None] + pos % 16)
        coo_keep.append(keep)
    rows = np.concatenate([e.ravel() for e in ents_r] +
                          [r[kp] for r, kp in zip(coo_r, coo_keep)])
    cols = np.concatenate([e.ravel() for e in ents_c] +
                          [c[kp] for c, kp in zip(coo_c, coo_keep)])
    del ents_r, ents_c, coo_r, coo_c
    order = np.lexsort((cols, rows))
    rows, cols = rows[order], cols[order]
    assert np.all((rows[1:] != rows[:-1]) | (cols[1:] != cols[:-1])), "duplicate"
    vals = values_for(vseed, rows, cols, m, values)
    return csr_from_sorted(m, m, rows, cols, vals, f"mixed_{T}")


# ----------------------------------------------------------------------------
# small special matrices (edge cases and oracle pins)
# ----------------------------------------------------------------------------

def identity(n: int) -> CSR:
    i = np.arange(n, dtype=np.int64)
    return csr_from_sorted(n, n, i, i, np.ones(n), f"eye_{n}")


def diagonal(n: int, seed: int = 11) -> CSR:
    i = np.arange(n, dtype=np.int64)
    return csr_from_sorted(n, n, i, i, uniform_pm1(seed, i.astype(np.uint64)),
                           f"diag_{n}")


def permutation(n: int, seed: int = 12) -> tuple[CSR, np.ndarray]:
    """Row i has a single 1 at column pi[i]; returns (A, pi)."""
    pi = np.argsort(hash_u64(seed, np.arange(n, dtype=np.uint64)), kind="stable")
    i = np.arange(n, dtype=np.int64)
    return csr_from_sorted(n, n, i, pi, np.ones(n), f"perm_{n}"), pi


def random_sparse(m: int, n: int, density: float, seed: int = 13,
                  values: str = "uniform", empty_rows=()) -> CSR:
    """Bernoulli(density) pattern from the counter (seed, i*n+j)."""
    if m == 0 or n == 0:
        return CSR(m, n, np.zeros(m + 1, np.int32), np.zeros(0, np.int32),
                   np.zeros(0), f"rand_{m}x{n}")
    rows_out, cols_out = [], []
    step = max(1, (1 << 22) // n)
    for r0 in range(0, m, step):
        r1 = min(m, r0 + step)
        idx = (np.arange(r0, r1, dtype=np.uint64)[:, None] * np.uint64(n)
               + np.arange(n, dtype=np.uint64)[None, :])
        mask = uniform01(seed ^ 0xABCDEF, idx) < density
        rr, cc = np.nonzero(mask)
        rows_out.append(rr + r0)
        cols_out.append(cc)
    rows = np.concatenate(rows_out).astype(np.int64)
    cols = np.concatenate(cols_out).astype(np.int64)
    if len(empty_rows):
        keep = ~np.isin(rows, np.asarray(empty_rows))
        rows, cols = rows[keep], cols[keep]
    vals = values_for(seed, rows, cols, n, values)
    return csr_from_sorted(m, n, rows, cols, vals, f"rand_{m}x{n}_{density}")


def dense(m: int, n: int, seed: int = 14, values: str = "uniform") -> CSR:
    return random_sparse(m, n, 1.1, seed, values)


def from_dense(Ad: np.ndarray, name: str = "dense") -> CSR:
    """Every non-zero of a dense array becomes an entry."""
    rr, cc = np.nonzero(Ad)
    return csr_from_sorted(Ad.shape[0], Ad.shape[1], rr.astype(np.int64),
                           cc.astype(np.int64), Ad[rr, cc], name)


def tile_pattern(mask_rows, values_seed: int = 21, tiles=((0, 0),),
                 m: int = 16, n: int = 16) -> CSR:
    """Place one 16x16 tile pattern (list of 16 column bitmasks, bit c = column
    c present in row r) at each tile (I, J) of `tiles` of an m x n matrix."""
    rows, cols = [], []
    for (I, J) in tiles:
        for r, msk in enumerate(mask_rows):
            for c in range(16):
                if (msk >> c) & 1:
                    rows.append(16 * I + r)
                    cols.append(16 * J + c)
    return csr_from_coo(m, n, rows, cols, seed=values_seed, name="tile_pattern")


# ----------------------------------------------------------------------------
# the five BASELINE.json configs and their small twins
# ----------------------------------------------------------------------------

CONFIGS = {
    # name: (constructor, kwargs, x seed)
    "lap2d_64": (lap2d, dict(nx=64), 101),
    "fem": (fem, dict(tile_rows=3904), 101),
    "rmat20": (rmat, dict(scale=20, edge_factor=16), 101),
    "mixed": (mixed, dict(tile_rows=65536), 101),
    "stencil27_200": (stencil27, dict(nx=200), 101),
    # small twins (oracle finishes in seconds; several tiles + ragged tails)
    "fem_small": (fem, dict(tile_rows=97), 101),
    "rmat12": (rmat, dict(scale=12, edge_factor=16), 101),
    "mixed_small": (mixed, dict(tile_rows=64), 101),
    "stencil27_48": (stencil27, dict(nx=48), 101),
    "stencil27_40": (stencil27, dict(nx=40), 101),
    "stencil27_21": (stencil27, dict(nx=21), 101),
    "lap2d_37x29": (lap2d, dict(nx=37, ny=29), 101),
}


def make(name: str) -> tuple[CSR, np.ndarray]:
    fn, kw, xseed = CONFIGS[name]
    A = fn(**kw)
    A.name = name
    return A, dense_x(A.n, xseed)
