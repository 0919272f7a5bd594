"""ctypes wrapper around liboracle.so (oracle.c).

TEST INFRASTRUCTURE ONLY: imported by tests/, __graft_entry__.smoke() and the
cpu_baseline / --impl reference legs of bench.py, never by the product path
(paper_conf_ipps_niuldj0t21_b200).  See oracle.c for the citations.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass, field

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
LIB = os.path.join(HERE, "liboracle.so")
SRC = os.path.join(HERE, "oracle.c")

FMT_NAMES = ["CSR", "COO", "ELL", "HYB", "DNS", "DNSROW", "DNSCOL"]
CSR, COO, ELL, HYB, DNS, DNSROW, DNSCOL = range(7)
MODES = {"ADPT": 0, "DEFERRED": 1, "AUTO": 2, "FORCE_CSR": 3, "BYTES": 4}


OMP_SRC = os.path.join(HERE, "cpu_csr_omp.c")
OMP_LIB = os.path.join(HERE, "libcpu_csr_omp.so")


def build(force: bool = False) -> str:
    """gcc the oracle (plain C, -O2, no fast-math) and the multi-threaded CPU
    CSR baseline beside it (not the oracle; bench context only)."""
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < os.path.getmtime(SRC):
        subprocess.check_call(["gcc", "-O2", "-ffp-contract=off", "-std=c11", "-Wall", "-fPIC", "-shared",
                               "-o", LIB, SRC])
    if force or not os.path.exists(OMP_LIB) or os.path.getmtime(OMP_LIB) < os.path.getmtime(OMP_SRC):
        subprocess.check_call(["gcc", "-O3", "-std=c11", "-Wall", "-fopenmp", "-fPIC", "-shared",
                               "-o", OMP_LIB, OMP_SRC])
    return LIB


def cpu_csr_omp(A, x: np.ndarray):
    """y = A x by the OpenMP CSR baseline (all threads of the process);
    returns (y, threads).  Not the oracle: fp64 running sums."""
    build()
    L = ctypes.CDLL(OMP_LIB)
    p = ctypes.c_void_p
    L.cpu_csr_omp_spmv.argtypes = [ctypes.c_int64, p, p, p, p, p]
    L.cpu_csr_omp_threads.restype = ctypes.c_int
    rp, ci, va = _csr_arrays(A)
    x = np.ascontiguousarray(x, dtype=np.float64)
    y = np.empty(A.m, dtype=np.float64)
    L.cpu_csr_omp_spmv(A.m, _ptr(rp), _ptr(ci), _ptr(va), _ptr(x), _ptr(y))
    return y, int(L.cpu_csr_omp_threads())


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(LIB)
        p = ctypes.c_void_p
        L.oracle_spmv_rows.argtypes = [ctypes.c_int64, p, p, p, p, p, ctypes.c_int64, p, p]
        L.oracle_spmv_rows.restype = ctypes.c_int
        L.oracle_spmv_f64.argtypes = [ctypes.c_int64, p, p, p, p, p]
        L.oracle_spmv_f64.restype = None
        L.oracle_select.argtypes = [p, ctypes.c_int32, p]
        L.oracle_select.restype = ctypes.c_int
        L.oracle_select_bytes.argtypes = [p, p]
        L.oracle_select_bytes.restype = ctypes.c_int
        L.oracle_hyb_width.argtypes = [p]
        L.oracle_hyb_width.restype = ctypes.c_int
        L.oracle_tile.argtypes = [ctypes.c_int64, ctypes.c_int64, p, p, p, ctypes.c_int32]
        L.oracle_tile.restype = ctypes.c_void_p
        L.oracle_tiling_free.argtypes = [p]
        L.oracle_tiling_scalar.argtypes = [p, ctypes.c_int32]
        L.oracle_tiling_scalar.restype = ctypes.c_int64
        L.oracle_tiling_array.argtypes = [p, ctypes.c_int32]
        L.oracle_tiling_array.restype = ctypes.c_void_p
        L.oracle_decode.argtypes = [p, ctypes.c_int64, p, p, p]
        L.oracle_decode.restype = ctypes.c_int64
        _lib = L
    return _lib


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def _csr_arrays(A):
    rp = np.ascontiguousarray(A.rowptr, dtype=np.int32)
    ci = np.ascontiguousarray(A.colidx, dtype=np.int32)
    va = np.ascontiguousarray(A.val, dtype=np.float64)
    if ci.size == 0:
        ci = np.zeros(1, np.int32)
        va = np.zeros(1, np.float64)
    return rp, ci, va


def spmv(A, x: np.ndarray, rows: np.ndarray | None = None):
    """Alg. 1.  Returns (y, absy) for all rows or the given rows."""
    rp, ci, va = _csr_arrays(A)
    x = np.ascontiguousarray(x, dtype=np.float64)
    if x.size == 0:
        x = np.zeros(1)
    if rows is None:
        nr = A.m
        rws = None
    else:
        rws = np.ascontiguousarray(rows, dtype=np.int64)
        nr = rws.size
    y = np.zeros(max(nr, 1))
    ay = np.zeros(max(nr, 1))
    rc = lib().oracle_spmv_rows(A.m, _ptr(rp), _ptr(ci), _ptr(va), _ptr(x),
                                None if rws is None else _ptr(rws), nr, _ptr(y), _ptr(ay))
    assert rc == 0
    return y[:nr], ay[:nr]


def spmv_f64(A, x: np.ndarray) -> np.ndarray:
    """Alg. 1 as printed, in double (oracle_spmv_f64): the plain
    fp64 row loop timed as the CPU baseline.  Correctness checks use spmv()."""
    rp, ci, va = _csr_arrays(A)
    x = np.ascontiguousarray(x, dtype=np.float64)
    if x.size == 0:
        x = np.zeros(1)
    y = np.zeros(max(A.m, 1))
    lib().oracle_spmv_f64(A.m, _ptr(rp), _ptr(ci), _ptr(va), _ptr(x), _ptr(y))
    return y[:A.m]


def select(masks, force_csr: bool = False):
    """Format rule for one tile given 16 row bitmasks -> (fmt, aux)."""
    m = np.ascontiguousarray(np.asarray(masks, dtype=np.uint16))
    assert m.shape == (16,)
    aux = np.zeros(1, np.int32)
    f = lib().oracle_select(_ptr(m), int(force_csr), _ptr(aux))
    return int(f), int(aux[0])


def select_bytes(masks):
    """B200 byte-cost format rule for one tile (oracle_select_bytes) -> (fmt, aux)."""
    m = np.ascontiguousarray(np.asarray(masks, dtype=np.uint16))
    aux = ctypes.c_int32()
    f = lib().oracle_select_bytes(_ptr(m), ctypes.byref(aux))
    return f, aux.value


def hyb_width(lens) -> int:
    l = np.ascontiguousarray(np.asarray(lens, dtype=np.int32))
    assert l.shape == (16,)
    return int(lib().oracle_hyb_width(_ptr(l)))


@dataclass
class Tiling:
    m: int
    n: int
    nnz: int
    tilem: int
    tilen: int
    mode: int
    numtile: int
    payload_bytes: int
    rem_nnz: int
    tilePtr: np.ndarray
    tileColIdx: np.ndarray
    tileNnz: np.ndarray
    tileFmt: np.ndarray
    tileAux: np.ndarray
    tileOff: np.ndarray
    payload: np.ndarray
    remRowPtr: np.ndarray
    remCol: np.ndarray
    remVal: np.ndarray
    sel_tiles: np.ndarray = field(default_factory=lambda: np.zeros(7, np.int64))
    sel_nnz: np.ndarray = field(default_factory=lambda: np.zeros(7, np.int64))
    kept_tiles: np.ndarray = field(default_factory=lambda: np.zeros(7, np.int64))
    kept_nnz: np.ndarray = field(default_factory=lambda: np.zeros(7, np.int64))
    _handle: int = 0

    def arrays(self) -> dict:
        return {k: getattr(self, k) for k in
                ("tilePtr", "tileColIdx", "tileNnz", "tileFmt", "tileAux", "tileOff",
                 "payload", "remRowPtr", "remCol", "remVal")}


def tile(A, mode: str | int = "DEFERRED", keep_handle: bool = False) -> Tiling:
    """Reference tiler.  Raises on non-canonical input."""
    md = MODES[mode] if isinstance(mode, str) else int(mode)
    rp, ci, va = _csr_arrays(A)
    L = lib()
    h = L.oracle_tile(A.m, A.n, _ptr(rp), _ptr(ci), _ptr(va), md)
    if not h:
        raise ValueError("oracle_tile: non-canonical CSR input or out of memory")
    s = lambda w: int(L.oracle_tiling_scalar(h, w))
    m, numtile, pb, nr, tilem = s(0), s(6), s(7), s(8), s(3)

    def arr(which, dtype, count):
        if count == 0:
            return np.zeros(0, dtype)
        p = L.oracle_tiling_array(h, which)
        buf = (ctypes.c_char * (count * np.dtype(dtype).itemsize)).from_address(p)
        return np.frombuffer(buf, dtype=dtype, count=count).copy()

    T = Tiling(m=m, n=s(1), nnz=s(2), tilem=tilem, tilen=s(4), mode=s(5), numtile=numtile,
               payload_bytes=pb, rem_nnz=nr,
               tilePtr=arr(0, np.int32, tilem + 1), tileColIdx=arr(1, np.int32, numtile),
               tileNnz=arr(2, np.int32, numtile + 1), tileFmt=arr(3, np.uint8, numtile),
               tileAux=arr(4, np.uint8, numtile), tileOff=arr(5, np.uint32, numtile + 1),
               payload=arr(6, np.uint8, pb), remRowPtr=arr(7, np.int32, m + 1),
               remCol=arr(8, np.int32, nr), remVal=arr(9, np.float64, nr))
    if tilem == 0:
        T.tilePtr = np.zeros(1, np.int32)
    T.sel_tiles = np.array([s(100 + f) for f in range(7)], np.int64)
    T.sel_nnz = np.array([s(110 + f) for f in range(7)], np.int64)
    T.kept_tiles = np.array([s(120 + f) for f in range(7)], np.int64)
    T.kept_nnz = np.array([s(130 + f) for f in range(7)], np.int64)
    if keep_handle:
        T._handle = h
    else:
        L.oracle_tiling_free(h)
    return T


def decode(A, mode: str | int = "DEFERRED"):
    """Tile A with the reference tiler, then decode it back to sorted triplets."""
    T = tile(A, mode, keep_handle=True)
    L = lib()
    try:
        cap = A.nnz + 256 * T.numtile + 1
        rows = np.zeros(cap, np.int32)
        cols = np.zeros(cap, np.int32)
        vals = np.zeros(cap, np.float64)
        q = L.oracle_decode(T._handle, cap, _ptr(rows), _ptr(cols), _ptr(vals))
        assert q >= 0
    finally:
        L.oracle_tiling_free(T._handle)
        T._handle = 0
    return rows[:q], cols[:q], vals[:q]


def tile_row_sizes(T: Tiling) -> np.ndarray:
    """Payload bytes per tile (16-byte rounded) from tileOff."""
    return (np.diff(T.tileOff.astype(np.int64)) * 16) if T.numtile else np.zeros(0, np.int64)


def cg(A, b: np.ndarray, x0: np.ndarray | None = None, tol: float = 1e-10, maxit: int = 1000):
    """Conjugate gradients for SPD A (the iterative-solver
    use of SpMV), written out as the textbook Hestenes-Stiefel
    recurrence (e.g. Saad, Iterative Methods for Sparse Linear Systems,
    Alg. 6.18), in the order the GPU path (csrc/cg.cu) states it:

        r0 = b - A x0, p0 = r0
        q = A p_j;  alpha = (r_j, r_j) / (p_j, q)
        x_{j+1} = x_j + alpha p_j;  r_{j+1} = r_j - alpha q
        stop if ||r_{j+1}|| <= tol ||b||
        beta = (r_{j+1}, r_{j+1}) / (r_j, r_j);  p_{j+1} = r_{j+1} + beta p_j

    The matrix-vector products are this oracle's spmv (Alg. 1, long-double
    rows); dot products are numpy's.  Returns (x, iterations, ||r||/||b||)."""
    b = np.asarray(b, dtype=np.float64)
    x = np.zeros_like(b) if x0 is None else np.array(x0, dtype=np.float64)
    q, _ = spmv(A, x)
    r = b - q
    p = r.copy()
    rr = float(np.dot(r, r))
    bb = float(np.dot(b, b))
    it = 0
    if rr == 0.0:
        return x, 0, 0.0
    for j in range(maxit):
        q, _ = spmv(A, p)
        alpha = rr / float(np.dot(p, q))
        x = x + alpha * p
        r = r - alpha * q
        rr_new = float(np.dot(r, r))
        it = j + 1
        if rr_new <= tol * tol * bb:
            rr = rr_new
            break
        beta = rr_new / rr
        p = r + beta * p
        rr = rr_new
    return x, it, (np.sqrt(rr / bb) if bb > 0 else 0.0)
