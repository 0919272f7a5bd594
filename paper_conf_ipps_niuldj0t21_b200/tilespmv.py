"""Thin ctypes binding of include/tilespmv.h (argument marshalling only).

Every step of the path -- validation, tiling, format selection, extraction,
packing, scheduling and the SpMV itself -- runs in libtilespmv.so's CUDA
kernels.  PyTorch only provides device memory and streams.  There is no CPU
fallback: if the library or a CUDA device is missing, every call raises.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

from . import _build

FORMATS = ["CSR", "COO", "ELL", "HYB", "DNS", "DNSROW", "DNSCOL"]
MODES = {"ADPT": 0, "DEFERRED": 1, "AUTO": 2, "FORCE_CSR": 3, "BYTES": 4}
KERNELS = {"AUTO": 0, "SM_QUEUE": 1, "DENSE_ROWS": 2, "GATHER": 3}
ARRAYS = {"tilePtr": (0, np.int32), "tileColIdx": (1, np.int32), "tileNnz": (2, np.int32),
          "tileFmt": (3, np.uint8), "tileAux": (4, np.uint8), "tileOff": (5, np.uint32),
          "payload": (6, np.uint8), "remRowPtr": (7, np.int32), "remCol": (8, np.int32),
          "remVal": (9, np.float64)}
EXPORTED_SYMBOLS = ["tilespmv_create_from_csr", "tilespmv_run", "tilespmv_run_host",
                    "tilespmv_destroy", "tilespmv_get_info", "tilespmv_export_size",
                    "tilespmv_export", "tilespmv_status_string", "tilespmv_last_error",
                    "tilespmv_launch_shape", "tilespmv_kernel_name", "tilespmv_cg",
                    "tilespmv_auto_kernel", "tilespmv_run_scatter", "tilespmv_ipc_alloc",
                    "tilespmv_ipc_free", "tilespmv_ipc_open", "tilespmv_ipc_close"]


class TileSpMVError(RuntimeError):
    pass


class Opts(ctypes.Structure):
    _fields_ = [("mode", ctypes.c_int32), ("validate", ctypes.c_int32), ("kernel", ctypes.c_int32),
                ("keep_layout", ctypes.c_int32)]


class Info(ctypes.Structure):
    _fields_ = [("m", ctypes.c_int64), ("n", ctypes.c_int64), ("nnz", ctypes.c_int64),
                ("tilem", ctypes.c_int64), ("tilen", ctypes.c_int64), ("numtile", ctypes.c_int64),
                ("mode", ctypes.c_int32), ("device", ctypes.c_int32),
                ("sel_tiles", ctypes.c_int64 * 7), ("sel_nnz", ctypes.c_int64 * 7),
                ("kept_tiles", ctypes.c_int64 * 7), ("kept_nnz", ctypes.c_int64 * 7),
                ("rem_nnz", ctypes.c_int64), ("payload_bytes", ctypes.c_int64),
                ("meta_bytes", ctypes.c_int64), ("alg_bytes", ctypes.c_int64),
                ("flops", ctypes.c_int64), ("num_items", ctypes.c_int64),
                ("num_split_rows", ctypes.c_int64), ("device_bytes", ctypes.c_int64),
                ("create_ms", ctypes.c_double), ("kernel", ctypes.c_int32), ("xcache_cols", ctypes.c_int32)]

    def as_dict(self) -> dict:
        d = {}
        for name, _ in self._fields_:
            v = getattr(self, name)
            d[name] = list(v) if hasattr(v, "__len__") else v
        return d


_lib = None


def load(build_if_missing: bool = True):
    """Load libtilespmv.so (building it first if stale and nvcc is present)."""
    global _lib
    if _lib is not None:
        return _lib
    if build_if_missing and _build.stale():
        try:
            _build.build()
        except Exception as e:  # pragma: no cover
            if not os.path.exists(_build.LIB):
                raise TileSpMVError(f"libtilespmv.so missing and build failed: {e}") from e
    if not os.path.exists(_build.LIB):
        raise TileSpMVError(f"CUDA extension not built: {_build.LIB}")
    L = ctypes.CDLL(_build.LIB)
    p, i64, i32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32
    L.tilespmv_create_from_csr.argtypes = [ctypes.POINTER(p), i64, i64, i64, p, p, p,
                                           ctypes.POINTER(Opts), p]
    L.tilespmv_run.argtypes = [p, p, p, p]
    L.tilespmv_run_host.argtypes = [p, p, p, p]
    L.tilespmv_destroy.argtypes = [p]
    L.tilespmv_get_info.argtypes = [p, ctypes.POINTER(Info)]
    L.tilespmv_export_size.argtypes = [p, i32]
    L.tilespmv_export_size.restype = i64
    L.tilespmv_export.argtypes = [p, i32, p, ctypes.c_size_t]
    L.tilespmv_status_string.argtypes = [ctypes.c_int]
    L.tilespmv_status_string.restype = ctypes.c_char_p
    L.tilespmv_last_error.restype = ctypes.c_char_p
    L.tilespmv_launch_shape.argtypes = [p, ctypes.POINTER(i32), ctypes.POINTER(i32),
                                        ctypes.POINTER(i32)]
    L.tilespmv_cg.argtypes = [p, p, p, ctypes.c_double, i32, ctypes.POINTER(i32), ctypes.POINTER(ctypes.c_double), p]
    if hasattr(L, "tilespmv_auto_kernel"):  # (absent from round-1 builds used in A/B runs)
        L.tilespmv_auto_kernel.argtypes = [i64, i64, i64, i64]
        L.tilespmv_auto_kernel.restype = i32
    if hasattr(L, "tilespmv_run_scatter"):  # (absent from older builds used in A/B runs)
        L.tilespmv_run_scatter.argtypes = [p, p, p, ctypes.POINTER(p), i32, p]
        L.tilespmv_ipc_alloc.argtypes = [i64, ctypes.POINTER(p), p]
        L.tilespmv_ipc_free.argtypes = [p]
        L.tilespmv_ipc_open.argtypes = [p, ctypes.POINTER(p)]
        L.tilespmv_ipc_close.argtypes = [p]
        for name in ("tilespmv_run_scatter", "tilespmv_ipc_alloc", "tilespmv_ipc_free", "tilespmv_ipc_open",
                     "tilespmv_ipc_close"):
            getattr(L, name).restype = ctypes.c_int
    L.tilespmv_kernel_name.argtypes = [p]
    L.tilespmv_kernel_name.restype = ctypes.c_char_p
    for name in ("tilespmv_create_from_csr", "tilespmv_run", "tilespmv_run_host",
                 "tilespmv_destroy", "tilespmv_get_info", "tilespmv_export",
                 "tilespmv_launch_shape", "tilespmv_cg"):
        getattr(L, name).restype = ctypes.c_int
    _lib = L
    return L


def auto_kernel(payload_bytes: int, tilem: int, rem_nnz: int, alg_bytes: int) -> int:
    """TILESPMV_KERNEL_AUTO's choice for these totals (tilespmv_auto_kernel)."""
    return int(load().tilespmv_auto_kernel(int(payload_bytes), int(tilem), int(rem_nnz), int(alg_bytes)))


def _check(rc: int, what: str):
    if rc != 0:
        L = load()
        raise TileSpMVError(f"{what}: {L.tilespmv_status_string(rc).decode()} "
                            f"({L.tilespmv_last_error().decode()}) [status {rc}]")


def _stream_ptr(stream) -> int | None:
    if stream is None:
        import torch
        return torch.cuda.current_stream().cuda_stream or None
    return getattr(stream, "cuda_stream", stream) or None


def _require_cuda():
    import torch
    if not torch.cuda.is_available():
        raise TileSpMVError("no CUDA device: the tiled SpMV has no CPU fallback")


class TiledMatrix:
    """A device-resident tiled matrix (one handle of the C ABI)."""

    def __init__(self, handle: int, m: int, n: int):
        self._h = ctypes.c_void_p(handle)
        self.m, self.n = m, n

    # ---------------------------------------------------------------- create
    @classmethod
    def from_csr(cls, rowptr, colidx, val, m: int, n: int, mode: str | int = "DEFERRED",
                 validate: bool = True, stream=None, kernel: str | int = "AUTO",
                 keep_layout: bool = False) -> "TiledMatrix":
        """rowptr/colidx (int32) and val (float64) are CUDA tensors.  kernel:
        TILESPMV_KERNEL_* by name or number; keep_layout: keep the canonical
        tiled arrays for export() (tests)."""
        import torch
        _require_cuda()
        for t, dt in ((rowptr, torch.int32), (colidx, torch.int32), (val, torch.float64)):
            if not (t.is_cuda and t.dtype == dt and t.is_contiguous()):
                raise TileSpMVError("rowptr/colidx must be contiguous CUDA int32, val CUDA float64")
        L = load()
        md = MODES[mode] if isinstance(mode, str) else int(mode)
        kn = KERNELS[kernel] if isinstance(kernel, str) else int(kernel)
        opts = Opts(md, int(validate), kn, int(keep_layout))
        h = ctypes.c_void_p()
        nnz = int(colidx.numel())
        rc = L.tilespmv_create_from_csr(ctypes.byref(h), m, n, nnz, rowptr.data_ptr(),
                                        colidx.data_ptr() if nnz else None,
                                        val.data_ptr() if nnz else None, ctypes.byref(opts),
                                        _stream_ptr(stream))
        _check(rc, "tilespmv_create_from_csr")
        return cls(h.value, m, n)

    @classmethod
    def from_host_csr(cls, A, mode="DEFERRED", validate=True, device=None, stream=None, kernel="AUTO",
                      keep_layout=False):
        """Copies a host CSR (synthetic.gen.CSR-like: m, n, rowptr, colidx, val)."""
        import torch
        _require_cuda()
        dev = device or torch.device("cuda", torch.cuda.current_device())
        rp = torch.from_numpy(np.ascontiguousarray(A.rowptr, np.int32)).to(dev)
        ci = torch.from_numpy(np.ascontiguousarray(A.colidx, np.int32)).to(dev)
        va = torch.from_numpy(np.ascontiguousarray(A.val, np.float64)).to(dev)
        return cls.from_csr(rp, ci, va, A.m, A.n, mode, validate, stream, kernel, keep_layout)

    # -------------------------------------------------------------------- run
    def run(self, x, y=None, stream=None):
        """y = A @ x on the GPU (x, y float64 CUDA tensors).  Asynchronous."""
        import torch
        if y is None:
            y = torch.empty(self.m, dtype=torch.float64, device=x.device)
        if not (x.is_cuda and y.is_cuda and x.dtype == torch.float64 and y.dtype == torch.float64
                and x.is_contiguous() and y.is_contiguous()):
            raise TileSpMVError("x and y must be contiguous float64 CUDA tensors")
        if x.numel() != self.n or y.numel() != self.m:
            raise TileSpMVError(f"shape mismatch: A is {self.m}x{self.n}, x {x.numel()}, y {y.numel()}")
        rc = load().tilespmv_run(self._h, x.data_ptr() if self.n else None,
                                 y.data_ptr() if self.m else None, _stream_ptr(stream))
        _check(rc, "tilespmv_run")
        return y

    def run_scatter(self, x, y, peer_ptrs, stream=None):
        """y = A @ x, every row also stored to each peer pointer (device
        addresses of m doubles each, e.g. IpcBuffer.open peers at this rank's
        row offset): tilespmv_run_scatter.  Asynchronous."""
        import torch
        if not (x.is_cuda and y.is_cuda and x.dtype == torch.float64 and y.dtype == torch.float64
                and x.is_contiguous() and y.is_contiguous()):
            raise TileSpMVError("x and y must be contiguous float64 CUDA tensors")
        if x.numel() != self.n or y.numel() != self.m:
            raise TileSpMVError(f"shape mismatch: A is {self.m}x{self.n}, x {x.numel()}, y {y.numel()}")
        arr = (ctypes.c_void_p * max(len(peer_ptrs), 1))(*[int(q) for q in peer_ptrs])
        rc = load().tilespmv_run_scatter(self._h, x.data_ptr() if self.n else None,
                                         y.data_ptr() if self.m else None, arr, len(peer_ptrs),
                                         _stream_ptr(stream))
        _check(rc, "tilespmv_run_scatter")
        return y

    def run_host(self, hx, hy, stream=None):
        """Host buffers (pinned torch CPU tensors or numpy arrays): H2D, run, D2H, sync."""
        def ptr(a):
            return a.data_ptr() if hasattr(a, "data_ptr") else a.ctypes.data
        rc = load().tilespmv_run_host(self._h, ptr(hx) if self.n else None,
                                      ptr(hy) if self.m else None, _stream_ptr(stream))
        _check(rc, "tilespmv_run_host")
        return hy

    def cg(self, b, x=None, tol: float = 1e-10, maxit: int = 1000, stream=None):
        """Solve A x = b by conjugate gradients on the GPU (tilespmv_cg); A
        must be square SPD.  b (and x, the initial guess, zeros if None) are
        contiguous float64 CUDA tensors; returns (x, iterations, relres)."""
        import torch
        if x is None:
            x = torch.zeros(self.n, dtype=torch.float64, device=b.device)
        for t in (b, x):
            if not (t.is_cuda and t.dtype == torch.float64 and t.is_contiguous() and t.numel() == self.n):
                raise TileSpMVError("b and x must be contiguous float64 CUDA tensors of length n")
        it, rel = ctypes.c_int32(), ctypes.c_double()
        rc = load().tilespmv_cg(self._h, b.data_ptr() if self.n else None, x.data_ptr() if self.n else None,
                                float(tol), int(maxit), ctypes.byref(it), ctypes.byref(rel), _stream_ptr(stream))
        _check(rc, "tilespmv_cg")
        return x, it.value, rel.value

    # ------------------------------------------------------------------ info
    def info(self) -> dict:
        inf = Info()
        _check(load().tilespmv_get_info(self._h, ctypes.byref(inf)), "tilespmv_get_info")
        return inf.as_dict()

    def export(self, name: str) -> np.ndarray:
        which, dt = ARRAYS[name]
        L = load()
        nbytes = L.tilespmv_export_size(self._h, which)
        if nbytes < 0:
            _check(int(nbytes), "tilespmv_export_size")
        out = np.zeros(nbytes // np.dtype(dt).itemsize, dtype=dt)
        if nbytes:
            _check(L.tilespmv_export(self._h, which, out.ctypes.data, nbytes), "tilespmv_export")
        return out

    def export_all(self) -> dict:
        return {k: self.export(k) for k in ARRAYS}

    def launch_shape(self) -> tuple[int, int, int]:
        g, b, s = ctypes.c_int32(), ctypes.c_int32(), ctypes.c_int32()
        _check(load().tilespmv_launch_shape(self._h, ctypes.byref(g), ctypes.byref(b),
                                            ctypes.byref(s)), "tilespmv_launch_shape")
        return g.value, b.value, s.value

    def kernel_name(self) -> str:
        return load().tilespmv_kernel_name(self._h).decode()

    # --------------------------------------------------------------- cleanup
    def close(self):
        if self._h is not None and self._h.value:
            load().tilespmv_destroy(self._h)
        self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()


class IpcBuffer:
    """A cudaMalloc'd float64 buffer shareable with other processes (CUDA IPC
    through the ABI's tilespmv_ipc_*): .tensor is a zero-copy torch view,
    .handle the 64-byte IPC handle; IpcBuffer.open(handle) maps a peer's."""

    def __init__(self, n: int):
        _require_cuda()
        L = load()
        p, h = ctypes.c_void_p(), ctypes.create_string_buffer(64)
        _check(L.tilespmv_ipc_alloc(8 * max(n, 1), ctypes.byref(p), h), "tilespmv_ipc_alloc")
        self.ptr, self.n, self.handle = p.value, n, h.raw
        self.tensor = _device_tensor(self.ptr, n)

    @staticmethod
    def open(handle: bytes) -> int:
        """Maps a peer's buffer; returns its device address (close with close())."""
        p = ctypes.c_void_p()
        _check(load().tilespmv_ipc_open(ctypes.create_string_buffer(handle, 64), ctypes.byref(p)), "tilespmv_ipc_open")
        return p.value

    @staticmethod
    def close(ptr: int):
        _check(load().tilespmv_ipc_close(ctypes.c_void_p(ptr)), "tilespmv_ipc_close")

    def free(self):
        if self.ptr:
            self.tensor = None
            _check(load().tilespmv_ipc_free(ctypes.c_void_p(self.ptr)), "tilespmv_ipc_free")
            self.ptr = None


def _device_tensor(ptr: int, n: int):
    """A float64 CUDA tensor viewing n doubles at device address ptr (no copy)."""
    import torch

    class _View:
        __cuda_array_interface__ = {"shape": (n,), "typestr": "<f8", "data": (ptr, False), "version": 3,
                                    "strides": None}
    return torch.as_tensor(_View(), device=torch.device("cuda", torch.cuda.current_device()))
