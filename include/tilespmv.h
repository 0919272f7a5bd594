/*
 * tilespmv.h -- C ABI of the B200-native TileSpMV hot path.
 *
 * Operation (Alg. 1): y = A * x in fp64
 * (P:237), A sparse m x n given in CSR, converted to the paper's
 * two-level 16x16 tiled storage with per-tile formats chosen by
 * the TileSpMV_ADPT rules and, by default, the DeferredCOO
 * extraction of all COO data into a CSR remainder.  The
 * preprocess-then-multiply split follows P:285-289.
 *
 * Conventions for every entry point
 *   - plain pointers and sizes only; `stream` is a cudaStream_t passed as
 *     void* (NULL = the legacy default stream);
 *   - "d_" pointers are device memory on the device current at create time,
 *     "h_" pointers are host memory;
 *   - every call returns an int status: TILESPMV_OK (0) or a negative code
 *     below.  Nothing throws or aborts across the ABI; the last error message
 *     of the calling thread is available from tilespmv_last_error().
 */
#ifndef TILESPMV_H
#define TILESPMV_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* status codes */
#define TILESPMV_OK 0
#define TILESPMV_INVALID_ARG (-1)       /* null pointer, negative size, bad mode/array id,
                                           x/y overlap, handle used on another device   */
#define TILESPMV_NOT_CANONICAL (-2)     /* rowptr not monotone / not 0..nnz, column out of
                                           range, or columns not strictly increasing      */
#define TILESPMV_OVERFLOW (-3)          /* nnz >= 2^31, m or n >= 2^31, payload >= 64 GiB */
#define TILESPMV_OOM (-4)               /* device or host allocation failed               */
#define TILESPMV_CUDA (-5)              /* any other CUDA runtime error                   */

/* methods of P:177 (+ the size switch of P:235) */
#define TILESPMV_MODE_ADPT 0      /* TileSpMV_ADPT: adaptive format per tile, no extraction */
#define TILESPMV_MODE_DEFERRED 1  /* TileSpMV_DeferredCOO: COO data -> CSR remainder (default) */
#define TILESPMV_MODE_AUTO 2      /* DEFERRED iff nnz >= 1.8e6 (reading R18), else ADPT */
#define TILESPMV_MODE_FORCE_CSR 3 /* TileSpMV_CSR: every tile CSR */
#define TILESPMV_MODE_BYTES 4     /* NOT the paper's rule: per tile, the format
                                     with the fewest payload bytes (DESIGN.md §4 sizes, rounded
                                     to 16; ELL only if every row is non-empty; ties to the
                                     lower format code); no extraction.  The paper's thresholds
                                     (Dns >= 128) were set on A100; a 136-entry FEM
                                     triangle is 1,184 B as CSR against 2,048 B as Dns        */

/* SpMV kernel of a handle (tilespmv_opts_t.kernel).  Both compute the same
 * y within the north-star bound; the work-item byte budget (and so the
 * order of the sums) is the kernel's, so handles that must agree bitwise
 * (row slices of one matrix, tilespmv sharding) must use the same kernel. */
#define TILESPMV_KERNEL_AUTO 0       /* GATHER if the CSR remainder holds more than half of the
                                        algorithmic bytes (power-law graphs in DEFERRED mode), else
                                        DENSE_ROWS if the mean stored payload per tile row exceeds
                                        6 KiB (dense, FEM-like tile rows), else SM_QUEUE          */
#define TILESPMV_KERNEL_SM_QUEUE 1   /* one 32-warp CTA per SM, 4.5 KiB items, shared-memory queue */
#define TILESPMV_KERNEL_DENSE_ROWS 2 /* 16 warps per SM, 10.5 KiB items, static per-warp chunks    */
#define TILESPMV_KERNEL_GATHER 3     /* SM_QUEUE with ~3 KiB items of at most 4 tiles and a 16 KiB
                                        x cache of the most-gathered remainder columns: 131 KiB of
                                        shared memory per SM instead of 209 KiB leaves ~124 KiB of
                                        L1 to the remainder's x gathers                            */

/* tile format codes, in the order of P:20 / P:96 */
#define TILESPMV_FMT_CSR 0
#define TILESPMV_FMT_COO 1
#define TILESPMV_FMT_ELL 2
#define TILESPMV_FMT_HYB 3
#define TILESPMV_FMT_DNS 4
#define TILESPMV_FMT_DNSROW 5
#define TILESPMV_FMT_DNSCOL 6

/* arrays for tilespmv_export (canonical layout, DESIGN.md §"Canonical layout") */
#define TILESPMV_ARR_TILEPTR 0    /* int32  [tilem+1]   tiles per tile row, prefix        */
#define TILESPMV_ARR_TILECOLIDX 1 /* int32  [numtile]   tile column index                 */
#define TILESPMV_ARR_TILENNZ 2    /* int32  [numtile+1] prefix of nonzeros held per tile  */
#define TILESPMV_ARR_TILEFMT 3    /* uint8  [numtile]   format code                               */
#define TILESPMV_ARR_TILEAUX 4    /* uint8  [numtile]   ELL/HYB width, DnsRow/DnsCol count, else 0 */
#define TILESPMV_ARR_TILEOFF 5    /* uint32 [numtile+1] payload offset in 16-byte units          */
#define TILESPMV_ARR_PAYLOAD 6    /* uint8  [payload_bytes] level-2 per-tile payloads */
#define TILESPMV_ARR_REMROWPTR 7  /* int32  [m+1]       remainder CSR; empty if no extraction */
#define TILESPMV_ARR_REMCOL 8     /* int32  [rem_nnz]   global column indices                     */
#define TILESPMV_ARR_REMVAL 9     /* double [rem_nnz]                                             */

typedef struct tilespmv_matrix *tilespmv_handle_t; /* opaque; owns all its device storage */

typedef struct {
    int32_t mode;        /* TILESPMV_MODE_*; default DEFERRED                               */
    int32_t validate;    /* 1 (default): check the CSR is canonical; 0: trust the caller   */
    int32_t kernel;      /* TILESPMV_KERNEL_*; default AUTO                                 */
    int32_t keep_layout; /* 0 (default): after create the handle keeps only what the SpMV
                            kernel reads (the execution schedule, about the matrix's
                            algorithmic bytes); 1: also keep the canonical tiled arrays for
                            tilespmv_export (bit-exact parity tests)                       */
} tilespmv_opts_t;

typedef struct {
    int64_t m, n, nnz;
    int64_t tilem, tilen; /* ceil(m/16), ceil(n/16) */
    int64_t numtile;      /* tiles stored (after extraction) */
    int32_t mode;         /* resolved mode (AUTO never appears here) */
    int32_t device;
    int64_t sel_tiles[7], sel_nnz[7];   /* formats chosen by the ADPT rules, before extraction */
    int64_t kept_tiles[7], kept_nnz[7]; /* tiles stored and the nonzeros they hold */
    int64_t rem_nnz;                    /* nonzeros in the CSR remainder */
    int64_t payload_bytes;              /* level-2 payload (16-byte aligned per tile) */
    int64_t meta_bytes;                 /* level-1 arrays read per SpMV */
    int64_t alg_bytes;                  /* algorithmic bytes per SpMV (DESIGN.md §"Bytes model") */
    int64_t flops;                      /* 2 * nnz */
    int64_t num_items;                  /* warp work items of the SpMV schedule */
    int64_t num_split_rows;             /* tile rows split over several items */
    int64_t device_bytes;               /* device memory owned by the handle */
    double create_ms;                   /* wall time of tilespmv_create_from_csr */
    int32_t kernel;                     /* resolved TILESPMV_KERNEL_* (never AUTO) */
    int32_t xcache_cols;                /* GATHER kernel: remainder columns held in its shared-memory
                                           x cache (the most-gathered ones, <= 2048); 0 otherwise */
} tilespmv_info_t;

/* Build a tiled matrix from a canonical device CSR ("converting a basic
 * CSR matrix to our tile form").  All preprocessing runs on the GPU.
 *   m, n        rows / columns (0 allowed; m,n < 2^31)
 *   nnz         number of stored entries (< 2^31); must equal d_rowptr[m]
 *   d_rowptr    int32[m+1], d_colidx int32[nnz], d_val double[nnz]: device,
 *               caller-owned, read only during this call.  Explicit zeros
 *               are entries.  d_colidx/d_val may be NULL when nnz == 0.
 *   opts        NULL = defaults {DEFERRED, validate=1, kernel=AUTO, keep_layout=0}
 *   stream      every kernel, copy and temporary allocation of the call is
 *               queued on it (stream-ordered; no device-wide synchronisation,
 *               other streams keep running); the call synchronises `stream`
 *               before return, so the inputs may be freed immediately.
 * On success *out receives a handle bound to the current device.
 * Errors: INVALID_ARG, NOT_CANONICAL (only detected with validate=1),
 * OVERFLOW, OOM, CUDA.  On error *out is set to NULL and nothing leaks.     */
int tilespmv_create_from_csr(tilespmv_handle_t *out, int64_t m, int64_t n, int64_t nnz,
                             const int32_t *d_rowptr, const int32_t *d_colidx,
                             const double *d_val, const tilespmv_opts_t *opts, void *stream);

/* y = A * x (Alg. 1: y_i <- 0, then y_i += a_ij * x_j).
 *   d_x double[n] device, read; must be finite (reading R19).
 *   d_y double[m] device, fully overwritten (no alpha/beta); must not overlap x.
 * Asynchronous on `stream`: one kernel launch, no host synchronisation.
 * The result is bitwise deterministic run to run.  Runs on the same handle
 * must be serialised (the handle owns one split-row workspace).             */
int tilespmv_run(tilespmv_handle_t h, const double *d_x, double *d_y, void *stream);

/* tilespmv_run with a fused scatter epilogue (SURVEY §8(e), B200-native
 * improvement 2): every row of y is stored to d_y AND to each of the n_peer
 * device pointers d_peer_ys[t] (double[m] each; typically the peers' copies of
 * the next iterate at this rank's row offset, mapped with tilespmv_ipc_open
 * so the stores travel over NVLink), so tile-row sharded iterated SpMV needs
 * no separate all-gather.  n_peer in 0..7 (0 = tilespmv_run).  Completion is
 * the kernel's: the caller synchronises with the peers (e.g. a barrier after
 * the stream) before they read.  Errors as tilespmv_run, plus INVALID_ARG for
 * n_peer out of range or a NULL peer pointer.                                */
int tilespmv_run_scatter(tilespmv_handle_t h, const double *d_x, double *d_y, double *const *d_peer_ys,
                         int32_t n_peer, void *stream);

/* CUDA IPC plumbing for tilespmv_run_scatter's peers (handles are 64 bytes).
 * ipc_alloc: cudaMalloc(bytes) into *d_ptr and its IPC handle into handle[64];
 * ipc_open: map a peer's handle (cudaIpcOpenMemHandle, lazy peer access);
 * ipc_close / ipc_free undo them.  Errors: INVALID_ARG, CUDA.                 */
int tilespmv_ipc_alloc(int64_t bytes, void **d_ptr, void *handle);
int tilespmv_ipc_free(void *d_ptr);
int tilespmv_ipc_open(const void *handle, void **d_ptr);
int tilespmv_ipc_close(void *d_ptr);

/* Host-buffer variant: copies h_x (double[n]) to a handle-owned device
 * buffer, runs, copies y back to h_y (double[m]) and synchronises `stream`.
 * h_x / h_y should be page-locked for asynchronous copies.                  */
int tilespmv_run_host(tilespmv_handle_t h, const double *h_x, double *h_y, void *stream);

/* Conjugate-gradient solve of A x = b (the iterative
 * solver use that motivates SpMV), built on tilespmv_run's kernel.
 * Hestenes-Stiefel CG in fp64 (cg.cu states the recurrence); A must be
 * square (m == n) and symmetric positive definite -- symmetry and
 * definiteness are NOT checked (an indefinite A may stall or diverge).
 *   d_b     double[n] device, read.
 *   d_x     double[n] device: the initial guess on entry, the iterate on
 *           exit; must be finite and must not overlap d_b.
 *   tol     stop once ||r_k|| <= tol * ||b|| (recursive residual), tol >= 0.
 *   maxit   at most this many iterations (>= 0).
 *   iters   (optional) iterations performed; relres (optional) ||r_k||/||b||.
 * Synchronous: work is queued on `stream`, which is synchronised before the
 * call returns.  Work memory (3 n doubles) is allocated and freed per call.
 * Errors: INVALID_ARG (m != n, NULL vectors, bad tol/maxit), OOM, CUDA.      */
int tilespmv_cg(tilespmv_handle_t h, const double *d_b, double *d_x, double tol, int32_t maxit,
                int32_t *iters, double *relres, void *stream);

/* Release all device storage; NULL is a no-op returning TILESPMV_OK. */
int tilespmv_destroy(tilespmv_handle_t h);

/* Statistics of the tiled matrix (format histogram P:229, space P:279). */
int tilespmv_get_info(tilespmv_handle_t h, tilespmv_info_t *info);

/* Size in bytes of an exported array (TILESPMV_ARR_*), or a negative status. */
int64_t tilespmv_export_size(tilespmv_handle_t h, int32_t which);

/* Copy one array of the canonical tiled layout to host memory (synchronous);
 * `bytes` must equal tilespmv_export_size(h, which).  Used for bit-exact
 * parity against the reference tiler.  Needs a handle created with
 * opts.keep_layout = 1 (else INVALID_ARG; tilespmv_export_size returns the
 * size either way).                                                          */
int tilespmv_export(tilespmv_handle_t h, int32_t which, void *host_dst, size_t bytes);

/* The kernel TILESPMV_KERNEL_AUTO resolves to for a matrix whose stored
 * tile payload is payload_bytes over tilem tile rows, with rem_nnz
 * remainder entries and alg_bytes algorithmic bytes (tilespmv_info_t).
 * Sharded callers apply it to the whole matrix's totals so that every shard
 * runs the kernel (and the item byte budget) of the unsharded matrix, and so
 * the unsharded summation order.                                            */
int32_t tilespmv_auto_kernel(int64_t payload_bytes, int64_t tilem, int64_t rem_nnz, int64_t alg_bytes);

/* Static description of a status code. */
const char *tilespmv_status_string(int status);

/* Message of the last failing call on this thread ("" if none). */
const char *tilespmv_last_error(void);

/* Launch shape of the SpMV kernel for this handle: grid CTAs, threads per
 * CTA, dynamic shared memory bytes. */
int tilespmv_launch_shape(tilespmv_handle_t h, int32_t *grid, int32_t *block, int32_t *smem_bytes);

/* Name of the SpMV kernel variant this handle launches (static string; ""
 * for a NULL handle). */
const char *tilespmv_kernel_name(tilespmv_handle_t h);

#ifdef __cplusplus
}
#endif
#endif /* TILESPMV_H */
