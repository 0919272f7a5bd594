// abi.cu -- the extern "C" boundary declared in include/tilespmv.h.
// Argument checking, handle lifetime, info/export, error strings.  All
// compute is in tiler.cu, schedule.cu (create) and spmv_warp.cu (run).
#include <chrono>
#include <cstring>
#include <string>

#include "internal.cuh"

namespace tsp {

static thread_local std::string g_last_error;

int set_error(int status, const std::string &msg) {
    g_last_error = msg;
    return status;
}

int cuda_status(cudaError_t e, const char *what) {
    std::string msg = std::string(what) + ": " + cudaGetErrorString(e);
    cudaGetLastError();  // clear sticky-free errors
    if (e == cudaErrorMemoryAllocation) return set_error(TILESPMV_OOM, msg);
    return set_error(TILESPMV_CUDA, msg);
}

}  // namespace tsp

struct tilespmv_matrix : tsp::Matrix {};

namespace tsp {

static void free_matrix(tilespmv_matrix *M) {
    if (!M) return;
    int cur = -1;
    cudaGetDevice(&cur);
    if (cur != M->device) cudaSetDevice(M->device);
    void *ptrs[] = {M->tilePtr, M->tileColIdx, M->tileNnz, M->tileFmt, M->tileAux, M->tileOff,
                    M->payload, M->remRowPtr, M->remCol, M->remVal, M->items, M->split_info,
                    M->partials, M->counters, M->xstage, M->ystage, M->tdesc, M->cta_begin, M->blob,
                    M->witems, M->jcols, M->wfirst, M->units, M->xc_cols};
    for (void *p : ptrs)
        if (p) cudaFree(p);
    if (cur >= 0 && cur != M->device) cudaSetDevice(cur);
    delete M;
}

int64_t alg_bytes(const Matrix &M) {
    // DESIGN.md §"Bytes model": payload + 14 B of level-1 meta
    // per stored tile + tilePtr + remainder CSR (if any) + x read once + y
    // written once.
    int64_t b = M.payload_bytes + 14 * M.numtile + 4 * (M.tilem + 1) + 8 * M.n + 8 * M.m;
    if (M.rem_nnz > 0) b += 12 * M.rem_nnz + 4 * (M.m + 1);
    return b;
}

}  // namespace tsp

using namespace tsp;

extern "C" {

const char *tilespmv_status_string(int s) {
    switch (s) {
    case TILESPMV_OK: return "ok";
    case TILESPMV_INVALID_ARG: return "invalid argument";
    case TILESPMV_NOT_CANONICAL: return "input CSR is not canonical";
    case TILESPMV_OVERFLOW: return "size overflow";
    case TILESPMV_OOM: return "out of memory";
    case TILESPMV_CUDA: return "CUDA error";
    default: return "unknown status";
    }
}

const char *tilespmv_last_error(void) { return g_last_error.c_str(); }

int tilespmv_create_from_csr(tilespmv_handle_t *out, int64_t m, int64_t n, int64_t nnz,
                             const int32_t *d_rowptr, const int32_t *d_colidx, const double *d_val,
                             const tilespmv_opts_t *opts, void *stream) {
    g_last_error.clear();
    if (!out) return set_error(TILESPMV_INVALID_ARG, "out is NULL");
    *out = nullptr;
    if (m < 0 || n < 0 || nnz < 0) return set_error(TILESPMV_INVALID_ARG, "negative size");
    if (m >= (int64_t(1) << 31) - 16 || n >= (int64_t(1) << 31) - 16 || nnz >= (int64_t(1) << 31) - 1)
        return set_error(TILESPMV_OVERFLOW, "m, n must be < 2^31 - 16 and nnz < 2^31 - 1");
    if (!d_rowptr) return set_error(TILESPMV_INVALID_ARG, "rowptr is NULL");
    if (m == 0 && nnz != 0) return set_error(TILESPMV_NOT_CANONICAL, "m == 0 requires nnz == 0");
    if (nnz > 0 && (!d_colidx || !d_val)) return set_error(TILESPMV_INVALID_ARG, "colidx/val is NULL");
    tilespmv_opts_t o{TILESPMV_MODE_DEFERRED, 1, TILESPMV_KERNEL_AUTO, 0};
    if (opts) o = *opts;
    if (o.mode < 0 || o.mode > TILESPMV_MODE_BYTES) return set_error(TILESPMV_INVALID_ARG, "unknown mode");
    if (o.kernel < TILESPMV_KERNEL_AUTO || o.kernel > TILESPMV_KERNEL_GATHER)
        return set_error(TILESPMV_INVALID_ARG, "unknown kernel");
    if (o.keep_layout != 0 && o.keep_layout != 1) return set_error(TILESPMV_INVALID_ARG, "keep_layout must be 0 or 1");
    auto t0 = std::chrono::steady_clock::now();
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    tilespmv_matrix *M = new (std::nothrow) tilespmv_matrix();
    if (!M) return set_error(TILESPMV_OOM, "host allocation failed");
    if (cudaGetDevice(&M->device) != cudaSuccess) {
        delete M;
        return cuda_status(cudaGetLastError(), "cudaGetDevice");
    }
    {  // the CSR arrays must live on the current device
        const void *ptrs[3] = {d_rowptr, nnz > 0 ? d_colidx : nullptr, nnz > 0 ? d_val : nullptr};
        const char *names[3] = {"rowptr", "colidx", "val"};
        for (int i = 0; i < 3; ++i) {
            if (!ptrs[i]) continue;
            cudaPointerAttributes a;
            if (cudaPointerGetAttributes(&a, ptrs[i]) != cudaSuccess || a.type != cudaMemoryTypeDevice ||
                a.device != M->device) {
                cudaGetLastError();
                delete M;
                return set_error(TILESPMV_INVALID_ARG,
                                 std::string(names[i]) + " is not device memory of the current device");
            }
        }
    }
    M->m = m;
    M->n = n;
    M->nnz = nnz;
    M->mode = o.mode == TILESPMV_MODE_AUTO ? (nnz >= 1800000 ? TILESPMV_MODE_DEFERRED : TILESPMV_MODE_ADPT)
                                           : o.mode;
    M->keep_layout = o.keep_layout != 0;
    int rc = build_tiled(*M, d_rowptr, d_colidx, d_val, o.validate, st);
    if (!rc) rc = choose_kernel(*M, o.kernel);
    if (!rc) rc = build_schedule(*M, st);
    if (!rc) rc = build_tdesc(*M, st);
    if (!rc) rc = configure_launch(*M, st);
    if (!rc) release_create_time(*M, st);
    if (!rc) {
        cudaError_t e = cudaStreamSynchronize(st);
        if (e != cudaSuccess) rc = cuda_status(e, "cudaStreamSynchronize(create)");
    }
    if (rc) {
        cudaStreamSynchronize(st);
        free_matrix(M);
        return rc;
    }
    M->create_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    *out = M;
    return TILESPMV_OK;
}

static int check_handle(tilespmv_handle_t h) {
    if (!h) return set_error(TILESPMV_INVALID_ARG, "handle is NULL");
    int cur = -1;
    if (cudaGetDevice(&cur) != cudaSuccess) return cuda_status(cudaGetLastError(), "cudaGetDevice");
    if (cur != h->device) return set_error(TILESPMV_INVALID_ARG, "handle belongs to another device");
    return 0;
}

int tilespmv_run(tilespmv_handle_t h, const double *d_x, double *d_y, void *stream) {
    if (int rc = check_handle(h)) return rc;
    if (h->m > 0 && !d_y) return set_error(TILESPMV_INVALID_ARG, "y is NULL");
    if (h->n > 0 && !d_x) return set_error(TILESPMV_INVALID_ARG, "x is NULL");
    if (h->m > 0 && h->n > 0) {
        const char *xa = reinterpret_cast<const char *>(d_x), *ya = reinterpret_cast<const char *>(d_y);
        if (xa < ya + 8 * h->m && ya < xa + 8 * h->n) return set_error(TILESPMV_INVALID_ARG, "x and y overlap");
    }
    return launch_spmv(*h, d_x, d_y, static_cast<cudaStream_t>(stream));
}

int tilespmv_run_scatter(tilespmv_handle_t h, const double *d_x, double *d_y, double *const *d_peer_ys,
                         int32_t n_peer, void *stream) {
    if (n_peer < 0 || n_peer > kMaxScatter) return set_error(TILESPMV_INVALID_ARG, "n_peer must be 0..7");
    if (n_peer > 0 && !d_peer_ys) return set_error(TILESPMV_INVALID_ARG, "d_peer_ys is NULL");
    double *ys[kMaxScatter] = {nullptr};
    for (int t = 0; t < n_peer; ++t) {
        if (h && h->m > 0 && !d_peer_ys[t]) return set_error(TILESPMV_INVALID_ARG, "a peer y is NULL");
        ys[t] = d_peer_ys[t];
    }
    if (int rc = check_handle(h)) return rc;
    if (h->m > 0 && !d_y) return set_error(TILESPMV_INVALID_ARG, "y is NULL");
    if (h->n > 0 && !d_x) return set_error(TILESPMV_INVALID_ARG, "x is NULL");
    if (h->m > 0 && h->n > 0) {
        const char *xa = reinterpret_cast<const char *>(d_x), *ya = reinterpret_cast<const char *>(d_y);
        if (xa < ya + 8 * h->m && ya < xa + 8 * h->n) return set_error(TILESPMV_INVALID_ARG, "x and y overlap");
    }
    return launch_spmv(*h, d_x, d_y, static_cast<cudaStream_t>(stream), ys, n_peer);
}

int tilespmv_ipc_alloc(int64_t bytes, void **d_ptr, void *handle) {
    if (!d_ptr || !handle || bytes <= 0) return set_error(TILESPMV_INVALID_ARG, "bad ipc_alloc arguments");
    *d_ptr = nullptr;
    void *p = nullptr;
    if (cudaMalloc(&p, (size_t)bytes) != cudaSuccess) return cuda_status(cudaGetLastError(), "cudaMalloc(ipc buffer)");
    cudaIpcMemHandle_t hd;
    cudaError_t e = cudaIpcGetMemHandle(&hd, p);
    if (e != cudaSuccess) {
        cudaFree(p);
        return cuda_status(e, "cudaIpcGetMemHandle");
    }
    std::memcpy(handle, &hd, sizeof(hd));
    *d_ptr = p;
    return TILESPMV_OK;
}

int tilespmv_ipc_free(void *d_ptr) {
    if (d_ptr && cudaFree(d_ptr) != cudaSuccess) return cuda_status(cudaGetLastError(), "cudaFree(ipc buffer)");
    return TILESPMV_OK;
}

int tilespmv_ipc_open(const void *handle, void **d_ptr) {
    if (!handle || !d_ptr) return set_error(TILESPMV_INVALID_ARG, "bad ipc_open arguments");
    *d_ptr = nullptr;
    cudaIpcMemHandle_t hd;
    std::memcpy(&hd, handle, sizeof(hd));
    cudaError_t e = cudaIpcOpenMemHandle(d_ptr, hd, cudaIpcMemLazyEnablePeerAccess);
    if (e != cudaSuccess) return cuda_status(e, "cudaIpcOpenMemHandle");
    return TILESPMV_OK;
}

int tilespmv_ipc_close(void *d_ptr) {
    if (d_ptr && cudaIpcCloseMemHandle(d_ptr) != cudaSuccess)
        return cuda_status(cudaGetLastError(), "cudaIpcCloseMemHandle");
    return TILESPMV_OK;
}

int tilespmv_run_host(tilespmv_handle_t h, const double *h_x, double *h_y, void *stream) {
    if (int rc = check_handle(h)) return rc;
    if ((h->m > 0 && !h_y) || (h->n > 0 && !h_x)) return set_error(TILESPMV_INVALID_ARG, "NULL host buffer");
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    if (!h->xstage || !h->ystage) {  // both staging buffers or neither
        double *xs = nullptr, *ys = nullptr;
        if (cudaMalloc(&xs, std::max<int64_t>(h->n, 1) * 8) != cudaSuccess ||
            cudaMalloc(&ys, std::max<int64_t>(h->m, 1) * 8) != cudaSuccess) {
            const int rc = cuda_status(cudaGetLastError(), "cudaMalloc(host-staging buffers)");
            if (xs) cudaFree(xs);
            return rc;
        }
        h->xstage = xs;
        h->ystage = ys;
        h->device_bytes += 8 * (h->m + h->n);
    }
    cudaError_t e;
    if (h->n > 0 && (e = cudaMemcpyAsync(h->xstage, h_x, h->n * 8, cudaMemcpyHostToDevice, st)) != cudaSuccess)
        return cuda_status(e, "cudaMemcpyAsync(x)");
    if (int rc = launch_spmv(*h, h->xstage, h->ystage, st)) return rc;
    if (h->m > 0 && (e = cudaMemcpyAsync(h_y, h->ystage, h->m * 8, cudaMemcpyDeviceToHost, st)) != cudaSuccess)
        return cuda_status(e, "cudaMemcpyAsync(y)");
    if ((e = cudaStreamSynchronize(st)) != cudaSuccess) return cuda_status(e, "cudaStreamSynchronize");
    return TILESPMV_OK;
}

int tilespmv_cg(tilespmv_handle_t h, const double *d_b, double *d_x, double tol, int32_t maxit, int32_t *iters,
                double *relres, void *stream) {
    if (int rc = check_handle(h)) return rc;
    if (h->m != h->n) return set_error(TILESPMV_INVALID_ARG, "CG needs a square matrix");
    if (h->n > 0 && (!d_b || !d_x)) return set_error(TILESPMV_INVALID_ARG, "NULL vector");
    if (!(tol >= 0.0) || maxit < 0) return set_error(TILESPMV_INVALID_ARG, "tol must be >= 0 and maxit >= 0");
    if (h->n > 0 && d_b < d_x + h->n && d_x < d_b + h->n) return set_error(TILESPMV_INVALID_ARG, "b and x overlap");
    int it = 0;
    double rel = 0.0;
    if (h->n > 0) {
        if (int rc = cg_solve(*h, d_b, d_x, tol, maxit, &it, &rel, static_cast<cudaStream_t>(stream))) return rc;
    }
    if (iters) *iters = it;
    if (relres) *relres = rel;
    return TILESPMV_OK;
}

int tilespmv_destroy(tilespmv_handle_t h) {
    if (!h) return TILESPMV_OK;
    free_matrix(h);
    return TILESPMV_OK;
}

int tilespmv_get_info(tilespmv_handle_t h, tilespmv_info_t *info) {
    if (!h || !info) return set_error(TILESPMV_INVALID_ARG, "NULL argument");
    std::memset(info, 0, sizeof *info);
    info->m = h->m;
    info->n = h->n;
    info->nnz = h->nnz;
    info->tilem = h->tilem;
    info->tilen = h->tilen;
    info->numtile = h->numtile;
    info->mode = h->mode;
    info->device = h->device;
    for (int f = 0; f < 7; ++f) {
        info->sel_tiles[f] = h->sel_tiles[f];
        info->sel_nnz[f] = h->sel_nnz[f];
        info->kept_tiles[f] = h->kept_tiles[f];
        info->kept_nnz[f] = h->kept_nnz[f];
    }
    info->rem_nnz = h->rem_nnz;
    info->payload_bytes = h->payload_bytes;
    info->meta_bytes = 14 * h->numtile + 4 * (h->tilem + 1);
    info->alg_bytes = alg_bytes(*h);
    info->flops = 2 * h->nnz;
    info->num_items = h->num_items;
    info->num_split_rows = h->num_split;
    info->device_bytes = h->device_bytes;
    info->create_ms = h->create_ms;
    info->kernel = h->kernel;
    info->xcache_cols = h->xc_n;
    return TILESPMV_OK;
}

static int64_t export_size(const Matrix &M, int32_t which, const void **src) {
    const void *p = nullptr;
    int64_t b = -1;
    switch (which) {
    case TILESPMV_ARR_TILEPTR: p = M.tilePtr; b = 4 * (M.tilem + 1); break;
    case TILESPMV_ARR_TILECOLIDX: p = M.tileColIdx; b = 4 * M.numtile; break;
    case TILESPMV_ARR_TILENNZ: p = M.tileNnz; b = 4 * (M.numtile + 1); break;
    case TILESPMV_ARR_TILEFMT: p = M.tileFmt; b = M.numtile; break;
    case TILESPMV_ARR_TILEAUX: p = M.tileAux; b = M.numtile; break;
    case TILESPMV_ARR_TILEOFF: p = M.tileOff; b = 4 * (M.numtile + 1); break;
    case TILESPMV_ARR_PAYLOAD: p = M.payload; b = M.payload_bytes; break;
    case TILESPMV_ARR_REMROWPTR: p = M.remRowPtr; b = M.rem_nnz > 0 ? 4 * (M.m + 1) : 0; break;
    case TILESPMV_ARR_REMCOL: p = M.remCol; b = 4 * M.rem_nnz; break;
    case TILESPMV_ARR_REMVAL: p = M.remVal; b = 8 * M.rem_nnz; break;
    default: return TILESPMV_INVALID_ARG;
    }
    if (src) *src = p;
    return b;
}

int64_t tilespmv_export_size(tilespmv_handle_t h, int32_t which) {
    if (!h) return set_error(TILESPMV_INVALID_ARG, "handle is NULL");
    int64_t b = export_size(*h, which, nullptr);
    if (b < 0) return set_error(TILESPMV_INVALID_ARG, "unknown array id");
    return b;
}

int tilespmv_export(tilespmv_handle_t h, int32_t which, void *host_dst, size_t bytes) {
    if (int rc = check_handle(h)) return rc;
    const void *src = nullptr;
    int64_t b = export_size(*h, which, &src);
    if (b < 0) return set_error(TILESPMV_INVALID_ARG, "unknown array id");
    if ((int64_t)bytes != b) return set_error(TILESPMV_INVALID_ARG, "byte count mismatch");
    if (b == 0) return TILESPMV_OK;
    if (!h->keep_layout)
        return set_error(TILESPMV_INVALID_ARG, "the canonical layout was not kept (create with opts.keep_layout = 1)");
    if (!host_dst) return set_error(TILESPMV_INVALID_ARG, "host_dst is NULL");
    cudaError_t e = cudaMemcpy(host_dst, src, b, cudaMemcpyDeviceToHost);
    if (e != cudaSuccess) return cuda_status(e, "cudaMemcpy(export)");
    return TILESPMV_OK;
}

int tilespmv_launch_shape(tilespmv_handle_t h, int32_t *grid, int32_t *block, int32_t *smem_bytes) {
    if (!h) return set_error(TILESPMV_INVALID_ARG, "handle is NULL");
    if (grid) *grid = h->grid;
    if (block) *block = h->block;
    if (smem_bytes) *smem_bytes = h->smem;
    return TILESPMV_OK;
}

const char *tilespmv_kernel_name(tilespmv_handle_t h) { return h ? h->kernel_name : ""; }

int32_t tilespmv_auto_kernel(int64_t payload_bytes, int64_t tilem, int64_t rem_nnz, int64_t alg) {
    return auto_kernel(payload_bytes, tilem, rem_nnz, alg);
}

}  // extern "C"
