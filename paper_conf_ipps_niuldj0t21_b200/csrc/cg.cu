// cg.cu -- conjugate-gradient solve on top of the tiled SpMV (SURVEY §8(f)
// f4: the iterative-solver use the paper motivates SpMV with).
//
// Hestenes-Stiefel CG (the textbook algorithm, e.g. Saad, "Iterative Methods
// for Sparse Linear Systems", Alg. 6.18), fp64, A symmetric positive definite:
//   r0 = b - A x0, p0 = r0
//   for j = 0, 1, ...:  q = A p_j                     (tilespmv kernel)
//                       alpha = (r_j, r_j) / (p_j, q)
//                       x_{j+1} = x_j + alpha p_j,  r_{j+1} = r_j - alpha q
//                       stop if ||r_{j+1}|| <= tol ||b||
//                       beta = (r_{j+1}, r_{j+1}) / (r_j, r_j)
//                       p_{j+1} = r_{j+1} + beta p_j
// One iteration = the SpMV + three vector kernels.  Dot products are
// deterministic: every block reduces a fixed grid-stride set in a fixed tree
// into one partial, and consumers sum the partials in index order, so the
// iterates are bitwise reproducible run to run.  The scalars never leave the
// device; a device flag freezes x once converged, and the host polls it every
// kCheckEvery iterations.
#include <algorithm>
#include <cmath>

#include "spmv_common.cuh"

namespace tsp {
namespace {

constexpr int kBlocks = 296;  // 2 x 148 SMs
constexpr int kThreads = 256;
constexpr int kCheckEvery = 8;

struct CgState {
    double bb;                 // (b, b)
    double rr;                 // (r_j, r_j) of the last finished iteration (host poll)
    int done;                  // converged: later kernels return at once
    int iters;                 // iterations finished
    double pq[kBlocks];        // partials of (p, q)
    double rrp[2][kBlocks];    // partials of (r_j, r_j), by parity of j
    double bbp[kBlocks];       // partials of (b, b)
};

__device__ __forceinline__ double block_sum(double v, double *sh) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
#pragma unroll
    for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(FULL, v, o);
    if (lane == 0) sh[w] = v;
    __syncthreads();
    double s = 0.0;
    if (threadIdx.x == 0)
        for (int i = 0; i < kThreads / 32; ++i) s += sh[i];
    __syncthreads();
    return s;  // valid in thread 0
}

// sum of kBlocks partials in a fixed order (every thread gets the result)
__device__ __forceinline__ double sum_partials(const double *part, double *sh) {
    double v = 0.0;
    for (int i = threadIdx.x; i < kBlocks; i += kThreads) v += part[i];
    const double s = block_sum(v, sh);
    if (threadIdx.x == 0) sh[32] = s;
    __syncthreads();
    const double r = sh[32];
    __syncthreads();
    return r;
}

// r = b - q (q = A x0), p = r; partials of (r, r) and (b, b)
__global__ void k_cg_init(const double *b, const double *q, double *r, double *p, int64_t n, CgState *st) {
    __shared__ double sh[40];
    double rr = 0.0, bb = 0.0;
    for (int64_t i = blockIdx.x * (int64_t)kThreads + threadIdx.x; i < n; i += (int64_t)kBlocks * kThreads) {
        const double ri = b[i] - q[i];
        r[i] = ri;
        p[i] = ri;
        rr = fma(ri, ri, rr);
        bb = fma(b[i], b[i], bb);
    }
    const double s1 = block_sum(rr, sh), s2 = block_sum(bb, sh);
    if (threadIdx.x == 0) {
        st->rrp[0][blockIdx.x] = s1;
        st->bbp[blockIdx.x] = s2;
    }
}

__global__ void k_cg_init_scalars(CgState *st) {
    __shared__ double sh[40];
    const double rr = sum_partials(st->rrp[0], sh), bb = sum_partials(st->bbp, sh);
    if (threadIdx.x == 0) {
        st->rr = rr;
        st->bb = bb;
        st->done = rr == 0.0 ? 1 : 0;
        st->iters = 0;
    }
}

// partials of (p, q)
__global__ void k_cg_pq(const double *p, const double *q, int64_t n, CgState *st) {
    if (st->done) return;
    __shared__ double sh[40];
    double s = 0.0;
    for (int64_t i = blockIdx.x * (int64_t)kThreads + threadIdx.x; i < n; i += (int64_t)kBlocks * kThreads)
        s = fma(p[i], q[i], s);
    s = block_sum(s, sh);
    if (threadIdx.x == 0) st->pq[blockIdx.x] = s;
}

// alpha = (r_j, r_j) / (p_j, q); x += alpha p; r -= alpha q; partials of (r_{j+1}, r_{j+1})
__global__ void k_cg_update(double *x, double *r, const double *p, const double *q, int64_t n, int j, CgState *st) {
    if (st->done) return;
    __shared__ double sh[40];
    const double rr = sum_partials(st->rrp[j & 1], sh), pq = sum_partials(st->pq, sh);
    const double alpha = rr / pq;
    double s = 0.0;
    for (int64_t i = blockIdx.x * (int64_t)kThreads + threadIdx.x; i < n; i += (int64_t)kBlocks * kThreads) {
        x[i] = fma(alpha, p[i], x[i]);
        const double ri = fma(-alpha, q[i], r[i]);
        r[i] = ri;
        s = fma(ri, ri, s);
    }
    s = block_sum(s, sh);
    if (threadIdx.x == 0) st->rrp[(j + 1) & 1][blockIdx.x] = s;
}

// convergence test; beta = (r_{j+1}, r_{j+1}) / (r_j, r_j); p = r + beta p
__global__ void k_cg_direction(double *p, const double *r, int64_t n, int j, double tol2, CgState *st) {
    if (st->done) return;
    __shared__ double sh[40];
    const double rr0 = sum_partials(st->rrp[j & 1], sh), rr1 = sum_partials(st->rrp[(j + 1) & 1], sh);
    const bool conv = rr1 <= tol2 * st->bb;
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        st->rr = rr1;
        st->iters = j + 1;
    }
    if (conv) {
        // every block sees the same rr1, so all skip the update; block 0 raises the flag
        if (blockIdx.x == 0 && threadIdx.x == 0) st->done = 1;
        return;
    }
    const double beta = rr1 / rr0;
    for (int64_t i = blockIdx.x * (int64_t)kThreads + threadIdx.x; i < n; i += (int64_t)kBlocks * kThreads)
        p[i] = fma(beta, p[i], r[i]);
}

}  // namespace

int cg_solve(const Matrix &M, const double *d_b, double *d_x, double tol, int maxit, int *iters, double *relres,
             cudaStream_t st) {
    const int64_t n = M.n;
    CgState *S = nullptr;
    double *work = nullptr;
    cudaError_t e = cudaMallocAsync(reinterpret_cast<void **>(&S), sizeof(CgState), st);
    if (e != cudaSuccess) return cuda_status(e, "cudaMallocAsync(cg state)");
    e = cudaMallocAsync(reinterpret_cast<void **>(&work), 3 * std::max<int64_t>(n, 1) * sizeof(double), st);
    if (e != cudaSuccess) {
        cudaFreeAsync(S, st);
        return cuda_status(e, "cudaMallocAsync(cg vectors)");
    }
    double *r = work, *p = work + n, *q = work + 2 * n;
    int rc = 0;
    struct {
        double bb, rr;
        int done, iters;
    } h{};
    do {
        if ((rc = launch_spmv(M, d_x, q, st))) break;  // q = A x0
        k_cg_init<<<kBlocks, kThreads, 0, st>>>(d_b, q, r, p, n, S);
        k_cg_init_scalars<<<1, kThreads, 0, st>>>(S);
        const double tol2 = tol * tol;
        int j = 0;
        for (; j < maxit; ++j) {
            if ((rc = launch_spmv(M, p, q, st))) break;
            k_cg_pq<<<kBlocks, kThreads, 0, st>>>(p, q, n, S);
            k_cg_update<<<kBlocks, kThreads, 0, st>>>(d_x, r, p, q, n, j, S);
            k_cg_direction<<<kBlocks, kThreads, 0, st>>>(p, r, n, j, tol2, S);
            if ((j + 1) % kCheckEvery == 0 || j + 1 == maxit) {
                if ((e = cudaMemcpyAsync(&h, S, sizeof h, cudaMemcpyDeviceToHost, st)) != cudaSuccess ||
                    (e = cudaStreamSynchronize(st)) != cudaSuccess) {
                    rc = cuda_status(e, "cg poll");
                    break;
                }
                if (h.done) break;
            }
        }
        if (rc) break;
        if ((e = cudaMemcpyAsync(&h, S, sizeof h, cudaMemcpyDeviceToHost, st)) != cudaSuccess ||
            (e = cudaStreamSynchronize(st)) != cudaSuccess) {
            rc = cuda_status(e, "cg result");
            break;
        }
        if (iters) *iters = h.iters;
        if (relres) *relres = h.bb > 0.0 ? std::sqrt(h.rr / h.bb) : 0.0;
    } while (0);
    cudaFreeAsync(work, st);
    cudaFreeAsync(S, st);
    if (!rc && (e = cudaStreamSynchronize(st)) != cudaSuccess) rc = cuda_status(e, "cg free");
    return rc;
}

}  // namespace tsp
