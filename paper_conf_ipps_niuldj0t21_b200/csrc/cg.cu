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

// one wave of 6 blocks of 8 warps per SM (48 warps; the update kernel's 42
// registers allow 6): the vector kernels are HBM-bound and need many loads
// in flight, every thread moves double2 pairs.  Measured per CG iteration on
// C5: 296 blocks 0.609 ms, 888 blocks 0.558 ms, 1184 (1.3 waves) 0.796 ms.
// TILESPMV_CG_BLOCKS overrides the grid (<= kBlocks partial slots).
constexpr int kBlocks = 6 * 148;
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

// sum of the G partials of a grid in a fixed order (every thread gets the result)
__device__ __forceinline__ double sum_partials(const double *part, double *sh, int G = (int)gridDim.x) {
    double v = 0.0;
    for (int i = threadIdx.x; i < G; i += kThreads) v += part[i];
    const double s = block_sum(v, sh);
    if (threadIdx.x == 0) sh[32] = s;
    __syncthreads();
    const double r = sh[32];
    __syncthreads();
    return r;
}

// Element loops: thread t of block g takes the pairs (2i, 2i+1) for i = g *
// kThreads + t + k * gridDim.x * kThreads (16-byte loads; vectors come from
// cudaMalloc or torch, 16-byte aligned), and block 0's thread 0 the last
// element when n is odd.  The partial sums follow that fixed order.
#define CG_PAIRS(i2) \
    for (int64_t i2 = blockIdx.x * (int64_t)kThreads + threadIdx.x; i2 < (n >> 1); i2 += (int64_t)gridDim.x * kThreads)
#define CG_TAIL(i) \
    if ((n & 1) && blockIdx.x == 0 && threadIdx.x == 0) \
        for (int64_t i = n - 1; i < n; ++i)

__device__ __forceinline__ double2 ld2(const double *a, int64_t i2) { return reinterpret_cast<const double2 *>(a)[i2]; }
__device__ __forceinline__ void st2(double *a, int64_t i2, double2 v) { reinterpret_cast<double2 *>(a)[i2] = v; }

// r = b - q (q = A x0), p = r; partials of (r, r) and (b, b)
__global__ void k_cg_init(const double *b, const double *q, double *r, double *p, int64_t n, CgState *st) {
    __shared__ double sh[40];
    double rr = 0.0, bb = 0.0;
    CG_PAIRS(i2) {
        const double2 bi = ld2(b, i2), qi = ld2(q, i2);
        const double2 ri = make_double2(bi.x - qi.x, bi.y - qi.y);
        st2(r, i2, ri);
        st2(p, i2, ri);
        rr = fma(ri.x, ri.x, rr);
        rr = fma(ri.y, ri.y, rr);
        bb = fma(bi.x, bi.x, bb);
        bb = fma(bi.y, bi.y, bb);
    }
    CG_TAIL(i) {
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

__global__ void k_cg_init_scalars(CgState *st, int G) {  // G: k_cg_init's grid
    __shared__ double sh[40];
    const double rr = sum_partials(st->rrp[0], sh, G), bb = sum_partials(st->bbp, sh, G);
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
#pragma unroll 2
    CG_PAIRS(i2) {
        const double2 pi = ld2(p, i2), qi = ld2(q, i2);
        s = fma(pi.x, qi.x, s);
        s = fma(pi.y, qi.y, s);
    }
    CG_TAIL(i) s = fma(p[i], q[i], s);
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
#pragma unroll 2
    CG_PAIRS(i2) {
        const double2 xi = ld2(x, i2), pi = ld2(p, i2), qi = ld2(q, i2), r0 = ld2(r, i2);
        st2(x, i2, make_double2(fma(alpha, pi.x, xi.x), fma(alpha, pi.y, xi.y)));
        const double2 ri = make_double2(fma(-alpha, qi.x, r0.x), fma(-alpha, qi.y, r0.y));
        st2(r, i2, ri);
        s = fma(ri.x, ri.x, s);
        s = fma(ri.y, ri.y, s);
    }
    CG_TAIL(i) {
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
#pragma unroll 2
    CG_PAIRS(i2) {
        const double2 pi = ld2(p, i2), ri = ld2(r, i2);
        st2(p, i2, make_double2(fma(beta, pi.x, ri.x), fma(beta, pi.y, ri.y)));
    }
    CG_TAIL(i) p[i] = fma(beta, p[i], r[i]);
}

}  // namespace

int cg_solve(const Matrix &M, const double *d_b, double *d_x, double tol, int maxit, int *iters, double *relres,
             cudaStream_t st) {
    const int64_t n = M.n;
    // the vector kernels move 16-byte pairs: every vector starts 16-byte
    // aligned (work vectors at an even stride; b and x staged when the
    // caller's are not)
    const int64_t n2 = (std::max<int64_t>(n, 1) + 1) & ~int64_t(1);
    const bool staged = ((reinterpret_cast<uintptr_t>(d_b) | reinterpret_cast<uintptr_t>(d_x)) & 15u) != 0;
    CgState *S = nullptr;
    double *work = nullptr;
    cudaError_t e = cudaMallocAsync(reinterpret_cast<void **>(&S), sizeof(CgState), st);
    if (e != cudaSuccess) return cuda_status(e, "cudaMallocAsync(cg state)");
    e = cudaMallocAsync(reinterpret_cast<void **>(&work), (staged ? 5 : 3) * n2 * sizeof(double), st);
    if (e != cudaSuccess) {
        cudaFreeAsync(S, st);
        return cuda_status(e, "cudaMallocAsync(cg vectors)");
    }
    double *r = work, *p = work + n2, *q = work + 2 * n2;
    double *const x_user = d_x;
    if (staged) {
        double *bs = work + 3 * n2, *xs = work + 4 * n2;
        cudaMemcpyAsync(bs, d_b, n * sizeof(double), cudaMemcpyDeviceToDevice, st);
        cudaMemcpyAsync(xs, d_x, n * sizeof(double), cudaMemcpyDeviceToDevice, st);
        d_b = bs;
        d_x = xs;
    }
    int rc = 0;
    struct {
        double bb, rr;
        int done, iters;
    } h{};
    do {
        if ((rc = launch_spmv(M, d_x, q, st))) break;  // q = A x0
        int G = kBlocks;
        k_cg_init<<<G, kThreads, 0, st>>>(d_b, q, r, p, n, S);
        k_cg_init_scalars<<<1, kThreads, 0, st>>>(S, G);
        const double tol2 = tol * tol;
        int j = 0;
        for (; j < maxit; ++j) {
            if ((rc = launch_spmv(M, p, q, st))) break;
            k_cg_pq<<<G, kThreads, 0, st>>>(p, q, n, S);
            k_cg_update<<<G, kThreads, 0, st>>>(d_x, r, p, q, n, j, S);
            k_cg_direction<<<G, kThreads, 0, st>>>(p, r, n, j, tol2, S);
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
        if (staged) cudaMemcpyAsync(x_user, d_x, n * sizeof(double), cudaMemcpyDeviceToDevice, st);
    } while (0);
    cudaFreeAsync(work, st);
    cudaFreeAsync(S, st);
    if (!rc && (e = cudaStreamSynchronize(st)) != cudaSuccess) rc = cuda_status(e, "cg free");
    return rc;
}

}  // namespace tsp
