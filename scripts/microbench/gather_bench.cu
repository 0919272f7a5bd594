// gather_bench.cu -- development microbenchmark (not part of the product):
// the x-gather ceiling of a CSR-remainder-like stream on B200.  Each thread
// walks entries i = tid, tid + stride, ... (coalesced col/val reads) and
// accumulates val[i] * x[col[i]]; variants differ in the load flavour of the
// gather and in the shared-memory carve-out (dynamic smem per CTA).
#include <cuda_runtime.h>
#include <stdint.h>

template <int KIND>
__device__ __forceinline__ double gx(const double *p, uint64_t pol) {
    double v;
    if (KIND == 0) asm volatile("ld.global.nc.f64 %0, [%1];" : "=d"(v) : "l"(p));
    if (KIND == 1) asm volatile("ld.global.cg.f64 %0, [%1];" : "=d"(v) : "l"(p));
    if (KIND == 2) asm volatile("ld.global.nc.L2::cache_hint.f64 %0, [%1], %2;" : "=d"(v) : "l"(p), "l"(pol));
    if (KIND == 3) asm volatile("ld.global.ca.f64 %0, [%1];" : "=d"(v) : "l"(p));
    if (KIND == 4) asm volatile("ld.global.nc.L1::no_allocate.f64 %0, [%1];" : "=d"(v) : "l"(p));
    return v;
}

// KIND 5: the column's top bit marks a cold line (read around the L1: no
// allocation), hot lines (the most-gathered ones) allocate in L1
__device__ __forceinline__ double gsplit(const double *x, int c) {
    double v;
    const double *p = x + (c & 0x7FFFFFFF);
    if (c < 0) asm volatile("ld.global.nc.L1::no_allocate.f64 %0, [%1];" : "=d"(v) : "l"(p));
    else asm volatile("ld.global.nc.f64 %0, [%1];" : "=d"(v) : "l"(p));
    return v;
}

template <int KIND, int U>
__global__ void k_gather(const int32_t *col, const double *val, const double *x, int64_t n, double *out) {
    extern __shared__ uint8_t smem[];
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
    const int64_t tid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    double acc = 0.0;
    int64_t i = tid;
    for (; i + (U - 1) * stride < n; i += U * stride) {
        int c[U];
        double v[U], xv[U];
#pragma unroll
        for (int u = 0; u < U; ++u) { c[u] = __ldcs(col + i + u * stride); v[u] = __ldcs(val + i + u * stride); }
#pragma unroll
        for (int u = 0; u < U; ++u) xv[u] = KIND == 5 ? gsplit(x, c[u]) : gx<KIND>(x + c[u], pol);
#pragma unroll
        for (int u = 0; u < U; ++u) acc += v[u] * xv[u];
    }
    for (; i < n; i += stride) acc += val[i] * (KIND == 5 ? gsplit(x, col[i]) : gx<KIND>(x + col[i], pol));
    if (acc == 123.456) smem[0] = 1;  // keep smem "used"
    out[tid] = acc;
}

typedef void (*kfn)(const int32_t *, const double *, const double *, int64_t, double *);

static kfn pick(int kind, int u) {
#define K(KD, UU) if (kind == KD && u == UU) return k_gather<KD, UU>;
    K(0, 1) K(0, 4) K(0, 8) K(1, 1) K(1, 4) K(1, 8) K(2, 1) K(2, 4) K(2, 8) K(3, 4) K(3, 8) K(4, 4) K(4, 8) K(5, 4) K(5, 8)
    return nullptr;
}

extern "C" int gather_bench(int kind, int unroll, int blocks, int threads, int smem, const int32_t *col,
                            const double *val, const double *x, int64_t n, double *out, int reps, float *ms) {
    kfn f = pick(kind, unroll);
    if (!f) return -1;
    cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    f<<<blocks, threads, smem>>>(col, val, x, n, out);
    cudaEventRecord(a);
    for (int r = 0; r < reps; ++r) f<<<blocks, threads, smem>>>(col, val, x, n, out);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    cudaEventElapsedTime(ms, a, b);
    *ms /= reps;
    cudaEventDestroy(a);
    cudaEventDestroy(b);
    return cudaGetLastError() == cudaSuccess ? 0 : -2;
}
