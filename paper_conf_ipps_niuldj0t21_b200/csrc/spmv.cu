// spmv.cu -- the timed hot path: y = A_tiles * x + A_rem * x in fp64
// (§III.C P:118-173 warp-level tile kernels, P:199 load balancing,
// P:201 DeferredCOO remainder), written for sm_100a.
//
// Design (DESIGN.md §"SpMV kernel"):
//   * persistent warps; each warp walks work items (byte-bounded pieces of
//     one tile row, see internal.cuh);
//   * a work item's tile payloads are one contiguous 16-byte-aligned byte
//     range, staged into the warp's shared-memory slot with ONE
//     cp.async.bulk (TMA, 1-D) completing on an mbarrier;
//   * the 16-entry x segment of each tile (one 128-byte line) is gathered
//     into shared memory by the warp (the paper's "x in on-chip memory",
//     P:122);
//   * lane l owns row (l & 15) of the tile row; every column-major format
//     (ELL, Dns, DnsCol, HYB-ELL) maps slot s to lane s mod 32 so the only
//     reduction is acc(l) + acc(l+16); row-major formats (CSR, COO,
//     HYB-COO) use the paper's two lanes per row; DnsRow reduces a
//     dense row with a 16-lane shuffle tree;
//   * the CSR remainder rows of the tile row are fused into the same item
//     (two lanes per short row, the whole warp per long row);
//   * y is written once per row with a 128-byte store; no floating-point
//     atomics anywhere, so y is bitwise deterministic.
#include <algorithm>
#include <cstdio>

#include "internal.cuh"

namespace tsp {

#define TSP_CK(call)                                                   \
    do {                                                               \
        cudaError_t e_ = (call);                                       \
        if (e_ != cudaSuccess) return cuda_status(e_, #call);          \
    } while (0)

namespace {

constexpr int kWarps = 4;                                   // warps per CTA
constexpr int kXBytes = kItemTiles * 16 * 8;                // x segments per item
constexpr int kWarpSmem = kItemPayload + kXBytes + 128;     // + mbarrier slot
constexpr int kSmemBytes = kWarps * kWarpSmem;
constexpr unsigned FULL = 0xffffffffu;

struct Params {
    const Item *items;
    int64_t num_items;
    const int32_t *tileColIdx;
    const uint8_t *tileFmt;
    const uint8_t *tileAux;
    const int32_t *tileNnz;
    const uint32_t *tileOff;
    const uint8_t *payload;
    const int32_t *remRowPtr;
    const int32_t *remCol;
    const double *remVal;
    const int2 *split_info;
    double *partials;
    int32_t *counters;
    const double *x;
    double *y;
    int64_t m, n;
};

// ---------------------------------------------------------------- PTX -----
__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void fence_proxy_async() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint32_t bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void bulk_g2s(uint32_t dst, const void *src, uint32_t bytes, uint32_t bar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
        "l"(src), "r"(bytes), "r"(bar)
        : "memory");
}
__device__ __forceinline__ bool mbar_try_wait(uint32_t bar, uint32_t parity) {
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(ok)
        : "r"(bar), "r"(parity)
        : "memory");
    return ok != 0;
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
    while (!mbar_try_wait(bar, parity)) {
    }
}
__device__ __forceinline__ int nib(const uint8_t *base, int idx) {
    return (base[idx >> 1] >> ((idx & 1) * 4)) & 15;
}

// ------------------------------------------------------- remainder rows ---
// Adds sum_{k in row r, k in [kb,ke)} remVal[k] * x[remCol[k]] to the owner
// lane of row r.  Rows of at most kShortRow entries: two lanes per row
// (lane l takes entries h, h+2, ... of row l & 15, h = l >> 4); longer rows:
// the whole warp strides the row and reduces with a butterfly.
__device__ __forceinline__ void remainder_rows(const Params &p, int64_t I, int kb, int ke, int lane,
                                               double &acc) {
    const int r = lane & 15, h = lane >> 4;
    int64_t row = 16 * I + (lane < 17 ? lane : 16);
    if (row > p.m) row = p.m;
    int rp = __ldg(p.remRowPtr + row);
    int b = __shfl_sync(FULL, rp, r), e = __shfl_sync(FULL, rp, r + 1);
    b = max(b, kb);
    e = min(e, ke);
    const int len = max(e - b, 0);
    const bool is_short = len <= kShortRow;
    {
        int cs[kShortRow / 2];
        double vs[kShortRow / 2], xs[kShortRow / 2];
#pragma unroll
        for (int i = 0; i < kShortRow / 2; ++i) {
            int k = b + h + 2 * i;
            bool ok = is_short && k < e;
            cs[i] = ok ? __ldg(p.remCol + k) : 0;
            vs[i] = ok ? __ldg(p.remVal + k) : 0.0;
        }
#pragma unroll
        for (int i = 0; i < kShortRow / 2; ++i) {
            int k = b + h + 2 * i;
            xs[i] = (is_short && k < e) ? __ldg(p.x + cs[i]) : 0.0;
        }
#pragma unroll
        for (int i = 0; i < kShortRow / 2; ++i) {
            int k = b + h + 2 * i;
            if (is_short && k < e) acc = fma(vs[i], xs[i], acc);
        }
    }
    unsigned longs = __ballot_sync(FULL, lane < 16 && !is_short);
    while (longs) {
        const int rr = __ffs(longs) - 1;
        longs &= longs - 1;
        const int bb = __shfl_sync(FULL, b, rr), ee = __shfl_sync(FULL, e, rr);
        double s = 0.0;
        for (int k0 = bb; k0 < ee; k0 += 128) {
            int cs[4];
            double vs[4];
#pragma unroll
            for (int i = 0; i < 4; ++i) {
                int k = k0 + lane + 32 * i;
                cs[i] = k < ee ? __ldg(p.remCol + k) : 0;
                vs[i] = k < ee ? __ldg(p.remVal + k) : 0.0;
            }
#pragma unroll
            for (int i = 0; i < 4; ++i) {
                int k = k0 + lane + 32 * i;
                if (k < ee) s = fma(vs[i], __ldg(p.x + cs[i]), s);
            }
        }
#pragma unroll
        for (int o = 16; o >= 1; o >>= 1) s += __shfl_xor_sync(FULL, s, o);
        if (lane == rr) acc += s;
    }
}

// ------------------------------------------------------------ one tile ----
// P points at the tile's payload in shared memory, X at its 16 x values.
__device__ __forceinline__ void tile_spmv(int fmt, int aux, int nz, const uint8_t *P, const double *X,
                                          int lane, double &acc) {
    const int r = lane & 15, h = lane >> 4;
    const double *V = reinterpret_cast<const double *>(P);
    switch (fmt) {
    case F_DNS: {  // 256 values column-major: lane takes slots lane + 32 i
#pragma unroll
        for (int i = 0; i < 8; ++i) acc = fma(V[lane + 32 * i], X[h + 2 * i], acc);
        break;
    }
    case F_ELL: {  // slots k*16 + r; pads (k >= 1, column 0) skipped (R26)
        const int w = aux;
        const uint8_t *ci = P + 128 * w;
        for (int i = 0; i < (w + 1) >> 1; ++i) {
            int s = lane + 32 * i;
            if (s < 16 * w) {
                int c = nib(ci, s);
                if (s < 16 || c != 0) acc = fma(V[s], X[c], acc);
            }
        }
        break;
    }
    case F_CSR: {  // two lanes per row (Alg. 2)
        const uint8_t *rp = P + 8 * nz;
        const uint8_t *ci = rp + 16;
        int beg = rp[r], end = r < 15 ? rp[r + 1] : nz;
        for (int j = beg + h; j < end; j += 2) acc = fma(V[j], X[nib(ci, j)], acc);
        break;
    }
    case F_COO: {  // lanes of row r pick their entries, no atomics
        const uint8_t *rc = P + 8 * nz;
        for (int j = h; j < nz; j += 2) {
            int b = rc[j];
            if ((b >> 4) == r) acc = fma(V[j], X[b & 15], acc);
        }
        break;
    }
    case F_HYB: {  // ELL part then COO part
        const int w = aux, kc = nz - 16 * w;
        const double *CV = V + 16 * w;
        const uint8_t *ei = P + 128 * w + 8 * kc;
        const uint8_t *rc = ei + 8 * w;
        for (int i = 0; i < (w + 1) >> 1; ++i) {
            int s = lane + 32 * i;
            if (s < 16 * w) acc = fma(V[s], X[nib(ei, s)], acc);
        }
        for (int j = h; j < kc; j += 2) {
            int b = rc[j];
            if ((b >> 4) == r) acc = fma(CV[j], X[b & 15], acc);
        }
        break;
    }
    case F_DNSCOL: {  // full column q: value q*16 + r times x[colid[q]]
        const int nc = aux;
        const uint8_t *cid = P + 128 * nc;
        for (int i = 0; i < (nc + 1) >> 1; ++i) {
            int q = h + 2 * i;
            if (q < nc) acc = fma(V[q * 16 + r], X[cid[q]], acc);
        }
        break;
    }
    case F_DNSROW: {  // full row q: 16 lanes, shuffle reduction-sum
        const int nr = aux;
        const uint8_t *rid = P + 128 * nr;
        for (int i = 0; i < (nr + 1) >> 1; ++i) {
            int q = h + 2 * i;
            double s = q < nr ? V[q * 16 + r] * X[r] : 0.0;
            s += __shfl_xor_sync(FULL, s, 8);
            s += __shfl_xor_sync(FULL, s, 4);
            s += __shfl_xor_sync(FULL, s, 2);
            s += __shfl_xor_sync(FULL, s, 1);
            if (q < nr && rid[q] == r) acc += s;
        }
        break;
    }
    default:
        break;
    }
}

// ------------------------------------------------------------- kernel -----
__global__ void __launch_bounds__(kWarps * 32) tilespmv_fp64_kernel(const Params p) {
    extern __shared__ __align__(128) uint8_t smem[];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    uint8_t *buf = smem + warp * kWarpSmem;
    double *sx = reinterpret_cast<double *>(buf + kItemPayload);
    const uint32_t bar = smem_u32(buf + kItemPayload + kXBytes);
    const uint32_t buf_s = smem_u32(buf);
    if (lane == 0) {
        mbar_init(bar, 1);
        fence_mbar_init();
    }
    __syncwarp();
    uint32_t phase = 0;
    const int64_t stride = (int64_t)gridDim.x * kWarps;
    for (int64_t it = (int64_t)blockIdx.x * kWarps + warp; it < p.num_items; it += stride) {
        const Item item = p.items[it];
        const int nt = item.part_nt >> 24;
        const uint32_t bytes = (item.offe - item.offb) * 16u;
        // 1. one bulk copy of the item's tile payloads into shared memory
        if (lane == 0 && bytes) {
            fence_proxy_async();
            mbar_expect_tx(bar, bytes);
            bulk_g2s(buf_s, p.payload + (size_t)item.offb * 16, bytes, bar);
        }
        // 2. level-1 meta of the item's tiles, one tile per lane
        int J = 0, fmt = 0, aux = 0, tnz = 0, toff = 0;
        if (lane < nt) {
            const int t = item.tb + lane;
            J = __ldg(p.tileColIdx + t);
            fmt = __ldg(p.tileFmt + t);
            aux = __ldg(p.tileAux + t);
            tnz = __ldg(p.tileNnz + t + 1) - __ldg(p.tileNnz + t);
            toff = (int)(__ldg(p.tileOff + t) - item.offb) * 16;
        }
        // 3. x segments: lane l loads x[16 J_t + (l & 15)] for tiles t = 2k + (l >> 4)
        {
            double xv[kItemTiles / 2];
#pragma unroll
            for (int k = 0; k < kItemTiles / 2; ++k) {
                const int t = 2 * k + (lane >> 4);
                const int Jt = __shfl_sync(FULL, J, t);
                const int64_t c = 16 * (int64_t)Jt + (lane & 15);
                xv[k] = (t < nt && c < p.n) ? __ldg(p.x + c) : 0.0;
            }
#pragma unroll
            for (int k = 0; k < kItemTiles / 2; ++k) sx[(2 * k + (lane >> 4)) * 16 + (lane & 15)] = xv[k];
        }
        double acc = 0.0;
        // 4. fused CSR remainder of this tile row
        if (item.ke > item.kb) remainder_rows(p, item.I, item.kb, item.ke, lane, acc);
        __syncwarp();
        // 5. tiles, in order, dispatched on their format (warp-uniform branch)
        if (bytes) {
            mbar_wait(bar, phase);
            phase ^= 1u;
        }
        for (int q = 0; q < nt; ++q) {
            const int f = __shfl_sync(FULL, fmt, q);
            const int a = __shfl_sync(FULL, aux, q);
            const int nz = __shfl_sync(FULL, tnz, q);
            const int o = __shfl_sync(FULL, toff, q);
            tile_spmv(f, a, nz, buf + o, sx + q * 16, lane, acc);
        }
        acc += __shfl_xor_sync(FULL, acc, 16);
        // 6. y, written once per row (or a partial for split tile rows)
        const int64_t row = 16 * (int64_t)item.I + lane;
        if (item.split < 0) {
            if (lane < 16 && row < p.m) p.y[row] = acc;
        } else {
            const int2 si = p.split_info[item.split];
            const int part = item.part_nt & 0xFFFFFF;
            if (lane < 16) __stcg(p.partials + (int64_t)(si.x + part) * 16 + lane, acc);
            __threadfence();
            __syncwarp();
            int old = 0;
            if (lane == 0) old = atomicAdd(p.counters + item.split, 1);
            old = __shfl_sync(FULL, old, 0);
            if (old == si.y - 1) {  // last part of this tile row: sum the parts in order
                __threadfence();
                const int r = lane & 15, hh = lane >> 4;
                double s = 0.0;
                for (int q = hh; q < si.y; q += 2) s += __ldcg(p.partials + (int64_t)(si.x + q) * 16 + r);
                s += __shfl_xor_sync(FULL, s, 16);
                if (lane < 16 && row < p.m) p.y[row] = s;
                if (lane == 0) p.counters[item.split] = 0;  // ready for the next run
            }
        }
        __syncwarp();  // shared slot free before the next item's bulk copy
    }
}

// ----------------------------------------------------------- schedule -----
template <bool WRITE>
__device__ int items_for_row(int64_t I, const int32_t *tilePtr, const uint32_t *tileOff,
                             const int32_t *remRowPtr, int64_t m, Item *out, int split) {
    const int tp0 = tilePtr[I], tp1 = tilePtr[I + 1];
    int k0 = 0, k1 = 0;
    if (remRowPtr) {
        k0 = remRowPtr[16 * I];
        k1 = remRowPtr[16 * I + 16 < m ? 16 * I + 16 : m];
    }
    int t = tp0, k = k0, cnt = 0;
    do {
        const int tb = t;
        while (t < tp1 && t - tb < kItemTiles &&
               (int64_t)(tileOff[t + 1] - tileOff[tb]) * 16 <= kItemPayload)
            t++;
        if (t == tb && t < tp1) t++;  // (cannot happen: a tile is <= 2176 bytes)
        int kb = k, ke = k;
        if (t == tp1) {
            ke = min(k1, k + kItemRem);
            k = ke;
        }
        if (WRITE) {
            Item it;
            it.I = (int32_t)I;
            it.tb = tb;
            it.kb = kb;
            it.ke = ke;
            it.offb = tileOff[tb];
            it.offe = tileOff[t];
            it.split = split;
            it.part_nt = (split >= 0 ? cnt : 0) | ((t - tb) << 24);
            out[cnt] = it;
        }
        cnt++;
    } while (t < tp1 || k < k1);
    return cnt;
}

__global__ void k_items_count(const int32_t *tilePtr, const uint32_t *tileOff, const int32_t *remRowPtr,
                              int64_t m, int64_t tilem, int32_t *nitems, int32_t *nsplit) {
    int64_t I = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (I >= tilem) return;
    int c = items_for_row<false>(I, tilePtr, tileOff, remRowPtr, m, nullptr, -1);
    nitems[I] = c;
    nsplit[I] = c > 1 ? 1 : 0;
}

__global__ void k_items_write(const int32_t *tilePtr, const uint32_t *tileOff, const int32_t *remRowPtr,
                              int64_t m, int64_t tilem, const int32_t *itemBase, const int32_t *splitId,
                              const int32_t *nitems, const int32_t *partBase, Item *items, int2 *split_info) {
    int64_t I = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (I >= tilem) return;
    const bool split = nitems[I] > 1;
    const int sid = split ? splitId[I] : -1;
    items_for_row<true>(I, tilePtr, tileOff, remRowPtr, m, items + itemBase[I], sid);
    if (split) split_info[sid] = make_int2(partBase[I], nitems[I]);
}

__global__ void k_split_parts(const int32_t *nitems, int64_t tilem, int32_t *parts) {
    int64_t I = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (I >= tilem) return;
    parts[I] = nitems[I] > 1 ? nitems[I] : 0;
}

}  // namespace
}  // namespace tsp

#include <cub/cub.cuh>

namespace tsp {

int build_schedule(Matrix &M, cudaStream_t st) {
    const int TB = 256;
    const int64_t T = M.tilem;
    if (T == 0) return 0;
    auto blocks = [&](int64_t n) { return (unsigned)std::max<int64_t>(1, (n + TB - 1) / TB); };
    int32_t *nitems = nullptr, *nsplit = nullptr, *itemBase = nullptr, *splitId = nullptr,
            *parts = nullptr, *partBase = nullptr;
    void *tmp = nullptr;
    size_t tmp_bytes = 0;
    int rc = 0;
    auto fail = [&](cudaError_t e, const char *what) {
        rc = cuda_status(e, what);
        return rc;
    };
#define SCK(call)                                   \
    do {                                            \
        cudaError_t e_ = (call);                    \
        if (e_ != cudaSuccess) { fail(e_, #call); goto done; } \
    } while (0)
    {
        SCK(cudaMalloc(&nitems, (T + 1) * 4));
        SCK(cudaMalloc(&nsplit, (T + 1) * 4));
        SCK(cudaMalloc(&itemBase, (T + 1) * 4));
        SCK(cudaMalloc(&splitId, (T + 1) * 4));
        SCK(cudaMalloc(&parts, (T + 1) * 4));
        SCK(cudaMalloc(&partBase, (T + 1) * 4));
        SCK(cudaMemsetAsync(nitems + T, 0, 4, st));
        SCK(cudaMemsetAsync(nsplit + T, 0, 4, st));
        SCK(cudaMemsetAsync(parts + T, 0, 4, st));
        k_items_count<<<blocks(T), TB, 0, st>>>(M.tilePtr, M.tileOff, M.remRowPtr, M.m, T, nitems, nsplit);
        k_split_parts<<<blocks(T), TB, 0, st>>>(nitems, T, parts);
        SCK(cudaGetLastError());
        size_t b1 = 0, b2 = 0, b3 = 0;
        SCK(cub::DeviceScan::ExclusiveSum(nullptr, b1, nitems, itemBase, (int)(T + 1), st));
        SCK(cub::DeviceScan::ExclusiveSum(nullptr, b2, nsplit, splitId, (int)(T + 1), st));
        SCK(cub::DeviceScan::ExclusiveSum(nullptr, b3, parts, partBase, (int)(T + 1), st));
        tmp_bytes = std::max(b1, std::max(b2, b3));
        SCK(cudaMalloc(&tmp, tmp_bytes));
        SCK(cub::DeviceScan::ExclusiveSum(tmp, tmp_bytes, nitems, itemBase, (int)(T + 1), st));
        SCK(cub::DeviceScan::ExclusiveSum(tmp, tmp_bytes, nsplit, splitId, (int)(T + 1), st));
        SCK(cub::DeviceScan::ExclusiveSum(tmp, tmp_bytes, parts, partBase, (int)(T + 1), st));
        int32_t h[3];
        SCK(cudaMemcpyAsync(&h[0], itemBase + T, 4, cudaMemcpyDeviceToHost, st));
        SCK(cudaMemcpyAsync(&h[1], splitId + T, 4, cudaMemcpyDeviceToHost, st));
        SCK(cudaMemcpyAsync(&h[2], partBase + T, 4, cudaMemcpyDeviceToHost, st));
        SCK(cudaStreamSynchronize(st));
        M.num_items = h[0];
        M.num_split = h[1];
        const int64_t nparts = h[2];
        SCK(cudaMalloc(&M.items, std::max<int64_t>(M.num_items, 1) * sizeof(Item)));
        SCK(cudaMalloc(&M.split_info, std::max<int64_t>(M.num_split, 1) * sizeof(int2)));
        SCK(cudaMalloc(&M.counters, std::max<int64_t>(M.num_split, 1) * sizeof(int32_t)));
        SCK(cudaMalloc(&M.partials, std::max<int64_t>(nparts, 1) * 16 * sizeof(double)));
        M.device_bytes += M.num_items * sizeof(Item) + M.num_split * 12 + nparts * 128;
        SCK(cudaMemsetAsync(M.counters, 0, std::max<int64_t>(M.num_split, 1) * sizeof(int32_t), st));
        k_items_write<<<blocks(T), TB, 0, st>>>(M.tilePtr, M.tileOff, M.remRowPtr, M.m, T, itemBase, splitId,
                                                nitems, partBase, M.items, M.split_info);
        SCK(cudaGetLastError());
        SCK(cudaStreamSynchronize(st));
    }
done:
#undef SCK
    cudaFree(nitems); cudaFree(nsplit); cudaFree(itemBase); cudaFree(splitId);
    cudaFree(parts); cudaFree(partBase); cudaFree(tmp);
    return rc;
}

int configure_launch(Matrix &M) {
    TSP_CK(cudaFuncSetAttribute(tilespmv_fp64_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                kSmemBytes));
    int sms = 0, per_sm = 0;
    TSP_CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, M.device));
    TSP_CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, tilespmv_fp64_kernel, kWarps * 32,
                                                         kSmemBytes));
    per_sm = std::max(per_sm, 1);
    const int64_t need = (M.num_items + kWarps - 1) / kWarps;
    M.grid = (int)std::max<int64_t>(1, std::min<int64_t>(need, (int64_t)sms * per_sm));
    M.block = kWarps * 32;
    M.smem = kSmemBytes;
    return 0;
}

int launch_spmv(const Matrix &M, const double *d_x, double *d_y, cudaStream_t st) {
    if (M.m == 0) return 0;
    Params p;
    p.items = M.items;
    p.num_items = M.num_items;
    p.tileColIdx = M.tileColIdx;
    p.tileFmt = M.tileFmt;
    p.tileAux = M.tileAux;
    p.tileNnz = M.tileNnz;
    p.tileOff = M.tileOff;
    p.payload = M.payload;
    p.remRowPtr = M.remRowPtr;
    p.remCol = M.remCol;
    p.remVal = M.remVal;
    p.split_info = M.split_info;
    p.partials = M.partials;
    p.counters = M.counters;
    p.x = d_x;
    p.y = d_y;
    p.m = M.m;
    p.n = M.n;
    tilespmv_fp64_kernel<<<M.grid, M.block, M.smem, st>>>(p);
    TSP_CK(cudaGetLastError());
    return 0;
}

}  // namespace tsp
