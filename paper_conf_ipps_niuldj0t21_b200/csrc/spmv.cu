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
    const uint2 *tdesc;        // v2: packed tile descriptors
    const int64_t *cta_begin;  // v2: contiguous item chunk per CTA
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
__device__ __forceinline__ int64_t imin64(int64_t a, int64_t b) { return a < b ? a : b; }
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
    case F_CSR: {  // two lanes per row (Alg. 2); warp-uniform trip count
        const uint8_t *rp = P + 8 * nz;
        const uint8_t *ci = rp + 16;
        const int beg = rp[r] + h, end = r < 15 ? rp[r + 1] : nz;
        const int trips = __reduce_max_sync(FULL, (unsigned)max(0, (end - beg + 1) >> 1));
#pragma unroll 2
        for (int i = 0; i < trips; ++i) {
            const int j = beg + 2 * i;
            if (j < end) acc = fma(V[j], X[nib(ci, j)], acc);
        }
        break;
    }
    case F_COO: {  // lanes of row r pick their entries, no atomics
        const uint8_t *rc = P + 8 * nz;
        const int trips = (nz + 1) >> 1;
#pragma unroll 2
        for (int i = 0; i < trips; ++i) {
            const int j = h + 2 * i;
            if (j < nz) {
                const int b = rc[j];
                if ((b >> 4) == r) acc = fma(V[j], X[b & 15], acc);
            }
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
        const int trips = (kc + 1) >> 1;
#pragma unroll 2
        for (int i = 0; i < trips; ++i) {
            const int j = h + 2 * i;
            if (j < kc) {
                const int b = rc[j];
                if ((b >> 4) == r) acc = fma(CV[j], X[b & 15], acc);
            }
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


// ======================================================================
// v2: warp-specialised persistent kernel.  Per CTA (one per SM): one
// producer warp streams the CTA's contiguous chunk of work items into a
// shared-memory byte ring with TMA bulk copies (payload, packed 8-byte tile
// descriptors, remainder rowptr/col/val), signalling a per-slot "full"
// mbarrier through its transaction count; C consumer warps compute from
// shared memory and release the slot through its "empty" mbarrier.  Slot s
// is always served by consumer s mod C (S is a multiple of C), so every
// consumer waits on its own slots in order and parity waits cannot alias.
// ======================================================================

// bytes of one item in the ring: payload | descriptors | rowptr | col | val
struct RingParts {
    uint32_t pay, dsc, rp, col, val, total;
    uint32_t dsc_skew, col_skew, val_skew;
};

__device__ __forceinline__ uint32_t up16(uint32_t v) { return (v + 15u) & ~15u; }

__device__ __forceinline__ RingParts ring_parts(const Item &it, int64_t m) {
    RingParts r;
    const int nt = it.part_nt >> 24;
    r.pay = (it.offe - it.offb) * 16u;
    r.dsc_skew = (it.tb & 1) * 8u;                       // tdesc[tb] may sit mid 16-byte line
    r.dsc = nt ? up16(r.dsc_skew + 8u * nt) : 0u;
    if (it.ke > it.kb) {
        const int64_t rows = imin64(16, m - 16 * (int64_t)it.I);
        r.rp = up16((uint32_t)(rows + 1) * 4u);            // remRowPtr[16I .. 16I+rows], 64I-aligned
        r.col_skew = ((uint32_t)it.kb * 4u) & 15u;
        r.col = up16(r.col_skew + 4u * (it.ke - it.kb));
        r.val_skew = ((uint32_t)it.kb * 8u) & 15u;
        r.val = up16(r.val_skew + 8u * (it.ke - it.kb));
    } else {
        r.rp = r.col = r.val = r.col_skew = r.val_skew = 0u;
    }
    r.total = r.pay + r.dsc + r.rp + r.col + r.val;
    return r;
}

// the largest item: payload + 16 descriptors + rowptr + kItemRem col/val
constexpr uint32_t kItemMaxBytes =
    kItemPayload + ((8 * kItemTiles + 8 + 15) & ~15) + 80 + ((4 * kItemRem + 12 + 15) & ~15) +
    ((8 * kItemRem + 8 + 15) & ~15);

template <int C, int S>
struct RingCfg {
    static_assert(S % C == 0, "slot s must always map to consumer s mod C");
    static constexpr uint32_t kRing = (S + 1) * kItemMaxBytes;   // no live item can be overwritten
    static constexpr uint32_t kX = C * 16 * kItemTiles * 8;       // per-consumer x segments
    static constexpr uint32_t kSlots = S * (uint32_t)sizeof(Item) + S * 4;
    static constexpr uint32_t kBars = 2 * S * 8;
    static constexpr uint32_t kSmem = kRing + kX + ((kSlots + 15) & ~15u) + kBars;
    static constexpr int kThreads = 32 * (C + 1);
};

__device__ __forceinline__ void mbar_arrive(uint32_t bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}

// remainder rows staged in shared memory (rowptr, col, val), x gathered from L2
__device__ __forceinline__ void remainder_rows_smem(const Params &p, int64_t I, int kb, int ke,
                                                    const int *rpS, const int *colS, const double *valS,
                                                    int lane, double &acc) {
    const int r = lane & 15, h = lane >> 4;
    const int mr = (int)imin64(16, p.m - 16 * I);
    int b = rpS[min(r, mr)], e = rpS[min(r + 1, mr)];
    b = max(b, kb);
    e = min(e, ke);
    const int len = max(e - b, 0);
    const bool is_short = len <= kShortRow;
    {
        int cs[kShortRow / 2];
        double vs[kShortRow / 2];
#pragma unroll
        for (int i = 0; i < kShortRow / 2; ++i) {
            int k = b + h + 2 * i;
            bool ok = is_short && k < e;
            cs[i] = ok ? colS[k - kb] : 0;
            vs[i] = ok ? valS[k - kb] : 0.0;
        }
        double xs[kShortRow / 2];
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
            double vs[4], xv[4];
#pragma unroll
            for (int i = 0; i < 4; ++i) {
                int k = k0 + lane + 32 * i;
                cs[i] = k < ee ? colS[k - kb] : 0;
                vs[i] = k < ee ? valS[k - kb] : 0.0;
            }
#pragma unroll
            for (int i = 0; i < 4; ++i) xv[i] = (k0 + lane + 32 * i < ee) ? __ldg(p.x + cs[i]) : 0.0;
#pragma unroll
            for (int i = 0; i < 4; ++i)
                if (k0 + lane + 32 * i < ee) s = fma(vs[i], xv[i], s);
        }
#pragma unroll
        for (int o = 16; o >= 1; o >>= 1) s += __shfl_xor_sync(FULL, s, o);
        if (lane == rr) acc += s;
    }
}

__device__ __forceinline__ void write_rows(const Params &p, const Item &item, int lane, double acc) {
    const int64_t row = 16 * (int64_t)item.I + lane;
    if (item.split < 0) {
        if (lane < 16 && row < p.m) p.y[row] = acc;
        return;
    }
    const int2 si = p.split_info[item.split];
    const int part = item.part_nt & 0xFFFFFF;
    if (lane < 16) __stcg(p.partials + (int64_t)(si.x + part) * 16 + lane, acc);
    __threadfence();
    __syncwarp();
    int old = 0;
    if (lane == 0) old = atomicAdd(p.counters + item.split, 1);
    old = __shfl_sync(FULL, old, 0);
    if (old == si.y - 1) {  // last part of this tile row: sum the parts in item order
        __threadfence();
        const int r = lane & 15, hh = lane >> 4;
        double s = 0.0;
        for (int q = hh; q < si.y; q += 2) s += __ldcg(p.partials + (int64_t)(si.x + q) * 16 + r);
        s += __shfl_xor_sync(FULL, s, 16);
        if (lane < 16 && row < p.m) p.y[row] = s;
        if (lane == 0) p.counters[item.split] = 0;  // ready for the next run
    }
}

template <int C, int S>
__global__ void __launch_bounds__(RingCfg<C, S>::kThreads, 1) tilespmv_fp64_ring_kernel(const Params p) {
    using Cfg = RingCfg<C, S>;
    extern __shared__ __align__(128) uint8_t smem[];
    uint8_t *ring = smem;
    double *xs_all = reinterpret_cast<double *>(smem + Cfg::kRing);
    Item *slot_item = reinterpret_cast<Item *>(smem + Cfg::kRing + Cfg::kX);
    uint32_t *slot_pos = reinterpret_cast<uint32_t *>(slot_item + S);
    uint64_t *bars = reinterpret_cast<uint64_t *>(smem + Cfg::kRing + Cfg::kX + ((Cfg::kSlots + 15) & ~15u));
    const uint32_t full0 = smem_u32(bars), empty0 = smem_u32(bars + S);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) {
            mbar_init(full0 + 8 * s, 1);
            mbar_init(empty0 + 8 * s, 1);
        }
        fence_mbar_init();
    }
    __syncthreads();
    const int64_t beg = p.cta_begin[blockIdx.x], end = p.cta_begin[blockIdx.x + 1];
    const uint32_t ring_s = smem_u32(ring);

    if (warp == 0) {
        // ---------------------------------------------------- producer ----
        uint32_t pos = 0;
        for (int64_t k0 = beg; k0 < end; k0 += 32) {
            const int cnt = (int)imin64(32, end - k0);
            int4 ia = make_int4(0, 0, 0, 0), ib = ia;
            if (lane < cnt) {
                const int4 *src = reinterpret_cast<const int4 *>(p.items + k0 + lane);
                ia = __ldg(src);
                ib = __ldg(src + 1);
            }
            for (int j = 0; j < cnt; ++j) {
                Item it;
                it.I = __shfl_sync(FULL, ia.x, j);
                it.tb = __shfl_sync(FULL, ia.y, j);
                it.kb = __shfl_sync(FULL, ia.z, j);
                it.ke = __shfl_sync(FULL, ia.w, j);
                it.offb = (uint32_t)__shfl_sync(FULL, ib.x, j);
                it.offe = (uint32_t)__shfl_sync(FULL, ib.y, j);
                it.split = __shfl_sync(FULL, ib.z, j);
                it.part_nt = __shfl_sync(FULL, ib.w, j);
                if (lane == 0) {
                    const int64_t q = k0 + j - beg;
                    const int slot = (int)(q % S);
                    const uint32_t round = (uint32_t)(q / S);
                    if (round > 0) mbar_wait(empty0 + 8 * slot, (round - 1) & 1u);
                    const RingParts rp = ring_parts(it, p.m);
                    if (pos + rp.total > Cfg::kRing) pos = 0;
                    slot_item[slot] = it;
                    slot_pos[slot] = pos;
                    const uint32_t bar = full0 + 8 * slot;
                    fence_proxy_async();
                    mbar_expect_tx(bar, rp.total);
                    uint32_t d = ring_s + pos;
                    if (rp.pay) bulk_g2s(d, p.payload + (size_t)it.offb * 16, rp.pay, bar);
                    d += rp.pay;
                    if (rp.dsc) bulk_g2s(d, reinterpret_cast<const uint8_t *>(p.tdesc + it.tb) - rp.dsc_skew, rp.dsc, bar);
                    d += rp.dsc;
                    if (rp.rp) {
                        bulk_g2s(d, p.remRowPtr + 16 * (int64_t)it.I, rp.rp, bar);
                        d += rp.rp;
                        bulk_g2s(d, reinterpret_cast<const uint8_t *>(p.remCol + it.kb) - rp.col_skew, rp.col, bar);
                        d += rp.col;
                        bulk_g2s(d, reinterpret_cast<const uint8_t *>(p.remVal + it.kb) - rp.val_skew, rp.val, bar);
                    }
                    pos += rp.total;
                }
                __syncwarp();
            }
        }
        return;
    }
    // -------------------------------------------------------- consumers ---
    const int c = warp - 1;
    double *xs = xs_all + c * 16 * kItemTiles;
    for (int64_t q = c; beg + q < end; q += C) {
        const int slot = (int)(q % S);
        const uint32_t round = (uint32_t)(q / S);
        mbar_wait(full0 + 8 * slot, round & 1u);
        const Item it = slot_item[slot];
        const uint32_t pos = slot_pos[slot];
        const RingParts rp = ring_parts(it, p.m);
        const uint8_t *pay = ring + pos;
        const uint2 *dsc = reinterpret_cast<const uint2 *>(pay + rp.pay + rp.dsc_skew);
        const int nt = it.part_nt >> 24;
        // x segments of the item's tiles (x stays in L2; 128-byte lines)
        {
            double xv[kItemTiles / 2];
#pragma unroll
            for (int k = 0; k < kItemTiles / 2; ++k) {
                const int t = 2 * k + (lane >> 4);
                xv[k] = 0.0;
                if (t < nt) {
                    const int64_t col = 16 * (int64_t)(dsc[t].x & 0x7FFFFFFu) + (lane & 15);
                    if (col < p.n) xv[k] = __ldg(p.x + col);
                }
            }
#pragma unroll
            for (int k = 0; k < kItemTiles / 2; ++k) xs[(2 * k + (lane >> 4)) * 16 + (lane & 15)] = xv[k];
        }
        double acc = 0.0;
        if (rp.rp) {
            const uint8_t *rb = pay + rp.pay + rp.dsc;
            remainder_rows_smem(p, it.I, it.kb, it.ke, reinterpret_cast<const int *>(rb),
                                reinterpret_cast<const int *>(rb + rp.rp + rp.col_skew),
                                reinterpret_cast<const double *>(rb + rp.rp + rp.col + rp.val_skew), lane, acc);
        }
        __syncwarp();
        uint32_t off = 0;
        for (int t = 0; t < nt; ++t) {
            const uint2 d = dsc[t];
            const int fmt = (int)(d.x >> 27);
            const int aux = (int)(d.y & 31u), nz = (int)((d.y >> 5) & 511u);
            tile_spmv(fmt, aux, nz, pay + off, xs + 16 * t, lane, acc);
            off += ((d.y >> 14) & 255u) * 16u;
        }
        acc += __shfl_xor_sync(FULL, acc, 16);
        write_rows(p, it, lane, acc);
        __syncwarp();
        if (lane == 0) mbar_arrive(empty0 + 8 * slot);
    }
}

// 8-byte tile descriptor read by the v2 kernel, derived from the canonical
// level-1 arrays: x = J | fmt << 27 ; y = aux | nnz << 5 | size16 << 14.
__global__ void k_build_tdesc(const int32_t *tileColIdx, const uint8_t *tileFmt, const uint8_t *tileAux,
                              const int32_t *tileNnz, const uint32_t *tileOff, int64_t numtile, uint2 *tdesc) {
    int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (t >= numtile) return;
    uint2 d;
    d.x = (uint32_t)tileColIdx[t] | ((uint32_t)tileFmt[t] << 27);
    d.y = (uint32_t)tileAux[t] | ((uint32_t)(tileNnz[t + 1] - tileNnz[t]) << 5) |
          ((tileOff[t + 1] - tileOff[t]) << 14);
    tdesc[t] = d;
}

// item cost for the CTA chunking: bytes moved + a fixed per-item overhead
__global__ void k_item_cost(const Item *items, int64_t n, int64_t *cost) {
    int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (k >= n) return;
    const Item it = items[k];
    cost[k] = (int64_t)(it.offe - it.offb) * 16 + 12 * (int64_t)(it.ke - it.kb) + 8 * (it.part_nt >> 24) + 256;
}

__global__ void k_cta_begin(const int64_t *incl, int64_t n, int G, int64_t *cta_begin) {
    int b = blockIdx.x * blockDim.x + threadIdx.x;
    if (b > G) return;
    if (b == G) { cta_begin[b] = n; return; }
    const int64_t total = n ? incl[n - 1] : 0;
    const int64_t target = total * b / G;   // first item whose prefix-before >= target
    int64_t lo = 0, hi = n;
    while (lo < hi) {
        int64_t mid = (lo + hi) / 2;
        int64_t before = mid ? incl[mid - 1] : 0;
        if (before < target) lo = mid + 1; else hi = mid;
    }
    cta_begin[b] = lo;
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

using KernelFn = void (*)(Params);

struct KernelChoice {
    const char *name;
    KernelFn fn;
    int threads, smem, ctas_per_sm;
};

template <int C, int S>
KernelChoice ring_choice(const char *name) {
    return {name, tilespmv_fp64_ring_kernel<C, S>, RingCfg<C, S>::kThreads, (int)RingCfg<C, S>::kSmem, 1};
}

static KernelChoice choose_kernel(int version) {
    switch (version) {
    case 1: return {"v1", tilespmv_fp64_kernel, kWarps * 32, kSmemBytes, 0};
    case 2: return ring_choice<6, 12>("ring_c6_s12");
    case 3: return ring_choice<4, 8>("ring_c4_s8");
    case 4: return ring_choice<4, 12>("ring_c4_s12");
    case 5: return ring_choice<8, 8>("ring_c8_s8");
    case 6: return ring_choice<3, 12>("ring_c3_s12");
    default: return ring_choice<6, 12>("ring_c6_s12");
    }
}

int configure_launch(Matrix &M) {
    int version = 2;
    if (const char *e = getenv("TILESPMV_KERNEL")) version = atoi(e);
    const KernelChoice kc = choose_kernel(version);
    TSP_CK(cudaFuncSetAttribute(kc.fn, cudaFuncAttributeMaxDynamicSharedMemorySize, kc.smem));
    int sms = 0, per_sm = 0;
    TSP_CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, M.device));
    TSP_CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kc.fn, kc.threads, kc.smem));
    if (per_sm < 1) return set_error(TILESPMV_CUDA, "SpMV kernel does not fit on an SM");
    M.kernel_version = version;
    M.block = kc.threads;
    M.smem = kc.smem;
    if (version == 1) {
        const int64_t need = (M.num_items + kWarps - 1) / kWarps;
        M.grid = (int)std::max<int64_t>(1, std::min<int64_t>(need, (int64_t)sms * per_sm));
        return 0;
    }
    // v2: one CTA per SM, each owning a contiguous, cost-balanced item chunk
    const int G = (int)std::max<int64_t>(1, std::min<int64_t>((int64_t)sms * kc.ctas_per_sm, M.num_items));
    M.grid = G;
    if (M.cta_begin) cudaFree(M.cta_begin);
    M.cta_begin = nullptr;
    TSP_CK(cudaMalloc(&M.cta_begin, (G + 1) * sizeof(int64_t)));
    M.device_bytes += (G + 1) * 8;
    if (M.num_items > 0) {
        int64_t *cost = nullptr, *incl = nullptr;
        void *tmp = nullptr;
        size_t tb = 0;
        TSP_CK(cudaMalloc(&cost, M.num_items * sizeof(int64_t)));
        TSP_CK(cudaMalloc(&incl, M.num_items * sizeof(int64_t)));
        k_item_cost<<<(unsigned)((M.num_items + 255) / 256), 256>>>(M.items, M.num_items, cost);
        TSP_CK(cub::DeviceScan::InclusiveSum(nullptr, tb, cost, incl, (int)M.num_items));
        TSP_CK(cudaMalloc(&tmp, tb));
        TSP_CK(cub::DeviceScan::InclusiveSum(tmp, tb, cost, incl, (int)M.num_items));
        k_cta_begin<<<(G + 1 + 255) / 256, 256>>>(incl, M.num_items, G, M.cta_begin);
        TSP_CK(cudaGetLastError());
        TSP_CK(cudaDeviceSynchronize());
        cudaFree(cost);
        cudaFree(incl);
        cudaFree(tmp);
    } else {
        TSP_CK(cudaMemset(M.cta_begin, 0, (G + 1) * sizeof(int64_t)));
    }
    return 0;
}

int build_tdesc(Matrix &M, cudaStream_t st) {
    TSP_CK(cudaMalloc(&M.tdesc, (M.numtile + 2) * sizeof(uint2)));
    M.device_bytes += (M.numtile + 2) * 8;
    if (M.numtile > 0) {
        k_build_tdesc<<<(unsigned)((M.numtile + 255) / 256), 256, 0, st>>>(M.tileColIdx, M.tileFmt, M.tileAux,
                                                                           M.tileNnz, M.tileOff, M.numtile,
                                                                           M.tdesc);
        TSP_CK(cudaGetLastError());
    }
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
    p.tdesc = M.tdesc;
    p.cta_begin = M.cta_begin;
    const KernelChoice kc = choose_kernel(M.kernel_version);
    kc.fn<<<M.grid, M.block, M.smem, st>>>(p);
    TSP_CK(cudaGetLastError());
    return 0;
}

}  // namespace tsp
