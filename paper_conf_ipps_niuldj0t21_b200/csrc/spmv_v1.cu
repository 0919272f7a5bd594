// spmv_v1.cu -- baseline kernel (round 1, v1): one warp per work item,
// non-pipelined.  Each warp stages its item's tile payloads with one
// cp.async.bulk (TMA, 1-D) into its own shared-memory slot, gathers the x
// segments, processes the CSR remainder from global memory and then runs the
// full-warp format routines.  Kept for A/B comparison with the default warp
// kernel (spmv_warp.cu); select with TILESPMV_KERNEL=1.
#include "spmv_common.cuh"

namespace tsp {
namespace {

constexpr int kWarps = 4;                                   // warps per CTA
constexpr int kXBytes = kItemTiles * 16 * 8;                // x segments per item
constexpr int kWarpSmem = kItemBytesMax + kXBytes + 128;       // + mbarrier slot
constexpr int kSmemBytes = kWarps * kWarpSmem;

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
    double *sx = reinterpret_cast<double *>(buf + kItemBytesMax);
    const uint32_t bar = smem_u32(buf + kItemBytesMax + kXBytes);
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
        const int nt = item_nt(item);
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
            const int part = item_part(item);
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



}  // namespace

KernelChoice kernel_v1() {
    return {"v1_warp_staged", tilespmv_fp64_kernel, kWarps * 32, kSmemBytes, 0, false, kItemBytesMax, false, false};
}

}  // namespace tsp
