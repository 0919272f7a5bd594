// spmv_warp.cu -- the default SpMV kernel (TILESPMV_KERNEL 20-29): y =
// A_tiles*x + A_rem*x in fp64 on sm_100a (§III.C P:118-173 warp-level
// tile SpMV, P:199 load balancing, P:201 DeferredCOO remainder).
//
// High occupancy (32 warps/SM): every warp is its own producer and consumer.
// Per work item, lane 0 stages the item's execution blob (descriptor list,
// tile columns, tile payloads, remainder rowptr/col/val; blob_parts) into the
// warp's shared-memory slot with ONE TMA bulk copy (cp.async.bulk, L2
// evict-first) completing on the warp's mbarrier; the warp then gathers the
// x segment of every tile (one 128-byte line, L2 evict-last), runs the
// half-warp tile routines of spmv_tiles.cuh two tiles at a time and writes
// y once per row.  Latency is hidden by warp count; the next item's
// descriptor is prefetched into registers.  No floating-point atomics.
#include "spmv_tiles.cuh"

namespace tsp {
namespace {

template <int WARPS, int SLOT>
struct WarpCfg {
    static_assert(SLOT % 16 == 0 && SLOT <= kItemBytesMax, "slot size");
    static constexpr uint32_t kX = kItemTiles * 16 * 8;
    static constexpr uint32_t kPer = SLOT + kX + 128 + 16;  // slot | x | row sums | mbarrier
    static constexpr uint32_t kSmem = WARPS * kPer + 256;   // +256: loads may overrun a slot
    static constexpr int kThreads = 32 * WARPS;
};

__device__ __forceinline__ Item load_item(const Item *items, int k) {
    const int4 *src = reinterpret_cast<const int4 *>(items + k);
    const int4 a = __ldg(src), b = __ldg(src + 1), e = __ldg(src + 2);
    Item it;
    it.I = a.x; it.tb = a.y; it.kb = a.z; it.ke = a.w;
    it.offb = (uint32_t)b.x; it.offe = (uint32_t)b.y; it.split = b.z; it.part_nt = b.w;
    it.dbeg = e.x; it.ndsc = e.y; it.blob16 = (uint32_t)e.z; it.blob_len = (uint32_t)e.w;
    return it;
}

template <int WARPS, int SLOT, int MINB>
__global__ void __launch_bounds__(WarpCfg<WARPS, SLOT>::kThreads, MINB) tilespmv_fp64_warp(const Params p) {
    using Cfg = WarpCfg<WARPS, SLOT>;
    extern __shared__ __align__(128) uint8_t smem[];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int h = lane >> 4, r = lane & 15;
    const uint32_t base = smem_u32(smem) + (uint32_t)warp * Cfg::kPer;
    const uint32_t slot = base, xs = base + SLOT, racc = xs + Cfg::kX, bar = racc + 128;
    if (lane == 0) {
        mbar_init(bar, 1);
        fence_mbar_init();
    }
    __syncwarp();
    const uint32_t n32 = (uint32_t)p.n;
    // contiguous, cost-balanced, row-aligned item chunk per warp (schedule.cu);
    // neighbouring tile rows share x segments
    const int64_t gw = (int64_t)blockIdx.x * WARPS + warp;
    const int kbeg = (int)p.cta_begin[gw], kend = (int)p.cta_begin[gw + 1];
    double carry = 0.0;  // partial row sums of a local split tile row
    uint32_t phase = 0;
    const uint64_t stream_policy = policy_evict_first(), x_policy = policy_evict_last();
    Item nxt;
    if (kbeg < kend) nxt = load_item(p.items, kbeg);
    for (int k = kbeg; k < kend; ++k) {
        const Item it = nxt;
        if (k + 1 < kend) nxt = load_item(p.items, k + 1);  // in flight during this item
        const BlobParts bp = blob_parts(it, p.m);
        // the whole item (descriptors, J, payload, remainder) in ONE TMA bulk copy
        if (lane == 0 && bp.total) {
            fence_proxy_async();
            mbar_expect_tx(bar, bp.total);
            bulk_g2s_hint(slot, p.blob + (size_t)it.blob16 * 16, bp.total, bar, stream_policy);
        }
        if (bp.total) {
            mbar_wait(bar, phase);
            phase ^= 1u;
        }
        const int nt = item_nt(it);
        const uint32_t dsc = slot, pay = slot + bp.pay;
        // x segments, J from the blob
        if (p.x_vec) {  // lane l: tile 4k + (l >> 3), elements 2(l & 7) .. +1, one 16-byte load
            const int q = lane & 7;
#pragma unroll
            for (int kk = 0; kk < kItemTiles / 4; ++kk) {
                const int t = 4 * kk + (lane >> 3);
                if (t < nt) {
                    const uint32_t c0 = 16u * (uint32_t)lds_s32(slot + bp.jt + 4 * t) + 2u * q;
                    double2 v;
                    if (c0 + 2 <= n32) {
                        v = ldg2_hint(p.x + c0, x_policy);
                    } else {
                        v.x = c0 < n32 ? ldg_hint(p.x + c0, x_policy) : 0.0;
                        v.y = 0.0;
                    }
                    sts_v2f64(xs + 128 * t + 16 * q, v);
                }
            }
        } else {  // lane l: tile 2k + h, element r
#pragma unroll
            for (int kk = 0; kk < kItemTiles / 2; ++kk) {
                const int t = 2 * kk + h;
                if (t < nt) {
                    const uint32_t col = 16u * (uint32_t)lds_s32(slot + bp.jt + 4 * t) + (uint32_t)r;
                    sts_f64(xs + 8 * (16 * t + r), col < n32 ? ldg_hint(p.x + col, x_policy) : 0.0);
                }
            }
        }
        double acc = 0.0;
        if (bp.total > bp.rp) {  // fused CSR remainder: two lanes per short row, or a flat pass
            const int rows = (int)imin64(16, p.m - 16 * (int64_t)it.I);
            const int b = lds_s32(slot + bp.rp + 4 * min(r, rows)), e = lds_s32(slot + bp.rp + 4 * min(r + 1, rows));
            const uint32_t colS = slot + bp.col, valS = slot + bp.val;
            const bool is_short = e - b <= kShortRow;
            if (!__any_sync(FULL, !is_short)) {
                // two lanes per short row; warp-uniform trip count, batches of four
                // (loads of a batch first, then its FMAs)
                const int trips = (int)__reduce_max_sync(FULL, is_short ? (unsigned)((e - b + 1 - h) >> 1) : 0u);
#pragma unroll 1
                for (int i0 = 0; i0 < trips; i0 += 4) {
                    double vs[4], xr[4];
                    bool oks[4];
#pragma unroll
                    for (int i = 0; i < 4; ++i) {
                        const int kq = b + h + 2 * (i0 + i);
                        oks[i] = is_short && kq < e;
                        vs[i] = xr[i] = 0.0;
                        if (i0 + i < trips) {
                            const int c = oks[i] ? lds_s32(colS + 4 * kq) : 0;
                            vs[i] = lds_f64(valS + 8 * (oks[i] ? kq : 0));
                            if (oks[i]) xr[i] = ldg_hint(p.x + (uint32_t)c, x_policy);
                        }
                    }
#pragma unroll
                    for (int i = 0; i < 4; ++i) fma_if(oks[i], vs[i], xr[i], acc);
                }
            } else {
                // a long row: every remainder entry of the item in one flat pass,
                // one lane per entry, x gathers batched four chunks deep, rows
                // summed by a segmented shuffle scan (fixed order)
                const uint32_t rpS = slot + bp.rp;
                const int etot = lds_s32(rpS + 4 * rows);
                if (lane < 16) sts_f64(racc + 8 * lane, 0.0);
                __syncwarp();
#pragma unroll 1
                for (int k0 = 0; k0 < etot; k0 += 128) {
                    double pv[4];
                    int rw[4];
                    bool okv[4];
#pragma unroll
                    for (int i = 0; i < 4; ++i) {
                        const int kq = k0 + 32 * i + lane;
                        okv[i] = kq < etot;
                        const int c = okv[i] ? lds_s32(colS + 4 * kq) : 0;
                        pv[i] = lds_f64(valS + 8 * (okv[i] ? kq : 0));
                        pv[i] = okv[i] ? pv[i] * ldg_hint(p.x + (uint32_t)c, x_policy) : 0.0;
                    }
#pragma unroll
                    for (int i = 0; i < 4; ++i) {  // row of entry kq: rp[row] <= kq < rp[row+1]
                        const int kq = k0 + 32 * i + lane;
                        int lo = 0, hi = rows;
#pragma unroll
                        for (int st = 0; st < 5; ++st) {
                            const int mid = (lo + hi) >> 1;
                            if (hi - lo > 1) {
                                if (lds_s32(rpS + 4 * mid) <= kq) lo = mid;
                                else hi = mid;
                            }
                        }
                        rw[i] = lo;
                    }
#pragma unroll
                    for (int d = 1; d < 32; d <<= 1) {
#pragma unroll
                        for (int i = 0; i < 4; ++i) {
                            const double t = __shfl_up_sync(FULL, pv[i], d);
                            const int rr = __shfl_up_sync(FULL, rw[i], d);
                            if (lane >= d && rr == rw[i]) pv[i] += t;
                        }
                    }
#pragma unroll
                    for (int i = 0; i < 4; ++i) {  // segment tails add to their row, chunk by chunk
                        const int nr = __shfl_down_sync(FULL, rw[i], 1);
                        const int kq = k0 + 32 * i + lane;
                        if (okv[i] && (lane == 31 || nr != rw[i] || kq + 1 >= etot)) {
                            const uint32_t a = racc + 8 * rw[i];
                            sts_f64(a, lds_f64(a) + pv[i]);
                        }
                        __syncwarp();
                    }
                }
                if (lane < 16) acc += lds_f64(racc + 8 * lane);
            }
        }
        __syncwarp();
        const int npairs = it.ndsc >> 1;
#pragma unroll 1
        for (int q = 0; q < npairs; ++q) run_pair(lds_v2u32(dsc + 16 * q + 8 * h), pay, xs, r, acc);
        acc += __shfl_xor_sync(FULL, acc, 16);
        if (it.split < 0) {
            const int64_t row = 16 * (int64_t)it.I + lane;
            if (lane < 16 && row < p.m) p.y[row] = acc;
        } else if (!item_last(it)) {  // a group of parts runs here, in part order
            carry += acc;
        } else {
            const double total = carry + acc;
            carry = 0.0;
            const int64_t row = 16 * (int64_t)it.I + lane;
            if (item_local(it)) {  // the row's only group
                if (lane < 16 && row < p.m) p.y[row] = total;
            } else {  // hub row: one partial per group, the last group sums them in order
                const int2 si = p.split_info[it.split];
                const int ngroups = (si.y + kLocalParts - 1) / kLocalParts;
                const int g = item_part(it) / kLocalParts;
                if (lane < 16) __stcg(p.partials + (int64_t)(si.x + g) * 16 + lane, total);
                __threadfence();
                __syncwarp();
                int old = 0;
                if (lane == 0) old = atomicAdd(p.counters + it.split, 1);
                old = __shfl_sync(FULL, old, 0);
                if (old == ngroups - 1) {  // half hh sums groups hh, hh+2, ... in order, 4 loads in flight
                    __threadfence();
                    double s = 0.0;
                    for (int q0 = h; q0 < ngroups; q0 += 8) {
                        double v[4];
#pragma unroll
                        for (int i = 0; i < 4; ++i) {
                            const int q = q0 + 2 * i;
                            v[i] = q < ngroups ? __ldcg(p.partials + (int64_t)(si.x + q) * 16 + r) : 0.0;
                        }
#pragma unroll
                        for (int i = 0; i < 4; ++i) s += v[i];
                    }
                    s += __shfl_xor_sync(FULL, s, 16);
                    if (lane < 16 && row < p.m) p.y[row] = s;
                    if (lane == 0) p.counters[it.split] = 0;  // ready for the next run
                }
            }
        }
        __syncwarp();  // slot, x and J scratch free for the next item
    }
}

template <int WARPS, int SLOT, int MINB>
KernelChoice warp_choice(const char *name) {
    using Cfg = WarpCfg<WARPS, SLOT>;
    return {name, tilespmv_fp64_warp<WARPS, SLOT, MINB>, Cfg::kThreads, (int)Cfg::kSmem, 0, false, SLOT};
}

}  // namespace

KernelChoice kernel_warp(int variant) {
    switch (variant) {
    case 21: return warp_choice<8, 4608, 4>("warp_w8x4_4.5k");
    case 22: return warp_choice<8, 5120, 3>("warp_w8x3_5k");
    case 23: return warp_choice<4, 4608, 8>("warp_w4x8_4.5k");
    case 24: return warp_choice<8, 4096, 4>("warp_w8x4_4k");
    default: return warp_choice<8, 4608, 4>("warp_w8x4_4.5k");
    }
}

}  // namespace tsp
