// spmv_ring.cu -- the timed hot path (default kernel): y = A_tiles*x + A_rem*x
// in fp64 on sm_100a (§III.C P:118-173 warp-level tile SpMV, P:199
// load balancing, P:201 DeferredCOO remainder).
//
// Warp-specialised persistent kernel, one CTA per SM, each CTA owning a
// contiguous, cost-balanced chunk of work items:
//   * producer warp: lane j streams item (k0 + j) of a batch of S items into
//     shared-memory slot j with TMA bulk copies (cp.async.bulk, 1-D):
//     tile payloads, 8-byte tile descriptors, remainder rowptr/col/val.
//     Completion is counted in bytes on the slot's "full" mbarrier.
//   * C consumer warps: consumer c serves slots c, c+C, ... (S % C == 0, so
//     every slot has one consumer and mbarrier parities cannot alias).  It
//     stages the x segments of the item's tiles (one 128-byte line each) in
//     shared memory, runs the format routines and writes y, then releases
//     the slot on its "empty" mbarrier.
//   * Tiles are processed TWO AT A TIME: after a warp ballot groups the
//     item's tiles by format, each half-warp takes one tile of a same-format
//     pair with one lane per tile row (the per-row decomposition of the
//     paper's CSR/ELL/DnsCol routines), so the per-tile
//     dispatch and setup cost is shared by two tiles and every loop has a
//     warp-uniform trip count with predicated FMAs (no divergent branches).
//     Row r's two half sums meet in acc(r) + acc(r + 16).
//   * No floating-point atomics: y is bitwise deterministic.
#include "spmv_common.cuh"

namespace tsp {
namespace {

template <int C, int S>
struct RingCfg {
    static_assert(S % C == 0, "slot s must always be served by consumer s mod C");
    static_assert(S <= 32, "one producer lane per slot");
    static constexpr uint32_t kRing = (uint32_t)S * kItemBytes;
    static constexpr uint32_t kX = (uint32_t)C * kItemTiles * 16 * 8;
    static constexpr uint32_t kSlots = (uint32_t)S * sizeof(Item);
    static constexpr uint32_t kBars = 2u * S * 8u;
    static constexpr uint32_t kSmem = kRing + kX + kSlots + kBars + 64;  // +64: loads may overrun a slot
    static constexpr int kThreads = 32 * (C + 1);
};

// ------------------------------------------------ remainder (from smem) ----
// rows of at most kShortRow entries: two lanes per row; longer rows: the
// whole warp strides the row and reduces with a butterfly (fixed order).
__device__ __forceinline__ void remainder_rows(const Params &p, int64_t I, int kb, int ke, const int *rpS,
                                               const int *colS, const double *valS, int lane, double &acc) {
    const int r = lane & 15, h = lane >> 4;
    const int mr = (int)imin64(16, p.m - 16 * I);
    int b = rpS[min(r, mr)], e = rpS[min(r + 1, mr)];
    b = max(b, kb);
    e = min(e, ke);
    const int len = max(e - b, 0);
    const bool is_short = len <= kShortRow;
    {
        int cs[kShortRow / 2];
        double vs[kShortRow / 2], xs[kShortRow / 2];
#pragma unroll
        for (int i = 0; i < kShortRow / 2; ++i) {
            const int k = b + h + 2 * i;
            const bool ok = is_short && k < e;
            cs[i] = ok ? colS[k - kb] : 0;
            vs[i] = ok ? valS[k - kb] : 0.0;
        }
#pragma unroll
        for (int i = 0; i < kShortRow / 2; ++i) {
            const int k = b + h + 2 * i;
            xs[i] = (is_short && k < e) ? __ldg(p.x + cs[i]) : 0.0;
        }
#pragma unroll
        for (int i = 0; i < kShortRow / 2; ++i) {
            const int k = b + h + 2 * i;
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
                const int k = k0 + lane + 32 * i;
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

// --------------------------------------------- half-warp tile routines -----
// Lane r of a half owns row r of its tile.  P: payload, X: 16 x values,
// ok: the half has a tile.  All loops have warp-uniform trip counts; the
// unconditional shared-memory loads past a tile's end stay inside the CTA's
// shared memory and are masked out of the FMA.

// CSR: csrVal row-major | csrRowPtr[16] u8 | 4-bit columns (Alg. 2)
__device__ __forceinline__ void half_csr(const uint8_t *P, int nz, const double *X, int r, bool ok, double &acc) {
    const double *V = reinterpret_cast<const double *>(P);
    const uint8_t *rp = P + 8 * nz;
    const uint8_t *ci = rp + 16;
    const int beg = ok ? rp[r] : 0;
    const int end = ok ? (r < 15 ? rp[r + 1] : nz) : 0;
    const int len = end - beg;
    const int trips = (int)__reduce_max_sync(FULL, (unsigned)len);
    const double *Vb = V + beg;
#pragma unroll 4
    for (int i = 0; i < trips; ++i) {
        const int j = beg + i;
        const double v = Vb[i];
        const double xv = X[nib(ci, j)];
        if (i < len) acc = fma(v, xv, acc);
    }
}

// ELL: slots k*16 + r column-major | 4-bit columns (Alg. 4).
// Pads (k >= 1 with column 0, reading R26) are skipped.
__device__ __forceinline__ void half_ell(const uint8_t *P, int w, const double *X, int r, bool ok, double &acc) {
    const double *V = reinterpret_cast<const double *>(P);
    const uint8_t *ci = P + 128 * w;
    const int wq = ok ? w : 0;
    const int trips = (int)__reduce_max_sync(FULL, (unsigned)wq);
    const int sh = 4 * (r & 1);
#pragma unroll 4
    for (int k = 0; k < trips; ++k) {
        const double v = V[16 * k + r];
        const int c = (ci[8 * k + (r >> 1)] >> sh) & 15;
        const double xv = X[c];
        if (k < wq && (k == 0 || c != 0)) acc = fma(v, xv, acc);
    }
}

// Dns: 256 values column-major
__device__ __forceinline__ void half_dns(const uint8_t *P, const double *X, int r, bool ok, double &acc) {
    const double *V = reinterpret_cast<const double *>(P) + r;
    double a0 = 0.0, a1 = 0.0;
#pragma unroll
    for (int c = 0; c < 16; c += 2) {
        a0 = fma(V[16 * c], X[c], a0);
        a1 = fma(V[16 * c + 16], X[c + 1], a1);
    }
    if (ok) acc += a0 + a1;
}

// DnsCol: full column q holds value q*16 + r, column id colid[q]
__device__ __forceinline__ void half_dnscol(const uint8_t *P, int nc, const double *X, int r, bool ok, double &acc) {
    const double *V = reinterpret_cast<const double *>(P);
    const uint8_t *cid = P + 128 * nc;
    const int nq = ok ? nc : 0;
    const int trips = (int)__reduce_max_sync(FULL, (unsigned)nq);
    for (int q = 0; q < trips; ++q) {
        const double v = V[16 * q + r];
        const double xv = X[cid[q] & 15];
        if (q < nq) acc = fma(v, xv, acc);
    }
}

// DnsRow: full row q (id rowid[q]) holds values q*16 + c; the
// lane of row rowid[q] sums the 16 products of its row.
__device__ __forceinline__ void half_dnsrow(const uint8_t *P, int nr, const double *X, int r, bool ok, double &acc) {
    const double *V = reinterpret_cast<const double *>(P);
    const uint8_t *rid = P + 128 * nr;
    int q_r = -1;
    const int nq = ok ? nr : 0;
    for (int q = 0; q < 7; ++q)
        if (q < nq && rid[q] == r) q_r = q;
    const bool mine = q_r >= 0;
    const double *Vr = V + 16 * (mine ? q_r : 0);
    const bool any = __any_sync(FULL, mine);
    if (any) {
        double a0 = 0.0, a1 = 0.0;
#pragma unroll
        for (int c = 0; c < 16; c += 2) {
            a0 = fma(Vr[c], X[c], a0);
            a1 = fma(Vr[c + 1], X[c + 1], a1);
        }
        if (mine) acc += a0 + a1;
    }
}

// COO part: value j, packed (row << 4 | col) byte (Alg. 3); the lane
// of the entry's row adds it (no atomics, fixed order)
__device__ __forceinline__ void half_coo(const double *V, const uint8_t *rc, int n, const double *X, int r, bool ok,
                                         double &acc) {
    const int nq = ok ? n : 0;
    const int trips = (int)__reduce_max_sync(FULL, (unsigned)nq);
#pragma unroll 2
    for (int j = 0; j < trips; ++j) {
        const int b = rc[j];
        const double v = V[j];
        const double xv = X[b & 15];
        if (j < nq && (b >> 4) == r) acc = fma(v, xv, acc);
    }
}

// HYB: ELL(w) values | COO values | ELL 4-bit columns | COO (row<<4|col)
__device__ __forceinline__ void half_hyb(const uint8_t *P, int w, int nz, const double *X, int r, bool ok,
                                         double &acc) {
    const double *V = reinterpret_cast<const double *>(P);
    const int kc = nz - 16 * w;
    const uint8_t *ei = P + 128 * w + 8 * kc;
    const int wq = ok ? w : 0;
    const int trips = (int)__reduce_max_sync(FULL, (unsigned)wq);
    const int sh = 4 * (r & 1);
    for (int k = 0; k < trips; ++k) {
        const double v = V[16 * k + r];
        const double xv = X[(ei[8 * k + (r >> 1)] >> sh) & 15];
        if (k < wq) acc = fma(v, xv, acc);
    }
    half_coo(V + 16 * w, ei + 8 * w, kc, X, r, ok, acc);
}

// ------------------------------------------------------------ kernel -------
template <int C, int S>
__global__ void __launch_bounds__(RingCfg<C, S>::kThreads, 1) tilespmv_fp64_ring(const Params p) {
    using Cfg = RingCfg<C, S>;
    extern __shared__ __align__(128) uint8_t smem[];
    uint8_t *ring = smem;
    double *xs_all = reinterpret_cast<double *>(smem + Cfg::kRing);
    Item *slot_item = reinterpret_cast<Item *>(smem + Cfg::kRing + Cfg::kX);
    uint64_t *bars = reinterpret_cast<uint64_t *>(smem + Cfg::kRing + Cfg::kX + Cfg::kSlots);
    const uint32_t full0 = smem_u32(bars), empty0 = smem_u32(bars + S);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x < S) {
        mbar_init(full0 + 8 * threadIdx.x, 1);
        mbar_init(empty0 + 8 * threadIdx.x, 1);
    }
    if (threadIdx.x == 0) fence_mbar_init();
    __syncthreads();
    const int64_t beg = p.cta_begin[blockIdx.x], end = p.cta_begin[blockIdx.x + 1];

    if (warp == 0) {
        // ---------------------------------------------------- producer ----
        // lane j owns slot j: items beg + j, beg + j + S, beg + j + 2S, ...
        if (lane < S) {
            const uint32_t full = full0 + 8 * lane, empty = empty0 + 8 * lane;
            const uint32_t dst0 = smem_u32(ring) + (uint32_t)lane * kItemBytes;
            uint32_t round = 0;
            for (int64_t k = beg + lane; k < end; k += S, ++round) {
                const int4 *src = reinterpret_cast<const int4 *>(p.items + k);
                const int4 a = __ldg(src), b = __ldg(src + 1);
                Item it;
                it.I = a.x; it.tb = a.y; it.kb = a.z; it.ke = a.w;
                it.offb = (uint32_t)b.x; it.offe = (uint32_t)b.y; it.split = b.z; it.part_nt = b.w;
                if (round > 0) mbar_wait(empty, (round - 1) & 1u);
                slot_item[lane] = it;
                const ItemParts pt = item_parts(it, p.m);
                fence_proxy_async();
                mbar_expect_tx(full, pt.total);
                uint32_t d = dst0;
                if (pt.pay) bulk_g2s(d, p.payload + (size_t)it.offb * 16, pt.pay, full);
                d += pt.pay;
                if (pt.dsc)
                    bulk_g2s(d, reinterpret_cast<const uint8_t *>(p.tdesc + it.tb) - pt.dsc_skew, pt.dsc, full);
                d += pt.dsc;
                if (pt.rp) {
                    bulk_g2s(d, p.remRowPtr + 16 * (int64_t)it.I, pt.rp, full);
                    d += pt.rp;
                    bulk_g2s(d, reinterpret_cast<const uint8_t *>(p.remCol + it.kb) - pt.col_skew, pt.col, full);
                    d += pt.col;
                    bulk_g2s(d, reinterpret_cast<const uint8_t *>(p.remVal + it.kb) - pt.val_skew, pt.val, full);
                }
            }
        }
        return;
    }

    // -------------------------------------------------------- consumers ---
    const int c = warp - 1;
    const int h = lane >> 4, r = lane & 15;
    double *xs = xs_all + c * 16 * kItemTiles;
    for (int64_t q = c; beg + q < end; q += C) {
        const int slot = (int)(q % S);
        mbar_wait(full0 + 8 * slot, (uint32_t)(q / S) & 1u);
        const Item it = slot_item[slot];
        const ItemParts pt = item_parts(it, p.m);
        const uint8_t *pay = ring + (uint32_t)slot * kItemBytes;
        const int nt = it.part_nt >> 24;
        // per-lane tile descriptor (lane t < nt holds tile tb + t)
        uint2 d = make_uint2(0u, 7u << 27);
        if (lane < nt) d = reinterpret_cast<const uint2 *>(pay + pt.pay + pt.dsc_skew)[lane];
        const int fmt = (int)(d.y >> 27) == 0 ? (int)(d.x >> 27) : 7;  // 7: no tile
        const int aux = (int)(d.y & 31u), nz = (int)((d.y >> 5) & 511u);
        // byte offset of each tile in the payload: exclusive warp scan of sizes
        int off = (int)((d.y >> 14) & 255u) * 16;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int v = __shfl_up_sync(FULL, off, o);
            if (lane >= o) off += v;
        }
        off -= (int)((d.y >> 14) & 255u) * 16;
        // x segments: lane l loads x[16 J_t + (l & 15)] for tiles t = 2k + h
        {
            const uint32_t J = d.x & 0x7FFFFFFu;
            double xv[kItemTiles / 2];
#pragma unroll
            for (int k = 0; k < kItemTiles / 2; ++k) {
                const int t = 2 * k + h;
                const int64_t col = 16 * (int64_t)__shfl_sync(FULL, J, t) + r;
                xv[k] = (t < nt && col < p.n) ? __ldg(p.x + col) : 0.0;
            }
#pragma unroll
            for (int k = 0; k < kItemTiles / 2; ++k) xs[(2 * k + h) * 16 + r] = xv[k];
        }
        double acc = 0.0;
        if (pt.rp) {
            const uint8_t *rb = pay + pt.pay + pt.dsc;
            remainder_rows(p, it.I, it.kb, it.ke, reinterpret_cast<const int *>(rb),
                           reinterpret_cast<const int *>(rb + pt.rp + pt.col_skew),
                           reinterpret_cast<const double *>(rb + pt.rp + pt.col + pt.val_skew), lane, acc);
        }
        __syncwarp();
        // tiles, grouped by format, two at a time (one per half-warp)
        const unsigned present = __reduce_or_sync(FULL, lane < nt ? 1u << fmt : 0u);
#pragma unroll 1
        for (int f = 0; f < 7; ++f) {
            if (!((present >> f) & 1u)) continue;
            unsigned mask = __ballot_sync(FULL, fmt == f);
            while (mask) {
                const int t0 = __ffs(mask) - 1;
                mask &= mask - 1;
                const int t1 = mask ? __ffs(mask) - 1 : -1;
                if (t1 >= 0) mask &= mask - 1;
                const int th = h ? t1 : t0;
                const bool ok = th >= 0;
                const int src = ok ? th : t0;
                const int a = __shfl_sync(FULL, aux, src);
                const int n_ = __shfl_sync(FULL, nz, src);
                const int o = __shfl_sync(FULL, off, src);
                const uint8_t *P = pay + o;
                const double *X = xs + 16 * src;
                switch (f) {
                case F_CSR: half_csr(P, n_, X, r, ok, acc); break;
                case F_ELL: half_ell(P, a, X, r, ok, acc); break;
                case F_DNS: half_dns(P, X, r, ok, acc); break;
                case F_DNSCOL: half_dnscol(P, a, X, r, ok, acc); break;
                case F_DNSROW: half_dnsrow(P, a, X, r, ok, acc); break;
                case F_COO:
                    half_coo(reinterpret_cast<const double *>(P), P + 8 * n_, n_, X, r, ok, acc);
                    break;
                case F_HYB: half_hyb(P, a, n_, X, r, ok, acc); break;
                default: break;
                }
            }
        }
        acc += __shfl_xor_sync(FULL, acc, 16);
        write_rows(p, it, lane, acc);
        __syncwarp();
        if (lane == 0) mbar_arrive(empty0 + 8 * slot);
    }
}

template <int C, int S>
KernelChoice ring_choice(const char *name) {
    return {name, tilespmv_fp64_ring<C, S>, RingCfg<C, S>::kThreads, (int)RingCfg<C, S>::kSmem, 1, true};
}

}  // namespace

KernelChoice kernel_ring(int variant) {
    switch (variant) {
    case 3: return ring_choice<8, 24>("ring_c8_s24");
    case 4: return ring_choice<6, 24>("ring_c6_s24");
    case 5: return ring_choice<12, 24>("ring_c12_s24");
    case 6: return ring_choice<4, 24>("ring_c4_s24");
    case 7: return ring_choice<10, 20>("ring_c10_s20");
    default: return ring_choice<12, 24>("ring_c12_s24");
    }
}

}  // namespace tsp
