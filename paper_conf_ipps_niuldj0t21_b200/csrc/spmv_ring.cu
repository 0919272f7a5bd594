// spmv_ring.cu -- the timed hot path (default kernel): y = A_tiles*x + A_rem*x
// in fp64 on sm_100a (§III.C P:118-173 warp-level tile SpMV, P:199
// load balancing, P:201 DeferredCOO remainder).
//
// Warp-specialised persistent kernel, one CTA per SM, each CTA owning a
// contiguous, cost-balanced chunk of work items:
//   * producer warp: lane j owns shared-memory slot j and streams items
//     beg + j, beg + j + S, ... into it with TMA bulk copies
//     (cp.async.bulk, 1-D): tile payloads, 8-byte tile descriptors,
//     remainder rowptr/col/val.  Completion is counted in bytes on the
//     slot's "full" mbarrier; the slot is reused after its "empty" mbarrier.
//   * C consumer warps: consumer c serves slots c, c+C, ... (S % C == 0, so
//     every slot has exactly one consumer and mbarrier parities cannot
//     alias).  Per item it stages the x segment of every tile (one 128-byte
//     line) in shared memory, lists the tiles grouped by format, runs the
//     format routines and writes y, then releases the slot.
//   * Tiles run TWO AT A TIME: each half-warp takes one tile of a
//     same-format pair, one lane per tile row (the per-row decomposition of
//     the paper's CSR/ELL/DnsCol routines), so dispatch
//     and setup are shared by two tiles and every loop has a warp-uniform
//     trip count with predicated FMAs.  Row r's two half sums meet in
//     acc(r) + acc(r + 16).  All shared-memory traffic uses 32-bit shared
//     addresses with immediate offsets.
//   * No floating-point atomics: y is bitwise deterministic.
#include "spmv_common.cuh"

namespace tsp {
namespace {

template <int C, int S, int SLOT>
struct RingCfg {
    static_assert(S % C == 0, "slot s must always be served by consumer s mod C");
    static_assert(S <= 32, "one producer lane per slot");
    static_assert(SLOT % 16 == 0 && SLOT <= kItemBytesMax, "slot size");
    static constexpr uint32_t kItemBytes = SLOT;
    static constexpr uint32_t kRing = (uint32_t)S * SLOT;
    static constexpr uint32_t kXPer = kItemTiles * 16 * 8;  // x segments per consumer
    static constexpr uint32_t kListPer = 128;               // tile list per consumer
    static constexpr uint32_t kX = (uint32_t)C * kXPer;
    static constexpr uint32_t kList = (uint32_t)C * kListPer;
    static constexpr uint32_t kSlots = (uint32_t)S * sizeof(Item);
    static constexpr uint32_t kBars = 2u * S * 8u;
    static constexpr uint32_t kSmem = kRing + kX + kList + kSlots + kBars + 256;  // +256: loads may overrun a slot
    static constexpr int kThreads = 32 * (C + 1);
};

// ------------------------------------------------- shared-memory access ----
__device__ __forceinline__ double lds_f64(uint32_t a) {
    double v;
    asm volatile("ld.shared.f64 %0, [%1];" : "=d"(v) : "r"(a));
    return v;
}
__device__ __forceinline__ uint32_t lds_u8(uint32_t a) {
    uint32_t v;
    asm volatile("ld.shared.u8 %0, [%1];" : "=r"(v) : "r"(a));
    return v;
}
__device__ __forceinline__ int lds_s32(uint32_t a) {
    int v;
    asm volatile("ld.shared.s32 %0, [%1];" : "=r"(v) : "r"(a));
    return v;
}
__device__ __forceinline__ uint2 lds_v2u32(uint32_t a) {
    uint2 v;
    asm volatile("ld.shared.v2.u32 {%0, %1}, [%2];" : "=r"(v.x), "=r"(v.y) : "r"(a));
    return v;
}
__device__ __forceinline__ void sts_u32(uint32_t a, uint32_t v) {
    asm volatile("st.shared.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
__device__ __forceinline__ void sts_f64(uint32_t a, double v) {
    asm volatile("st.shared.f64 [%0], %1;" ::"r"(a), "d"(v) : "memory");
}

// --------------------------------------------- half-warp tile routines -----
// Lane r of a half owns row r of its tile.  P: shared address of the tile's
// payload, X: of its 16 x values; ok: the half has a tile (else it runs the
// other half's tile with its FMAs masked).  Loads past a tile's end stay
// inside the CTA's shared memory and are masked out of the FMA.

// CSR: csrVal row-major | csrRowPtr[16] u8 | 4-bit columns (Alg. 2)
__device__ __forceinline__ void half_csr(uint32_t P, int nz, uint32_t X, int r, bool ok, double &acc) {
    const uint32_t rp = P + 8 * nz;
    const int beg = (int)lds_u8(rp + r);
    const int end = r < 15 ? (int)lds_u8(rp + r + 1) : nz;
    const int len = ok ? end - beg : 0;
    const int trips = (int)__reduce_max_sync(FULL, (unsigned)len);
    // nibble of entry beg+i: byte (beg+i)>>1 = b_even + i/2 (i even) or
    // b_odd + i/2 (i odd), shifted by s_even / s_odd
    const uint32_t cb = rp + 16 + (beg >> 1);
    const uint32_t odd = beg & 1;
    const uint32_t b_odd = cb + odd;
    const uint32_t s_even = 4 * odd, s_odd = 4 - 4 * odd;
    const uint32_t V = P + 8 * beg;
    // four entries per iteration: independent load chains, two FMA chains
    double a1 = 0.0;
#pragma unroll 1
    for (int i = 0; i < trips; i += 4) {
        const uint32_t c0 = (lds_u8(cb + (i >> 1)) >> s_even) & 15u;
        const uint32_t c1 = (lds_u8(b_odd + (i >> 1)) >> s_odd) & 15u;
        const uint32_t c2 = (lds_u8(cb + (i >> 1) + 1) >> s_even) & 15u;
        const uint32_t c3 = (lds_u8(b_odd + (i >> 1) + 1) >> s_odd) & 15u;
        const double v0 = lds_f64(V + 8 * i), v1 = lds_f64(V + 8 * i + 8);
        const double v2 = lds_f64(V + 8 * i + 16), v3 = lds_f64(V + 8 * i + 24);
        const double x0 = lds_f64(X + 8 * c0), x1 = lds_f64(X + 8 * c1);
        const double x2 = lds_f64(X + 8 * c2), x3 = lds_f64(X + 8 * c3);
        if (i < len) acc = fma(v0, x0, acc);
        if (i + 1 < len) a1 = fma(v1, x1, a1);
        if (i + 2 < len) acc = fma(v2, x2, acc);
        if (i + 3 < len) a1 = fma(v3, x3, a1);
    }
    acc += a1;
}

// ELL: slots k*16 + r column-major | 4-bit columns (Alg. 4).
// Pads (k >= 1 with column 0, reading R26) are skipped.
__device__ __forceinline__ void half_ell(uint32_t P, int w, uint32_t X, int r, bool ok, double &acc) {
    const int wq = ok ? w : 0;
    const int trips = (int)__reduce_max_sync(FULL, (unsigned)wq);
    const uint32_t ci = P + 128 * w + (r >> 1);
    const uint32_t sh = 4 * (r & 1);
    const uint32_t V = P + 8 * r;
#pragma unroll 4
    for (int k = 0; k < trips; ++k) {
        const uint32_t c = (lds_u8(ci + 8 * k) >> sh) & 15u;
        const double v = lds_f64(V + 128 * k);
        const double xv = lds_f64(X + 8 * c);
        if (k < wq && (k == 0 || c != 0)) acc = fma(v, xv, acc);
    }
}

// Dns: 256 values column-major
__device__ __forceinline__ void half_dns(uint32_t P, uint32_t X, int r, bool ok, double &acc) {
    const uint32_t V = P + 8 * r;
    double a0 = 0.0, a1 = 0.0;
#pragma unroll
    for (int c = 0; c < 16; c += 2) {
        a0 = fma(lds_f64(V + 128 * c), lds_f64(X + 8 * c), a0);
        a1 = fma(lds_f64(V + 128 * c + 128), lds_f64(X + 8 * c + 8), a1);
    }
    if (ok) acc += a0 + a1;
}

// DnsCol: full column q holds value q*16 + r, column id colid[q]
__device__ __forceinline__ void half_dnscol(uint32_t P, int nc, uint32_t X, int r, bool ok, double &acc) {
    const int nq = ok ? nc : 0;
    const int trips = (int)__reduce_max_sync(FULL, (unsigned)nq);
    const uint32_t cid = P + 128 * nc;
    for (int q = 0; q < trips; ++q) {
        const double v = lds_f64(P + 8 * (16 * q + r));
        const double xv = lds_f64(X + 8 * (lds_u8(cid + q) & 15u));
        if (q < nq) acc = fma(v, xv, acc);
    }
}

// DnsRow: full row q (id rowid[q]) holds values q*16 + c; the
// lane of row rowid[q] sums the 16 products of its row.
__device__ __forceinline__ void half_dnsrow(uint32_t P, int nr, uint32_t X, int r, bool ok, double &acc) {
    const uint32_t rid = P + 128 * nr;
    int q_r = -1;
    const int nq = ok ? nr : 0;
    for (int q = 0; q < 7; ++q)
        if (q < nq && (int)lds_u8(rid + q) == r) q_r = q;
    const bool mine = q_r >= 0;
    if (__any_sync(FULL, mine)) {
        const uint32_t Vr = P + 128 * (mine ? q_r : 0);
        double a0 = 0.0, a1 = 0.0;
#pragma unroll
        for (int c = 0; c < 16; c += 2) {
            a0 = fma(lds_f64(Vr + 8 * c), lds_f64(X + 8 * c), a0);
            a1 = fma(lds_f64(Vr + 8 * c + 8), lds_f64(X + 8 * c + 8), a1);
        }
        if (mine) acc += a0 + a1;
    }
}

// COO entries: value j, packed (row << 4 | col) byte (Alg. 3); the lane
// of the entry's row adds it (no atomics, fixed order)
__device__ __forceinline__ void half_coo(uint32_t V, uint32_t rc, int n, uint32_t X, int r, bool ok, double &acc) {
    const int nq = ok ? n : 0;
    const int trips = (int)__reduce_max_sync(FULL, (unsigned)nq);
#pragma unroll 2
    for (int j = 0; j < trips; ++j) {
        const uint32_t b = lds_u8(rc + j);
        const double v = lds_f64(V + 8 * j);
        const double xv = lds_f64(X + 8 * (b & 15u));
        if (j < nq && (int)(b >> 4) == r) acc = fma(v, xv, acc);
    }
}

// HYB: ELL(w) values | COO values | ELL 4-bit columns | COO (row<<4|col)
__device__ __forceinline__ void half_hyb(uint32_t P, int w, int nz, uint32_t X, int r, bool ok, double &acc) {
    const int kc = nz - 16 * w;
    const uint32_t ei = P + 128 * w + 8 * kc;
    const int wq = ok ? w : 0;
    const int trips = (int)__reduce_max_sync(FULL, (unsigned)wq);
    const uint32_t sh = 4 * (r & 1);
    for (int k = 0; k < trips; ++k) {
        const double v = lds_f64(P + 8 * (16 * k + r));
        const double xv = lds_f64(X + 8 * ((lds_u8(ei + 8 * k + (r >> 1)) >> sh) & 15u));
        if (k < wq) acc = fma(v, xv, acc);
    }
    half_coo(P + 128 * w, ei + 8 * w, kc, X, r, ok, acc);
}

// ------------------------------------------------------------ kernel -------
// descriptor entries: see k_dsc_write (schedule.cu)
template <int C, int S, int SLOT>
__global__ void __launch_bounds__(RingCfg<C, S, SLOT>::kThreads, 1) tilespmv_fp64_ring(const Params p) {
    using Cfg = RingCfg<C, S, SLOT>;
    constexpr uint32_t kItemBytes = Cfg::kItemBytes;
    extern __shared__ __align__(128) uint8_t smem[];
    Item *slot_item = reinterpret_cast<Item *>(smem + Cfg::kRing + Cfg::kX + Cfg::kList);
    uint64_t *bars = reinterpret_cast<uint64_t *>(smem + Cfg::kRing + Cfg::kX + Cfg::kList + Cfg::kSlots);
    const uint32_t sbase = smem_u32(smem);
    const uint32_t full0 = smem_u32(bars), empty0 = smem_u32(bars + S);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x < S) {
        mbar_init(full0 + 8 * threadIdx.x, 1);
        mbar_init(empty0 + 8 * threadIdx.x, 1);
    }
    if (threadIdx.x == 0) fence_mbar_init();
    __syncthreads();
    const int beg = (int)p.cta_begin[blockIdx.x], end = (int)p.cta_begin[blockIdx.x + 1];

    if (warp == 0) {
        // ---------------------------------------------------- producer ----
        if (lane < S) {
            const uint32_t full = full0 + 8 * lane, empty = empty0 + 8 * lane;
            const uint32_t dst0 = sbase + (uint32_t)lane * kItemBytes;
            uint32_t round = 0;
            for (int k = beg + lane; k < end; k += S, ++round) {
                const int4 *src = reinterpret_cast<const int4 *>(p.items + k);
                const int4 a = __ldg(src), b = __ldg(src + 1), e = __ldg(src + 2);
                Item it;
                it.I = a.x; it.tb = a.y; it.kb = a.z; it.ke = a.w;
                it.offb = (uint32_t)b.x; it.offe = (uint32_t)b.y; it.split = b.z; it.part_nt = b.w;
                it.dbeg = e.x; it.ndsc = e.y; it.pad0 = e.z; it.pad1 = e.w;
                if (round > 0) mbar_wait(empty, (round - 1) & 1u);
                slot_item[lane] = it;
                const ItemParts pt = item_parts(it, p.m);
                fence_proxy_async();
                mbar_expect_tx(full, pt.total);
                uint32_t d = dst0;
                if (pt.pay) bulk_g2s(d, p.payload + (size_t)it.offb * 16, pt.pay, full);
                d += pt.pay;
                if (pt.dsc)
                    bulk_g2s(d, reinterpret_cast<const uint8_t *>(p.tdesc + it.dbeg) - pt.dsc_skew, pt.dsc, full);
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
    // Software pipeline: while item k is computed, the global x loads of
    // item k + C (this consumer's next item) are already in flight.
    const int c = warp - 1;
    const int h = lane >> 4, r = lane & 15;
    const uint32_t xs = sbase + Cfg::kRing + (uint32_t)c * Cfg::kXPer;
    const uint32_t list = sbase + Cfg::kRing + Cfg::kX + (uint32_t)c * Cfg::kListPer;
    const uint32_t n32 = (uint32_t)p.n;

    struct Prep {
        Item it;
        ItemParts pt;
        uint32_t pay;
        double xt[kItemTiles / 2];  // x[16 J_t + r] for tiles t = 2k + h
        double xr[kShortRow / 2];   // x of this lane's short remainder entries
    };
    // list = per-consumer scratch: J of each tile by tile index (64 B)
    auto prepare = [&](Prep &P, int slot, uint32_t round) {
        mbar_wait(full0 + 8 * slot, round & 1u);
        P.it = slot_item[slot];
        P.pt = item_parts(P.it, p.m);
        P.pay = sbase + (uint32_t)slot * kItemBytes;
        const int nt = P.it.part_nt >> 24;
        if (lane < P.it.ndsc) {
            const uint2 d = lds_v2u32(P.pay + P.pt.pay + P.pt.dsc_skew + 8 * lane);
            if (!((d.y >> 27) & 1u)) sts_u32(list + 4 * ((d.y >> 23) & 15u), d.x & 0x7FFFFFFu);
        }
        __syncwarp();
#pragma unroll
        for (int kk = 0; kk < kItemTiles / 2; ++kk) {
            const int t = 2 * kk + h;
            P.xt[kk] = 0.0;
            if (t < nt) {
                const uint32_t col = 16u * (uint32_t)lds_s32(list + 4 * t) + (uint32_t)r;
                if (col < n32) P.xt[kk] = __ldg(p.x + col);
            }
        }
#pragma unroll
        for (int i = 0; i < kShortRow / 2; ++i) P.xr[i] = 0.0;
        if (P.pt.rp) {  // x of the short remainder rows (two lanes per row)
            const uint32_t rb = P.pay + P.pt.pay + P.pt.dsc;
            const int rows = (int)imin64(16, p.m - 16 * (int64_t)P.it.I);
            int b = lds_s32(rb + 4 * min(r, rows)), e = lds_s32(rb + 4 * min(r + 1, rows));
            b = max(b, P.it.kb) - P.it.kb;
            e = min(e, P.it.ke) - P.it.kb;
            const uint32_t colS = rb + P.pt.rp + P.pt.col_skew;
            if (e - b <= kShortRow) {
#pragma unroll
                for (int i = 0; i < kShortRow / 2; ++i) {
                    const int kq = b + h + 2 * i;
                    if (kq < e) P.xr[i] = __ldg(p.x + (uint32_t)lds_s32(colS + 4 * kq));
                }
            }
        }
        __syncwarp();  // list scratch reusable
    };

    int k = beg + c;
    if (k >= end) return;
    int slot = c;
    uint32_t round = 0;
    Prep cur;
    prepare(cur, slot, round);
    for (;;) {
        // next item of this consumer: issue its loads before computing this one
        int nslot = slot + C;
        uint32_t nround = round;
        if (nslot >= S) {
            nslot -= S;
            ++nround;
        }
        const bool has_next = k + C < end;
        Prep nxt;
        if (has_next) prepare(nxt, nslot, nround);

        const Item &it = cur.it;
        const ItemParts &pt = cur.pt;
        const uint32_t pay = cur.pay;
#pragma unroll
        for (int kk = 0; kk < kItemTiles / 2; ++kk) sts_f64(xs + 8 * ((2 * kk + h) * 16 + r), cur.xt[kk]);
        const int npairs = it.ndsc >> 1;
        const uint32_t dsc = pay + pt.pay + pt.dsc_skew;
        double acc = 0.0;
        if (pt.rp) {
            const uint32_t rb = pay + pt.pay + pt.dsc;
            const int rows = (int)imin64(16, p.m - 16 * (int64_t)it.I);
            int b = lds_s32(rb + 4 * min(r, rows)), e = lds_s32(rb + 4 * min(r + 1, rows));
            b = max(b, it.kb) - it.kb;
            e = min(e, it.ke) - it.kb;
            const uint32_t colS = rb + pt.rp + pt.col_skew, valS = rb + pt.rp + pt.col + pt.val_skew;
            const bool is_short = e - b <= kShortRow;
            if (is_short) {
#pragma unroll
                for (int i = 0; i < kShortRow / 2; ++i) {
                    const int kq = b + h + 2 * i;
                    if (kq < e) acc = fma(lds_f64(valS + 8 * kq), cur.xr[i], acc);
                }
            }
            unsigned longs = __ballot_sync(FULL, lane < 16 && !is_short);
            while (longs) {  // rows longer than kShortRow: the whole warp strides the row
                const int rr = __ffs(longs) - 1;
                longs &= longs - 1;
                const int bb = __shfl_sync(FULL, b, rr), ee = __shfl_sync(FULL, e, rr);
                double s = 0.0;
                for (int k0 = bb; k0 < ee; k0 += 128) {
                    int cs[4];
                    double vs[4], xv[4];
#pragma unroll
                    for (int i = 0; i < 4; ++i) {
                        const int kq = k0 + lane + 32 * i;
                        cs[i] = kq < ee ? lds_s32(colS + 4 * kq) : 0;
                        vs[i] = kq < ee ? lds_f64(valS + 8 * kq) : 0.0;
                    }
#pragma unroll
                    for (int i = 0; i < 4; ++i) xv[i] = (k0 + lane + 32 * i < ee) ? __ldg(p.x + (uint32_t)cs[i]) : 0.0;
#pragma unroll
                    for (int i = 0; i < 4; ++i)
                        if (k0 + lane + 32 * i < ee) s = fma(vs[i], xv[i], s);
                }
#pragma unroll
                for (int o = 16; o >= 1; o >>= 1) s += __shfl_xor_sync(FULL, s, o);
                if (lane == rr) acc += s;
            }
        }
        __syncwarp();
#pragma unroll 1
        for (int q = 0; q < npairs; ++q) {
            const uint2 e = lds_v2u32(dsc + 16 * q + 8 * h);
            const int f = (int)(e.x >> 27);  // same for both halves by construction
            const bool ok = !((e.y >> 27) & 1u);
            const int a = (int)(e.y & 31u);
            const int nz = (int)((e.y >> 5) & 511u);
            const uint32_t P = pay + 16 * ((e.y >> 14) & 511u);
            const uint32_t X = xs + 128 * ((e.y >> 23) & 15u);
            switch (f) {
            case F_CSR: half_csr(P, nz, X, r, ok, acc); break;
            case F_ELL: half_ell(P, a, X, r, ok, acc); break;
            case F_DNS: half_dns(P, X, r, ok, acc); break;
            case F_DNSCOL: half_dnscol(P, a, X, r, ok, acc); break;
            case F_DNSROW: half_dnsrow(P, a, X, r, ok, acc); break;
            case F_COO: half_coo(P, P + 8 * nz, nz, X, r, ok, acc); break;
            case F_HYB: half_hyb(P, a, nz, X, r, ok, acc); break;
            default: break;
            }
        }
        acc += __shfl_xor_sync(FULL, acc, 16);
        write_rows(p, it, lane, acc);
        __syncwarp();
        if (lane == 0) mbar_arrive(empty0 + 8 * slot);
        if (!has_next) break;
        k += C;
        slot = nslot;
        round = nround;
        cur = nxt;
    }
}

template <int C, int S, int SLOT>
KernelChoice ring_choice(const char *name) {
    using Cfg = RingCfg<C, S, SLOT>;
    return {name, tilespmv_fp64_ring<C, S, SLOT>, Cfg::kThreads, (int)Cfg::kSmem, 1, true, SLOT};
}

}  // namespace

// consumers C, slots S (S/C slots per consumer: >= 3 lets the next item's x
// loads overlap the current item), slot size SLOT bytes
KernelChoice kernel_ring(int variant) {
    switch (variant) {
    case 3: return ring_choice<8, 24, 8192>("ring_c8_s24_8k");
    case 4: return ring_choice<10, 30, 5120>("ring_c10_s30_5k");
    case 5: return ring_choice<8, 32, 6144>("ring_c8_s32_6k");
    case 6: return ring_choice<12, 24, 8192>("ring_c12_s24_8k");
    case 7: return ring_choice<9, 27, 6144>("ring_c9_s27_6k");
    case 8: return ring_choice<7, 28, 6144>("ring_c7_s28_6k");
    case 9: return ring_choice<10, 30, 6144>("ring_c10_s30_6k");
    case 10: return ring_choice<16, 32, 5632>("ring_c16_s32_5.5k");
    case 11: return ring_choice<14, 28, 6144>("ring_c14_s28_6k");
    case 12: return ring_choice<13, 26, 6656>("ring_c13_s26_6.5k");
    default: return ring_choice<10, 30, 5120>("ring_c10_s30_5k");
    }
}

}  // namespace tsp
