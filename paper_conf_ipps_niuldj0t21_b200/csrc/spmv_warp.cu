// spmv_warp.cu -- the SpMV kernels: y = A_tiles*x + A_rem*x in fp64 on
// sm_100a (§III.C P:118-173 warp-level tile SpMV, P:199 load
// balancing, P:201 DeferredCOO remainder).
//
// Every warp is its own producer and consumer.  Per work item, lane 0 stages
// the item's execution blob (descriptor list, tile payloads, remainder
// rowptr/col/val; blob_parts) into the warp's shared-memory slot with ONE TMA
// bulk copy (cp.async.bulk, L2 evict-first) completing on the warp's
// mbarrier.  The warp then
//   1. starts the x segment of every tile (one 128-byte line) with cp.async
//      (L2 evict-last; the tail of x past n reads as 0),
//   2. runs the fused CSR remainder rows of the tile row,
//   3. runs the tiles two at a time, format group by format group, with the
//      half-warp routines of spmv_tiles.cuh (one lane per tile row),
//   4. writes y once per row (split tile rows: register carry inside a group
//      of parts, one partial per group for hub rows).
// Latency is hidden by warp count; the next item's record is prefetched into
// registers.  No floating-point atomics: y is bitwise deterministic.
//
// Three kernels share this item code (schedule.cu picks one per handle):
//   tilespmv_fp64_sm<32,4608,16> SM_QUEUE: one CTA of 32 warps per SM, 4.5 KB
//                                 slots, warps claim units from a
//                                 shared-memory queue (222 KB of shared memory)
//   tilespmv_fp64_sm<32,3136,4,1024> GATHER: the same with 3 KB slots, at
//                                 most 4 tiles per item and an 8 KB x cache of
//                                 the 1,024 most-gathered remainder columns
//                                 (130 KB in all: the 132 KB carve-out leaves
//                                 ~124 KB of L1 to the remainder's x gathers;
//                                 power-law matrices in DEFERRED mode), every
//                                 remainder through the product pre-pass, units
//                                 claimed costliest first
//   tilespmv_fp64_warp<4,10752>  DENSE_ROWS: 16 warps per SM, 10.5 KB slots,
//                                 a static cost-balanced item chunk per warp
//                                 (dense tile rows: one tile row stays one item)
#include "spmv_tiles.cuh"

namespace tsp {

#ifdef TSP_TRACE
// development build only (scripts/trace_items.py): %globaltimer stamps of the
// first kTraceItems items of every warp: start, blob landed, item info, end
constexpr int kTraceItems = 192;
__device__ unsigned long long *g_trace = nullptr;
__device__ __forceinline__ unsigned long long gtimer() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}
#define TSP_STAMP(gw, j, slot) \
    do { if (g_trace && lane == 0 && (j) < kTraceItems) g_trace[((size_t)(gw) * kTraceItems + (j)) * 4 + (slot)] = gtimer(); } while (0)
// item k, blob bytes, row-group tile rows, tiles
#define TSP_INFO(gw, j, k, it) \
    do { if (g_trace && lane == 0 && (j) < kTraceItems) g_trace[((size_t)(gw) * kTraceItems + (j)) * 4 + 2] = \
        ((unsigned long long)(k) << 32) | ((it).val_tot & 0xFFFF0000u) | (((it).jt_rows_pay & 0xFFu) << 8) | (((it).part_nt >> 24) & 31u); } while (0)
// the warp's SM, after the item stamps
#define TSP_SMID(gw, nw) \
    do { if (g_trace && lane == 0) { unsigned sm; asm volatile("mov.u32 %0, %smid;" : "=r"(sm)); \
         g_trace[(size_t)(nw) * kTraceItems * 4 + (gw)] = sm; } } while (0)
#else
#define TSP_STAMP(gw, j, slot) do { } while (0)
#define TSP_INFO(gw, j, k, it) do { } while (0)
#define TSP_SMID(gw, nw) do { } while (0)
#endif

namespace {


template <int WARPS, int SLOT, int XT = kItemTiles, int XC = 0>
struct WarpCfg {
    static_assert(SLOT % 16 == 0 && SLOT <= kItemBytesMax && XT % 4 == 0 && XT <= kItemTiles, "slot size");
    // [x stage of every warp, XT x 128 B, 128-byte aligned] [per warp: slot |
    // mbarrier] [x cache: XC x 8 B]
    static constexpr uint32_t kX = XT * 16 * 8;
    static constexpr uint32_t kPer = SLOT + 16;
    static constexpr uint32_t kXc = WARPS * (kX + kPer);  // x cache offset
    static constexpr uint32_t kSmem = kXc + XC * 8 + 256;  // +256: loads may overrun a slot
    static constexpr int kThreads = 32 * WARPS;
};

__device__ __forceinline__ WItem load_witem(const WItem *w, int k) {
    const int4 *src = reinterpret_cast<const int4 *>(w + k);
    const int4 a = __ldg(src), b = __ldg(src + 1);
    WItem it;
    it.blob16 = (uint32_t)a.x; it.I = (uint32_t)a.y; it.split = a.z; it.part_nt = a.w;
    it.jt_rows_pay = (uint32_t)b.x; it.rp_col = (uint32_t)b.y; it.val_tot = (uint32_t)b.z; it.groups = (uint32_t)b.w;
    return it;
}

// ------------------------------------------------ fused CSR remainder -------
// The remainder rows of a tile row are summed by their own lanes:
// lane r (or r + 16) owns row r.  Which routine runs depends only on the
// item's content (its longest row), so every sum order is a function of the
// tile row's own entries (shard and grouping invariant):
//   <= 4 entries per row (stencils): two lanes per row, one round of gathers;
//   <= 32: two lanes per row, two entries each per step, all rows at once;
//   longer (power-law hubs): the flat pass below.
// A masked term never reads an x entry the item does not reference (a halo
// rank holds only its own rows and its halo): the two-lane paths multiply
// 0.0 by x at the item's first remainder column, the flat pass rounds each
// product on its own and selects +0.0.
constexpr int kShortRow = 16;  // flat pass: rows of up to this many entries two lanes per row

// Product pre-pass (GATHER kernel, PRE = true): the x gathers of all E
// remainder entries of an item, one lane per entry and kGatherDepth gathers
// in flight per lane, each product v*x rounded on its own and stored over its
// value in the slot; x comes from the CTA's shared-memory x cache for the
// most-gathered columns (blob column ~slot).  The row sums then read
// products from shared memory in the same order as the inline-gather form
// (PRE = false, the other kernels), so the flat pass and row groups give the
// same bits either way.  The slot was written through the generic proxy: the
// caller fences before the next TMA copy into it.
constexpr int kGatherDepth = 2;  // 2 / 4 / 8 in flight: R-MAT 94.3 / 95.8 / 109 us (more thrash the L1)
__device__ __forceinline__ void rem_products(const Params &p, uint32_t colS, uint32_t valS, int E, uint64_t x_policy,
                                             uint32_t xcS, int lane) {
#pragma unroll 1
    for (int base = 0; base < E; base += 32 * kGatherDepth) {
        double xv[kGatherDepth];
#pragma unroll
        for (int j = 0; j < kGatherDepth; ++j) {
            const int k = base + lane + 32 * j;
            xv[j] = 0.0;
            if (k < E) {
                const int c = lds_s32(colS + 4 * k);  // < 0: slot ~c of the CTA's x cache (GATHER)
                TSP_CHECK(c < 0 ? ~c < p.xc_n : c < p.n);
                xv[j] = c < 0 ? lds_f64(xcS + 8u * (uint32_t)~c) : ldg_hint(p.x + (uint32_t)c, x_policy);
            }
        }
#pragma unroll
        for (int j = 0; j < kGatherDepth; ++j) {
            const int k = base + lane + 32 * j;
            if (k < E) sts_f64(valS + 8 * k, __dmul_rn(lds_f64(valS + 8 * k), xv[j]));
        }
    }
    __syncwarp();
}

// product of staged remainder entry k if k < e, else +0.0 (rounded on its
// own): read back after rem_products (PRE), or gathered here
template <bool PRE>
__device__ __forceinline__ double rem_product(const Params &p, int k, int e, uint32_t colS, uint32_t valS,
                                              uint64_t x_policy) {
    if (PRE) return lds_f64_lt(k, e, valS + 8 * k);
    int c;
    double v;
    lds_entry_lt(k, e, colS + 4 * k, valS + 8 * k, c, v);
    TSP_CHECK(c >= 0 && c < p.n);
    const double pr = __dmul_rn(v, ldg_hint(p.x + (uint32_t)c, x_policy));
    return k < e ? pr : 0.0;
}

// y[row] = v, and the same value into every peer copy of y (the fused
// scatter epilogue of tilespmv_run_scatter: the next iterate's rows stored
// straight into the peers' x over NVLink; nyx = 0 for a plain run)
// (SC: the scatter instantiation of each kernel; the plain one stores y only)
template <bool SC>
__device__ __forceinline__ void store_y(const Params &p, int64_t row, double v) {
    p.y[row] = v;
    if (SC) {
#pragma unroll 1
        for (int t = 0; t < p.nyx; ++t) p.yx[t][row] = v;
    }
}

// Flat remainder pass for one tile row (rows <= 16, row pointers at
// rq): rows of <= kShortRow products two lanes per row, longer rows a
// half-warp per row (two rows at a time, the whole warp for the last one)
// with an xor tree.  Returns lane r's (or r + 16's) share of row r.  The order
// of every sum depends only on this tile row.
template <bool PRE>
__device__ __forceinline__ double flat_rows(const Params &p, uint32_t rq, uint32_t colS, uint32_t valS, int rows,
                                            uint64_t x_policy, int lane) {
    const int r = lane & 15, h = lane >> 4;
    const int b = lds_s32(rq + 4 * min(r, rows)), e = lds_s32(rq + 4 * min(r + 1, rows));
    const bool lng = e - b > kShortRow;
    const int ee = lng ? b : e;
    const int trips = (int)__reduce_max_sync(FULL, (unsigned)((ee - b + 1 - h) >> 1));
    double s0 = 0.0, s1 = 0.0;
#pragma unroll 1
    for (int i = 0; i < trips; i += 2) {
        const int k0 = b + h + 2 * i;
        s0 += rem_product<PRE>(p, k0, ee, colS, valS, x_policy);
        s1 += rem_product<PRE>(p, k0 + 2, ee, colS, valS, x_policy);
    }
    double acc = s0 + s1;
    uint32_t lm = __ballot_sync(FULL, lng && h == 0 && r < rows);
#pragma unroll 1
    while (lm) {
        const int r0 = __ffs(lm) - 1;
        lm &= lm - 1;
        const int r1 = lm ? __ffs(lm) - 1 : -1;
        if (lm) lm &= lm - 1;
        const bool pair = r1 >= 0;  // warp-uniform
        const int myrow = (pair && h) ? r1 : r0;
        const int off = pair ? r : lane, stride = pair ? 16 : 32;
        const int bb = lds_s32(rq + 4 * myrow), e2 = lds_s32(rq + 4 * myrow + 4);
        const int t2 = (int)__reduce_max_sync(FULL, (unsigned)((e2 - bb + 4 * stride - 1) >> (pair ? 6 : 7)));
        double q0 = 0.0, q1 = 0.0, q2 = 0.0, q3 = 0.0;
#pragma unroll 1
        for (int t = 0; t < t2; ++t) {
            const int k = bb + off + 4 * stride * t;
            q0 += rem_product<PRE>(p, k, e2, colS, valS, x_policy);
            q1 += rem_product<PRE>(p, k + stride, e2, colS, valS, x_policy);
            q2 += rem_product<PRE>(p, k + 2 * stride, e2, colS, valS, x_policy);
            q3 += rem_product<PRE>(p, k + 3 * stride, e2, colS, valS, x_policy);
        }
        double sq = (q0 + q1) + (q2 + q3);
        if (!pair) sq += __shfl_xor_sync(FULL, sq, 16);
        sq += __shfl_xor_sync(FULL, sq, 8);
        sq += __shfl_xor_sync(FULL, sq, 4);
        sq += __shfl_xor_sync(FULL, sq, 2);
        sq += __shfl_xor_sync(FULL, sq, 1);
        if (pair ? r == myrow : lane == r0) acc += sq;
    }
    return acc;
}

// returns true if the slot now holds products (PRE: the kernel's choice, so
// every handle of one kernel sums a row the same way)
template <bool PRE>
__device__ __forceinline__ bool remainder(const Params &p, uint32_t rpS, uint32_t colS, uint32_t valS, int rows,
                                          uint64_t x_policy, uint32_t xcS, int lane, double &acc) {
    const int r = lane & 15, h = lane >> 4;
    const int b = lds_s32(rpS + 4 * min(r, rows)), e = lds_s32(rpS + 4 * min(r + 1, rows));
    const int maxlen = (int)__reduce_max_sync(FULL, (unsigned)(e - b));
    if (PRE) {  // all gathers first, then the row sums over the products
        rem_products(p, colS, valS, lds_s32(rpS + 4 * rows), x_policy, xcS, lane);
        if (maxlen > 32) {
            acc += flat_rows<true>(p, rpS, colS, valS, rows, x_policy, lane);
            return true;
        }
        // entries b + h + 2i of row r, in order
        const int trips = (int)__reduce_max_sync(FULL, (unsigned)((e - b + 1 - h) >> 1));
#pragma unroll 1
        for (int i = 0; i < trips; i += 2) {
            const int k0 = b + h + 2 * i;
            const double p0 = lds_f64_lt(k0, e, valS + 8 * k0), p1 = lds_f64_lt(k0 + 2, e, valS + 8 * k0 + 16);
            acc += p0;
            acc += p1;
        }
        return true;
    }
    if (maxlen > 32) {
        acc += flat_rows<false>(p, rpS, colS, valS, rows, x_policy, lane);
        return false;
    }
    // entries b + h + 2i and b + h + 2i + 2 of row r per step (stencils, <= 4
    // entries per row: one round of gathers); a masked entry multiplies 0.0 by
    // x at the item's first remainder column
    const int cdef = lds_s32(colS);
    const int trips = maxlen <= 4 ? 1 : (int)__reduce_max_sync(FULL, (unsigned)((e - b + 1 - h) >> 1));
#pragma unroll 1
    for (int i = 0; i < trips; i += 2) {
        const int k0 = b + h + 2 * i, k1 = k0 + 2;
        int c0, c1;
        double v0, v1;
        lds_entry_or(k0, e, colS + 4 * k0, valS + 8 * k0, cdef, c0, v0);
        lds_entry_or(k1, e, colS + 4 * k1, valS + 8 * k1, cdef, c1, v1);
        TSP_CHECK(c0 >= 0 && c0 < p.n && c1 >= 0 && c1 < p.n);
        const double x0 = ldg_hint(p.x + (uint32_t)c0, x_policy), x1 = ldg_hint(p.x + (uint32_t)c1, x_policy);
        acc = fma(v0, x0, acc);
        acc = fma(v1, x1, acc);
    }
    return false;
}

// Row-group item (internal.cuh): ntr consecutive tile rows without stored
// tiles, only remainder rows.  Two tile rows at a time, half-warp h
// on tile row g + h and lane r on its row r alone (4 running sums over the
// row's products, in entry order mod 4); rows longer than kShortRow entries
// are summed by the whole warp with an xor tree.  y is written once per row.
// A tile row's sums depend only on its own entries, so grouping never
// changes a bit of y.
template <bool PRE, bool SC>
__device__ __forceinline__ bool group_item(const Params &p, const WItem &it, uint32_t slot, uint64_t x_policy,
                                           uint32_t xcS, int lane) {
    const int ntr = (int)(it.jt_rows_pay & 0xFFu);
    const int rows_last = (int)((it.jt_rows_pay >> 8) & 31u);
    const uint32_t total = it.val_tot >> 16, rp = it.rp_col & 0xFFFFu;
    const bool has_rem = total > rp;
    const uint32_t rpS = slot + rp, colS = slot + (it.rp_col >> 16), valS = slot + (it.val_tot & 0xFFFFu);
    const int h = lane >> 4, r = lane & 15;
    if (PRE && has_rem) rem_products(p, colS, valS, lds_s32(rpS + 4 * (16 * (ntr - 1) + rows_last)), x_policy, xcS, lane);
#pragma unroll 1
    for (int g = 0; g < ntr; g += 2) {
        const int gg = g + h;
        const int rows = gg < ntr ? (gg + 1 < ntr ? 16 : rows_last) : 0;
        double acc = 0.0;
        if (has_rem) {
            const uint32_t rq = rpS + 64u * (uint32_t)min(gg, ntr - 1);
            const int b = lds_s32(rq + 4 * min(r, rows)), e = lds_s32(rq + 4 * min(r + 1, rows));
            const bool lng = e - b > kShortRow;
            const int ee = lng ? b : e;
            const int trips = (int)__reduce_max_sync(FULL, (unsigned)((ee - b + 3) >> 2));
            double s0 = 0.0, s1 = 0.0, s2 = 0.0, s3 = 0.0;
#pragma unroll 1
            for (int t = 0; t < trips; ++t) {
                const int k = b + 4 * t;
                s0 += rem_product<PRE>(p, k, ee, colS, valS, x_policy);
                s1 += rem_product<PRE>(p, k + 1, ee, colS, valS, x_policy);
                s2 += rem_product<PRE>(p, k + 2, ee, colS, valS, x_policy);
                s3 += rem_product<PRE>(p, k + 3, ee, colS, valS, x_policy);
            }
            acc = (s0 + s1) + (s2 + s3);
            uint32_t lm = __ballot_sync(FULL, lng);
#pragma unroll 1
            while (lm) {  // one long row at a time, the whole warp
                const int src = __ffs(lm) - 1;
                lm &= lm - 1;
                const int bb = __shfl_sync(FULL, b, src), e2 = __shfl_sync(FULL, e, src);
                const int t2 = (e2 - bb + 127) >> 7;
                double q0 = 0.0, q1 = 0.0, q2 = 0.0, q3 = 0.0;
#pragma unroll 1
                for (int t = 0; t < t2; ++t) {
                    const int k = bb + lane + 128 * t;
                    q0 += rem_product<PRE>(p, k, e2, colS, valS, x_policy);
                    q1 += rem_product<PRE>(p, k + 32, e2, colS, valS, x_policy);
                    q2 += rem_product<PRE>(p, k + 64, e2, colS, valS, x_policy);
                    q3 += rem_product<PRE>(p, k + 96, e2, colS, valS, x_policy);
                }
                double sq = (q0 + q1) + (q2 + q3);
                sq += __shfl_xor_sync(FULL, sq, 16);
                sq += __shfl_xor_sync(FULL, sq, 8);
                sq += __shfl_xor_sync(FULL, sq, 4);
                sq += __shfl_xor_sync(FULL, sq, 2);
                sq += __shfl_xor_sync(FULL, sq, 1);
                if (lane == src) acc += sq;
            }
        }
        const int64_t row = 16 * ((int64_t)it.I + gg) + r;
        if (gg < ntr && row < p.m) store_y<SC>(p, row, acc);
    }
    return PRE && has_rem;
}

// ADPT's COO run (blob_parts): the item's COO tiles and HYB COO parts as one
// row-sorted list, summed two lanes per row like the remainder's short rows
// (lane (r, h) takes entries b + h, b + h + 2, ...; the halves meet in the
// final acc(r) + acc(r + 16)), each value times x from the staged segment of
// its tile (x slot = tile index * 16 + column).  Replaces the per-tile COO
// routines: 1..11-entry tiles left most of a half-warp idle.
// A masked step multiplies 0.0 by x slot 0 (a staged x entry: finite).
__device__ __forceinline__ void coo_run(uint32_t rpS, uint32_t xslS, uint32_t valS, int rows, uint32_t xs, int lane,
                                        double &acc) {
    const int r = lane & 15, h = lane >> 4;
    const int b = lds_s32(rpS + 4 * min(r, rows)), e = lds_s32(rpS + 4 * min(r + 1, rows));
    const int trips = (int)__reduce_max_sync(FULL, (unsigned)((e - b + 1 - h) >> 1));
#pragma unroll 1
    for (int i = 0; i < trips; i += 2) {
        const int k0 = b + h + 2 * i, k1 = k0 + 2;
        const double v0 = lds_f64_lt(k0, e, valS + 8 * k0), v1 = lds_f64_lt(k1, e, valS + 8 * k1);
        const double x0 = lds_f64(xs + 8 * lds_u8_lt(k0, e, xslS + k0)), x1 = lds_f64(xs + 8 * lds_u8_lt(k1, e, xslS + k1));
        acc = fma(v0, x0, acc);
        acc = fma(v1, x1, acc);
    }
}

// the tiles of one format group, two per step.  d: shared address of this
// half's descriptor (see k_blob_fill): x = distance from the descriptor to the
// tile's payload (CSR: to its csrRowPtr), y = aux | t*128 | nz << 11 | tm << 20 |
// invalid << 31 (tm: the pair's longest CSR row / larger ELL width / larger
// COO entry count).  N = 3: every CSR row / ELL width of the item is <= 3.
template <int F, int N = 0>
__device__ __forceinline__ void run_group(int np, uint32_t &d, uint32_t xs, int r, double &acc) {
    const int lane_h = (int)(threadIdx.x >> 4) & 1;
    // (not the N = 3 CSR / ELL paths: a masked pair's straight-line steps
    // beat the split loop there, C5 +3.5%)
    constexpr bool kSplit =
        F == F_DNS || F == F_DNSCOL || F == F_DNSROW || ((F == F_CSR || F == F_ELL) && N == 0);
#pragma unroll 1
    for (int i = 0; i < np; ++i, d += 16) {
        const uint2 e = lds_v2u32(d);
        const bool ok = (int)e.y >= 0;
        const uint32_t P = d + e.x;
        const uint32_t X = xs + (e.y & 0x780u);
        const int aux = (int)(e.y & 31u), nz = (int)(e.y >> 11) & 511;
        const int tm = (int)(e.y >> 20) & 31;
        // the last pair of an odd group: half 1 holds a masked copy of half
        // 0's tile, so both halves share that tile (split routines)
        if (kSplit && i == np - 1 && !__shfl_sync(FULL, (int)ok, 16)) {
            if (F == F_DNS) split_dns(P, X, r, lane_h, acc);
            if (F == F_CSR) split_csr(P, nz, tm, X, r, lane_h, acc);
            if (F == F_ELL) split_ell(P, aux, X, r, lane_h, acc);
            if (F == F_DNSCOL) split_dnscol(P, aux, X, r, lane_h, acc);
            if (F == F_DNSROW) split_dnsrow(P, aux, X, r, lane_h, acc);
            continue;
        }
        if (F == F_CSR && N == 3) half_csr_n<3>(P, nz, X, r, ok, acc);
        if (F == F_CSR && N == 0) half_csr_tm(P, nz, tm, X, r, ok, acc);
        if (F == F_ELL && N == 3) half_ell_n<3>(P, aux, X, r, ok, acc);
        if (F == F_ELL && N == 0) half_ell_tm(P, aux, tm, X, r, ok, acc);
        if (F == F_DNS) half_dns(P, X, r, ok, acc);
        if (F == F_DNSCOL) half_dnscol(P, aux, X, r, ok, acc);
        if (F == F_DNSROW) half_dnsrow_tree(P, aux, X, r, ok, acc);
        if (F == F_CSR2) half_csr2_n3(P, nz, X, r, ok, acc);  // merged CSR pairs (schedule.cu)
    }
}

// lane 0: the whole item (descriptors, payload, remainder) in ONE TMA bulk
// copy.  The slot is only ever read through the generic proxy (the kernels
// never store to it), so no proxy fence precedes the async-proxy write.
__device__ __forceinline__ void issue_blob(const Params &p, const WItem &it, uint32_t slot, uint32_t bar,
                                           uint64_t policy, int lane) {
    const uint32_t total = it.val_tot >> 16;
    TSP_CHECK(total <= (uint32_t)p.slot_bytes && (int64_t)it.blob16 * 16 + total <= p.blob_bytes);
    if (lane == 0 && total) {
        mbar_expect_tx(bar, total);
        bulk_g2s_hint(slot, p.blob + (size_t)it.blob16 * 16, total, bar, policy);
    }
}

// the x segment of every tile of the item (J: tile column of tile `lane`),
// issued before the blob lands.  tail: the item's WItem bit 30 (its last
// tile column reaches the ragged end of x)
template <int XT>
__device__ __forceinline__ void issue_x(const Params &p, int J, int nt, uint32_t xs, uint64_t x_policy, int lane,
                                        bool tail) {
    const uint32_t n32 = (uint32_t)p.n;
    if (p.x_vec && !tail) {  // lane l: tile 4k + (l >> 3), 16 bytes at elements 2(l & 7)
        const double *xq = p.x + 2 * (lane & 7);
        const uint32_t xs_l = xs + 16 * (lane & 7);
#pragma unroll
        for (int kk = 0; kk < XT / 4; ++kk) {
            const int t = 4 * kk + (lane >> 3);
            const uint32_t Jt = (uint32_t)__shfl_sync(FULL, J, t);
            TSP_CHECK(t >= nt || (int64_t)Jt * 16 + 16 <= p.n);
            if (t < nt) cp_async16(xs_l + 128 * t, xq + 16u * Jt, 16u, x_policy);
        }
        cp_async_commit();
    } else if (p.x_vec) {
        const uint32_t qq = lane & 7;
#pragma unroll
        for (int kk = 0; kk < XT / 4; ++kk) {
            const int t = 4 * kk + (lane >> 3);
            const uint32_t c0 = 16u * (uint32_t)__shfl_sync(FULL, J, t) + 2u * qq;
            if (t < nt) {
                if (c0 + 2 <= n32) {
                    cp_async16(xs + 128 * t + 16 * qq, p.x + c0, 16u, x_policy);
                } else {  // the tail of x: never read past x[n-1]
                    const double v0 = c0 < n32 ? ldg_hint(p.x + c0, x_policy) : 0.0;
                    sts_v2f64(xs + 128 * t + 16 * qq, make_double2(v0, 0.0));
                }
            }
        }
        cp_async_commit();
    } else {  // x not 16-byte aligned: lane l: tile 2k + h, element r
        const int h = lane >> 4, r = lane & 15;
#pragma unroll
        for (int kk = 0; kk < XT / 2; ++kk) {
            const int t = 2 * kk + h;
            const uint32_t col = 16u * (uint32_t)__shfl_sync(FULL, J, t) + (uint32_t)r;
            if (t < nt) sts_f64(xs + 8 * (16 * t + r), col < n32 ? ldg_hint(p.x + col, x_policy) : 0.0);
        }
    }
}

// steps 2-4 of an item whose blob is in `slot` and whose x segments are in
// flight into `xs`: remainder, tiles, y (or the split-row carry).  Returns
// true if the slot was written (products), so the caller fences the generic
// proxy writes before the next TMA copy into the slot.
template <bool PRE, bool SC>
__device__ __forceinline__ bool compute_item(const Params &p, const WItem &it, uint32_t slot, uint32_t xs,
                                             uint64_t x_policy, uint32_t xcS, int lane, double &carry) {
    if (it.jt_rows_pay & 0xFFu)  // row-group item (no tiles, no x segments)
        return group_item<PRE, SC>(p, it, slot, x_policy, xcS, lane);
    const int h = lane >> 4, r = lane & 15;
    const uint32_t total = it.val_tot >> 16;
    // 2. fused CSR remainder, while the x segments land
    double acc = 0.0;
    const uint32_t rp = it.rp_col & 0xFFFFu;
    const bool run = it.groups >> 31;  // the rp/col/val parts hold a COO run (ADPT), not a remainder
    bool wrote = false;
    if (total > rp && !run)
        wrote = remainder<PRE>(p, slot + rp, slot + (it.rp_col >> 16), slot + (it.val_tot & 0xFFFFu),
                  (int)((it.jt_rows_pay >> 8) & 31u), x_policy, xcS, lane, acc);
    if (p.x_vec) cp_async_wait_all();
    __syncwarp();
    if (run)
        coo_run(slot + rp, slot + (it.rp_col >> 16), slot + (it.val_tot & 0xFFFFu), (int)((it.jt_rows_pay >> 8) & 31u),
                xs, lane, acc);
    // 3. tiles: format group by format group, two tiles per step
    {
        const uint32_t g = it.groups;
        uint32_t d = slot + 8 * h;
        // items whose CSR rows / ELL widths are all <= 3 (bits 28, 29) run
        // those groups without per-pair dispatch
        if ((g >> 28) & 1u) run_group<F_CSR, 3>((int)(g & 15u), d, xs, r, acc);
        else run_group<F_CSR>((int)(g & 15u), d, xs, r, acc);
        if (g & 0xF0u) run_group<F_CSR2>((int)((g >> 4) & 15u), d, xs, r, acc);
        if ((g >> 29) & 1u) run_group<F_ELL, 3>((int)((g >> 8) & 15u), d, xs, r, acc);
        else run_group<F_ELL>((int)((g >> 8) & 15u), d, xs, r, acc);
        // HYB descriptors never occur: a HYB tile is ELL(w) + COO run (ADPT,
        // BYTES) or ELL(w) + remainder (DEFERRED, reading R17)
        TSP_CHECK(((g >> 12) & 15u) == 0);
        if (g & 0x0FFF0000u) {  // one test skips the three rarer formats
            run_group<F_DNS>((int)((g >> 16) & 15u), d, xs, r, acc);
            run_group<F_DNSROW>((int)((g >> 20) & 15u), d, xs, r, acc);
            run_group<F_DNSCOL>((int)((g >> 24) & 15u), d, xs, r, acc);
        }
    }
    acc += __shfl_xor_sync(FULL, acc, 16);
    // 4. y, once per row
    const int64_t row = 16 * (int64_t)it.I + lane;
    if (it.split < 0) {
        if (lane < 16 && row < p.m) store_y<SC>(p, row, acc);
    } else if (!((it.part_nt >> 30) & 1)) {  // a group of parts runs here, in part order
        carry += acc;
    } else {
        const double sum = carry + acc;
        carry = 0.0;
        if ((it.part_nt >> 29) & 1) {  // the row's only group
            if (lane < 16 && row < p.m) store_y<SC>(p, row, sum);
        } else {  // hub row: one partial per group, the last group sums them in order
            const int2 si = p.split_info[it.split];
            const int ngroups = (si.y + kLocalParts - 1) / kLocalParts;
            const int gidx = (it.part_nt & 0xFFFFFF) / kLocalParts;
            if (lane < 16) __stcg(p.partials + (int64_t)(si.x + gidx) * 16 + lane, sum);
            // the warp's partial stores, then lane 0's counter increment with
            // release (and acquire) semantics at gpu scope: the last group to
            // arrive sees every group's partial (no full membar.gl fences)
            __syncwarp();
            int old = 0;
            if (lane == 0) old = atom_add_acq_rel_gpu(p.counters + it.split, 1);
            old = __shfl_sync(FULL, old, 0);
            if (old == ngroups - 1) {  // half h sums groups h, h+2, ... in order, 4 loads in flight
                __syncwarp();
                double s = 0.0;
                for (int q0 = h; q0 < ngroups; q0 += 8) {
                    double v[4];
#pragma unroll
                    for (int i = 0; i < 4; ++i) {
                        const int qg = q0 + 2 * i;
                        v[i] = qg < ngroups ? __ldcg(p.partials + (int64_t)(si.x + qg) * 16 + r) : 0.0;
                    }
#pragma unroll
                    for (int i = 0; i < 4; ++i) s += v[i];
                }
                s += __shfl_xor_sync(FULL, s, 16);
                if (lane < 16 && row < p.m) store_y<SC>(p, row, s);
                if (lane == 0) p.counters[it.split] = 0;  // ready for the next run
            }
        }
    }
    return wrote;
}

// Dense-row kernel: WARPS warps per CTA, several CTAs per SM, one blob in
// flight per warp; each warp owns a contiguous, cost-balanced, row-aligned
// item chunk (schedule.cu) and its start record (chunk + first item).
template <int WARPS, int SLOT, int MINB, bool SC>
__global__ void __launch_bounds__(WarpCfg<WARPS, SLOT>::kThreads, MINB) tilespmv_fp64_warp(const Params p) {
    using Cfg = WarpCfg<WARPS, SLOT>;
    extern __shared__ __align__(128) uint8_t smem[];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint32_t xs = smem_u32(smem) + (uint32_t)warp * Cfg::kX;
    const uint32_t slot = smem_u32(smem) + WARPS * Cfg::kX + (uint32_t)warp * Cfg::kPer;
    const uint32_t bar = slot + SLOT;
    if (lane == 0) {
        mbar_init(bar, 1);
        fence_mbar_init();
    }
    __syncwarp();
    // PDL: the next SpMV in the stream may start its prologue now; it waits
    // (griddep_wait) before touching x or y, and so do we
    griddep_launch_dependents();
    const int64_t gw = (int64_t)blockIdx.x * WARPS + warp;
    TSP_SMID(gw, (int64_t)gridDim.x * WARPS);
    const WFirst *wf = p.wfirst + gw;
    const int4 wb = __ldg(reinterpret_cast<const int4 *>(wf));
    const int kbeg = wb.x, kend = wb.y;
    double carry = 0.0;  // partial row sums inside a group of parts of a split tile row
    uint32_t phase = 0;
    const uint64_t stream_policy = policy_evict_first(), x_policy = policy_evict_last();
    WItem nxt = load_witem(&wf->w, 0);
    int Jn = lane < 16 ? __ldg(wf->J + lane) : 0;
    for (int k = kbeg; k < kend; ++k) {
        const WItem it = nxt;
        const int J = Jn;
        TSP_STAMP(gw, k - kbeg, 0);
        issue_blob(p, it, slot, bar, stream_policy, lane);
        // the matrix is immutable; x and y may belong to the previous kernel
        if (k == kbeg) griddep_wait();
        // 1. x segments, issued before the blob lands (J came with the record)
        issue_x<kItemTiles>(p, J, (it.part_nt >> 24) & 31, xs, x_policy, lane, (it.groups >> 30) & 1u);
        if (k + 1 < kend) {  // the next record and its columns, in flight during this item
            nxt = load_witem(p.witems, k + 1);
            Jn = lane < 16 ? __ldg(p.jcols + (int64_t)(k + 1) * 16 + lane) : 0;
        }
        if (it.val_tot >> 16) {
            mbar_wait(bar, phase);
            phase ^= 1u;
        }
        TSP_STAMP(gw, k - kbeg, 1);
        TSP_INFO(gw, k - kbeg, k, it);
        if (compute_item<false, SC>(p, it, slot, xs, x_policy, 0u, lane, carry))
            fence_proxy_async();  // products written to the slot before the next TMA copy into it
        __syncwarp();  // slot and x scratch free for the next item
        TSP_STAMP(gw, k - kbeg, 3);
    }
}

// SM-queue kernel: one CTA per SM (WARPS warps, one blob in flight each).
// The CTA owns a contiguous, cost-balanced range of units (schedule.cu: a
// unit is one item, or the items of a group of parts of a split tile row,
// which must run in order in one warp); its warps claim units from a
// shared-memory counter, so warps that draw slow units take fewer and all
// warps of the SM finish together (with several CTAs per SM the hardware's
// oldest-first issue priority leaves the youngest CTAs as a serial tail).
// Each warp claims its next unit when it starts one, so the claim and the
// unit's bounds are in flight while the current unit runs.
// XT tiles per item (an x stage of XT segments per warp)
// XC > 0 (GATHER): an x cache of the XC most-gathered remainder columns in
// shared memory, filled at launch (schedule.cu: blob columns ~slot), and
// every remainder through the product pre-pass
template <int WARPS, int SLOT, int XT, int XC, bool SC>
__global__ void __launch_bounds__(WarpCfg<WARPS, SLOT, XT, XC>::kThreads, 1) tilespmv_fp64_sm(const Params p) {
    using Cfg = WarpCfg<WARPS, SLOT, XT, XC>;
    constexpr bool PRE = XC > 0;
    extern __shared__ __align__(128) uint8_t smem[];
    __shared__ int s_next;
    __shared__ __align__(8) uint64_t s_xc_bar;  // GATHER: the x cache is filled (every warp arrives once)
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint32_t xs = smem_u32(smem) + (uint32_t)warp * Cfg::kX;
    const uint32_t slot = smem_u32(smem) + WARPS * Cfg::kX + (uint32_t)warp * Cfg::kPer;
    const uint32_t bar = slot + SLOT;
    const uint32_t xc_bar = smem_u32(&s_xc_bar);
    const int ub = (int)__ldg(p.cta_begin + blockIdx.x), ue = (int)__ldg(p.cta_begin + blockIdx.x + 1);
    if (lane == 0) {
        mbar_init(bar, 1);
        if (XC > 0 && warp == 0) mbar_init(xc_bar, WARPS);
        fence_mbar_init();
    }
    if (threadIdx.x == 0) s_next = ub + WARPS;  // units ub .. ub+WARPS-1 are the warps' first
    __syncthreads();
    griddep_launch_dependents();
    const int64_t gw = (int64_t)blockIdx.x * WARPS + warp;
    TSP_SMID(gw, (int64_t)gridDim.x * WARPS);
    (void)gw;
    double carry = 0.0;  // partial row sums inside a group of parts of a split tile row
    uint32_t phase = 0;
    const uint64_t stream_policy = policy_evict_first(), x_policy = policy_evict_last();
    int k = -1, ke = 0, nb = -1, ne = 0;
    if (ub + warp < ue) {
        const int2 u = __ldg(p.units + ub + warp);
        k = u.x;
        ke = u.y;
    }
    int kb = k;
    WItem nxt{};
    int Jn = 0;
    if (k >= 0) {
        nxt = load_witem(p.witems, k);
        Jn = lane < 16 ? __ldg(p.jcols + (int64_t)k * 16 + lane) : 0;
    }
    bool waited = false, issued = false, xc_wait = false;
    const uint32_t xcS = smem_u32(smem) + Cfg::kXc;
    if (XC > 0 && p.xc_n > 0) {  // the first blob in flight, then the warp's share of the x cache
        if (k >= 0) issue_blob(p, nxt, slot, bar, stream_policy, lane);
        issued = true;
        griddep_wait();  // x is the previous kernel's
        waited = true;
        for (int i = threadIdx.x; i < p.xc_n; i += Cfg::kThreads) TSP_CHECK(p.xc_cols[i] >= 0 && p.xc_cols[i] < p.n);
        for (int i = threadIdx.x; i < p.xc_n; i += Cfg::kThreads) sts_f64(xcS + 8u * i, __ldg(p.x + __ldg(p.xc_cols + i)));
        __syncwarp();
        if (lane == 0) mbar_arrive(xc_bar);  // release: the warp's cache entries
        xc_wait = true;  // the whole cache is needed only once the first blob has landed
    }
    int j = 0;
    while (k >= 0) {
        const WItem it = nxt;
        const int J = Jn;
        TSP_STAMP(gw, j, 0);
        if (!issued) issue_blob(p, it, slot, bar, stream_policy, lane);
        issued = false;
        // the matrix is immutable; x and y may belong to the previous kernel
        if (!waited) {
            griddep_wait();
            waited = true;
        }
        if (k == kb) {  // a unit starts: claim the next one and fetch its bounds
            int c = 0;
            if (lane == 0) c = atomicAdd(&s_next, 1);
            c = __shfl_sync(FULL, c, 0);
            nb = -1;
            if (c < ue) {
                TSP_CHECK(c >= ub);
                const int2 u = __ldg(p.units + c);
                TSP_CHECK(u.x >= 0 && u.x < u.y && u.y <= p.num_items);
                nb = u.x;
                ne = u.y;
            }
        }
        // 1. x segments, issued before the blob lands (J came with the record)
        issue_x<XT>(p, J, (it.part_nt >> 24) & 31, xs, x_policy, lane, (it.groups >> 30) & 1u);
        const int kn = k + 1 < ke ? k + 1 : nb;
        TSP_CHECK(kn < p.num_items);
        if (kn >= 0) {  // the next record and its columns, in flight during this item
            nxt = load_witem(p.witems, kn);
            Jn = lane < 16 ? __ldg(p.jcols + (int64_t)kn * 16 + lane) : 0;
        }
        if (it.val_tot >> 16) {
            mbar_wait(bar, phase);
            phase ^= 1u;
        }
        if (XC > 0 && xc_wait) {  // acquire: every warp's cache entries
            mbar_wait(xc_bar, 0);
            xc_wait = false;
        }
        TSP_STAMP(gw, j, 1);
        TSP_INFO(gw, j, k, it);
        if (compute_item<PRE, SC>(p, it, slot, xs, x_policy, xcS, lane, carry))
            fence_proxy_async();  // products written to the slot before the next TMA copy into it
        __syncwarp();  // slot and x scratch free for the next item
        TSP_STAMP(gw, j, 3);
        ++j;
        if (k + 1 >= ke) {
            kb = nb;
            ke = ne;
        }
        k = kn;
    }
}

}  // namespace

KernelChoice kernel_choice(int kernel) {
    if (kernel == TILESPMV_KERNEL_DENSE_ROWS) {
        using Cfg = WarpCfg<4, 10752>;
        return {"tilespmv_fp64_warp<4,10752>", tilespmv_fp64_warp<4, 10752, 4, false>,
                tilespmv_fp64_warp<4, 10752, 4, true>, Cfg::kThreads, (int)Cfg::kSmem,
                10752, kItemTiles, false, 0};
    }
    if (kernel == TILESPMV_KERNEL_GATHER) {
        using Cfg = WarpCfg<32, kGatherSlot, 4, kXCache>;
        return {"tilespmv_fp64_sm<32,3136,4,2048>", tilespmv_fp64_sm<32, kGatherSlot, 4, kXCache, false>,
                tilespmv_fp64_sm<32, kGatherSlot, 4, kXCache, true>, Cfg::kThreads,
                (int)Cfg::kSmem, kGatherSlot, 4, true, kXCache};
    }
    using Cfg = WarpCfg<32, 4608>;
    return {"tilespmv_fp64_sm<32,4608>", tilespmv_fp64_sm<32, 4608, kItemTiles, 0, false>,
            tilespmv_fp64_sm<32, 4608, kItemTiles, 0, true>, Cfg::kThreads, (int)Cfg::kSmem,
            4608, kItemTiles, true, 0};
}

}  // namespace tsp

#ifdef TSP_TRACE
// development build only: point the item trace at a device buffer of
// (warps x kTraceItems x 4) uint64 (NULL disables it)
extern "C" int tilespmv_debug_set_trace(void *d_buf) {
    unsigned long long *p = reinterpret_cast<unsigned long long *>(d_buf);
    return cudaMemcpyToSymbol(tsp::g_trace, &p, sizeof(p)) == cudaSuccess ? 0 : -1;
}
#endif
