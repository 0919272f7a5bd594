// spmv_tiles.cuh -- the per-format tile routines of the tiled SpMV
// (§III.C) in their B200 form: one tile per half-warp,
// one lane per tile row, shared-memory operands addressed with 32-bit shared
// addresses.  Used by the warp kernel (spmv_warp.cu).
#pragma once

#include "spmv_common.cuh"

namespace tsp {

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
__device__ __forceinline__ double2 lds_v2f64(uint32_t a) {  // a 16-byte aligned
    double2 v;
    asm volatile("ld.shared.v2.f64 {%0, %1}, [%2];" : "=d"(v.x), "=d"(v.y) : "r"(a));
    return v;
}
__device__ __forceinline__ uint32_t lds_u32(uint32_t a) {
    uint32_t v;
    asm("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a));
    return v;
}
// v = (i < len) ? [a] : 0.0 -- a predicated load instead of a masked FMA:
// 0.0 * x adds nothing to the row sum because x is finite (reading R19)
__device__ __forceinline__ double lds_f64_lt(int i, int len, uint32_t a) {
    double v;
    asm("{\n\t.reg .pred q;\n\tsetp.lt.s32 q, %1, %2;\n\tmov.b64 %0, 0;\n\t@q ld.shared.f64 %0, [%3];\n\t}"
        : "=d"(v)
        : "r"(i), "r"(len), "r"(a));
    return v;
}
// u8 at a if i < len, else 0
__device__ __forceinline__ uint32_t lds_u8_lt(int i, int len, uint32_t a) {
    uint32_t v;
    asm("{\n\t.reg .pred q;\n\tsetp.lt.s32 q, %1, %2;\n\tmov.b32 %0, 0;\n\t@q ld.shared.u8 %0, [%3];\n\t}"
        : "=r"(v)
        : "r"(i), "r"(len), "r"(a));
    return v;
}
// a remainder entry k (column, value) if k < e, else (cdef, 0.0): cdef is a
// column the item itself references (so x[cdef] is a valid, finite x entry
// on any rank that runs the item) and 0.0 * x[cdef] adds an exact zero
__device__ __forceinline__ void lds_entry_or(int k, int e, uint32_t ca, uint32_t va, int cdef, int &c, double &v) {
    asm("{\n\t.reg .pred q;\n\tsetp.lt.s32 q, %2, %3;\n\tmov.b32 %0, %6;\n\tmov.b64 %1, 0;\n\t"
        "@q ld.shared.s32 %0, [%4];\n\t@q ld.shared.f64 %1, [%5];\n\t}"
        : "=r"(c), "=d"(v)
        : "r"(k), "r"(e), "r"(ca), "r"(va), "r"(cdef));
}
// a remainder entry k (column, value) if k < e, else (0, 0.0)
__device__ __forceinline__ void lds_entry_lt(int k, int e, uint32_t ca, uint32_t va, int &c, double &v) {
    asm("{\n\t.reg .pred q;\n\tsetp.lt.s32 q, %2, %3;\n\tmov.b32 %0, 0;\n\tmov.b64 %1, 0;\n\t"
        "@q ld.shared.s32 %0, [%4];\n\t@q ld.shared.f64 %1, [%5];\n\t}"
        : "=r"(c), "=d"(v)
        : "r"(k), "r"(e), "r"(ca), "r"(va));
}
// shared address of x[col] in a tile's 128-byte aligned x segment X, from a
// column nibble already shifted to bits 3..6 (w's other bits are masked off)
__device__ __forceinline__ uint32_t xaddr(uint32_t w8, uint32_t X) {
    uint32_t a;  // one LOP3: (w8 & 0x78) | X
    asm("lop3.b32 %0, %1, 0x78, %2, 0xEA;" : "=r"(a) : "r"(w8), "r"(X));
    return a;
}
__device__ __forceinline__ uint32_t funnel_r(uint32_t lo, uint32_t hi, uint32_t sh) {
    return __funnelshift_r(lo, hi, sh);
}
__device__ __forceinline__ void sts_u32(uint32_t a, uint32_t v) {
    asm volatile("st.shared.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
__device__ __forceinline__ void sts_f64(uint32_t a, double v) {
    asm volatile("st.shared.f64 [%0], %1;" ::"r"(a), "d"(v) : "memory");
}

// --------------------------------------------- half-warp tile routines -----
// Lane r of a half owns row r of its tile.  X: shared address of the tile's
// 16 x values (128-byte aligned); ok: the half has a tile (else it runs the
// other half's tile with its FMAs masked).  Loads past a tile's end stay
// inside the CTA's shared memory and are masked out of the sum; x addresses
// always stay inside the tile's x segment.

// Lane-rotated CSR rows: lane r starts at entry r mod 8 (mod 16) of its
// row and wraps, so 8 (16) steps cover every entry once and steps past the
// row's end are predicated off.  Rows of equal length laid end to end would
// otherwise put the lanes' values 8*len bytes apart, on the same
// shared-memory banks (4-way conflicts for rows of 8, 16-way for 16).
// u: the 8 column nibbles from entry beg on.
__device__ __forceinline__ void csr_rot8(uint32_t V, uint32_t u, uint32_t X, int r, int len, double &acc) {
#pragma unroll
    for (int j = 0; j < 8; ++j) {
        const int jj = (j + r) & 7;
        const double v = lds_f64_lt(jj, len, V + 8 * jj);
        const double xv = lds_f64(xaddr((u >> (4 * jj)) << 3, X));
        acc = fma(v, xv, acc);
    }
}
__device__ __forceinline__ void csr_rot16(uint32_t RP, int beg, uint32_t V, uint32_t u, uint32_t X, int r, int len,
                                          double &acc) {
    const uint32_t wb = RP + 16 + 4 * ((beg + 8) >> 3);
    const uint64_t u2 = (uint64_t)u | ((uint64_t)funnel_r(lds_u32(wb), lds_u32(wb + 4), 4u * (beg + 8)) << 32);
#pragma unroll 4
    for (int j = 0; j < 16; ++j) {
        const int jj = (j + r) & 15;
        const double v = lds_f64_lt(jj, len, V + 8 * jj);
        const double xv = lds_f64(xaddr((uint32_t)(u2 >> (4 * jj)) << 3, X));
        acc = fma(v, xv, acc);
    }
}

// Dns: 256 values column-major; x[c], x[c+1] arrive as one
// 16-byte broadcast load
__device__ __forceinline__ void half_dns(uint32_t P, uint32_t X, int r, bool ok, double &acc) {
    const uint32_t V = P + 8 * r;
    double a0 = 0.0, a1 = 0.0;
#pragma unroll
    for (int c = 0; c < 16; c += 2) {
        const double2 xc = lds_v2f64(X + 8 * c);
        a0 = fma(lds_f64(V + 128 * c), xc.x, a0);
        a1 = fma(lds_f64(V + 128 * c + 128), xc.y, a1);
    }
    if (ok) acc += a0 + a1;
}

// DnsCol: full column q holds value q*16 + r, column id colid[q]
__device__ __forceinline__ void half_dnscol(uint32_t P, int nc, uint32_t X, int r, bool ok, double &acc) {
    const int nq = ok ? nc : 0;
    const int trips = (int)__reduce_max_sync(FULL, (unsigned)nq);
    const uint32_t cid = P + 128 * nc;
    for (int q = 0; q < trips; ++q) {
        const double v = lds_f64_lt(q, nq, P + 8 * (16 * q + r));
        const double xv = lds_f64(X + 8 * (lds_u8(cid + q) & 15u));
        acc = fma(v, xv, acc);
    }
}

// DnsRow, the paper's mapping: lane c of the half multiplies value
// q*16 + c of every full row q by x[c] (one coalesced 128-byte row per q),
// a 16-lane xor tree sums the row, and the lane r == rowid[q] adds it.
__device__ __forceinline__ void half_dnsrow_tree(uint32_t P, int nr, uint32_t X, int r, bool ok, double &acc) {
    const uint32_t rid = P + 128 * nr;
    const int nq = ok ? nr : 0;
    const int trips = (int)__reduce_max_sync(FULL, (unsigned)nq);
    const double xc = lds_f64(X + 8 * r);
#pragma unroll 1
    for (int q = 0; q < trips; ++q) {
        double s = lds_f64_lt(q, nq, P + 8 * (16 * q + r)) * xc;
        s += __shfl_xor_sync(FULL, s, 8);
        s += __shfl_xor_sync(FULL, s, 4);
        s += __shfl_xor_sync(FULL, s, 2);
        s += __shfl_xor_sync(FULL, s, 1);
        if (q < nq && (int)lds_u8(rid + q) == r) acc += s;
    }
}

// ------------------------------- routines with the pair's extent known -----
// The schedule stores in every descriptor the longest row (CSR) or width
// (ELL) of the two tiles of its half-warp pair (bits 20-24), so the trip count
// is known without a warp vote and short tiles run straight-line code of
// exactly that many steps.  A step past a lane's own row loads the value +0.0
// (predicated load) and a column nibble that stays inside the x segment.

// CSR entries base .. base+N-1 of the lane's row: values at V, their column
// nibbles in u from bit 0
template <int N>
__device__ __forceinline__ void csr_steps(uint32_t V, uint32_t u, uint32_t X, int base, int len, double &acc) {
    double xv[N], v[N];
#pragma unroll
    for (int j = 0; j < N; ++j) {
        xv[j] = lds_f64(xaddr(j == 0 ? u << 3 : u >> (4 * j - 3), X));
        v[j] = lds_f64_lt(base + j, len, V + 8 * j);
    }
#pragma unroll
    for (int j = 0; j < N; ++j) acc = fma(v[j], xv[j], acc);
}

// CSR (Alg. 2), tm = longest row of the pair
__device__ __forceinline__ void half_csr_tm(uint32_t RP, int nz, int tm, uint32_t X, int r, bool ok, double &acc) {
    const int beg = (int)lds_u8(RP + r);
    const int end = r < 15 ? (int)lds_u8(RP + r + 1) : nz;
    const int len = ok ? end - beg : 0;
    const uint32_t V = RP + 8 * (beg - nz);
    const uint32_t wa = RP + 16 + 4 * (beg >> 3);
    const uint32_t u = funnel_r(lds_u32(wa), lds_u32(wa + 4), 4u * beg);
    if (tm == 3) {
        csr_steps<3>(V, u, X, 0, len, acc);
    } else if (tm <= 2) {
        if (tm == 2) csr_steps<2>(V, u, X, 0, len, acc);
        else csr_steps<1>(V, u, X, 0, len, acc);
    } else if (tm >= 6 && tm <= 8) {
        csr_rot8(V, u, X, r, len, acc);
    } else if (tm >= 13) {
        csr_rot16(RP, beg, V, u, X, r, len, acc);
    } else {
        csr_steps<4>(V, u, X, 0, len, acc);
#pragma unroll 1
        for (int i = 4; i < tm; i += 4) {
            const uint32_t wb = RP + 16 + 4 * ((beg + i) >> 3);
            const uint32_t ui = funnel_r(lds_u32(wb), lds_u32(wb + 4), 4u * (beg + i));
            csr_steps<4>(V + 8 * i, ui, X, i, len, acc);
        }
    }
}

// CSR of an item whose rows all hold <= N entries: N straight-line steps
template <int N>
__device__ __forceinline__ void half_csr_n(uint32_t RP, int nz, uint32_t X, int r, bool ok, double &acc) {
    const int beg = (int)lds_u8(RP + r);
    const int end = r < 15 ? (int)lds_u8(RP + r + 1) : nz;
    const int len = ok ? end - beg : 0;
    const uint32_t wa = RP + 16 + 4 * (beg >> 3);
    const uint32_t u = funnel_r(lds_u32(wa), lds_u32(wa + 4), 4u * beg);
    csr_steps<N>(RP + 8 * (beg - nz), u, X, 0, len, acc);
}

// ELL slots base .. base+N-1 of row r (column nibble bytes ci + 8k, shift sh)
// rot = 3 (even row: low nibble) or 31 (odd row: high nibble): rotating the
// nibble byte left by rot puts the row's column at bits 3..6
template <int N>
__device__ __forceinline__ void ell_steps(uint32_t V, uint32_t ci, uint32_t rot, uint32_t X, int base, int wq,
                                          double &acc) {
    double xv[N], v[N];
#pragma unroll
    for (int j = 0; j < N; ++j) {
        const uint32_t b = lds_u8(ci + 8 * j);
        xv[j] = lds_f64(xaddr(__funnelshift_l(b, b, rot), X));
        v[j] = lds_f64_lt(base + j, wq, V + 128 * j);
    }
#pragma unroll
    for (int j = 0; j < N; ++j) acc = fma(v[j], xv[j], acc);
}

// ELL (Alg. 4), tm = larger width of the pair; pads are +0.0
// at column 0 and are multiplied like entries (x finite, R19)
__device__ __forceinline__ void half_ell_tm(uint32_t P, int w, int tm, uint32_t X, int r, bool ok, double &acc) {
    const int wq = ok ? w : 0;
    const uint32_t ci = P + 128 * w + (r >> 1);
    const uint32_t rot = (r & 1) ? 31u : 3u;
    const uint32_t V = P + 8 * r;
    if (tm == 3) {
        ell_steps<3>(V, ci, rot, X, 0, wq, acc);
    } else if (tm <= 2) {
        if (tm == 2) ell_steps<2>(V, ci, rot, X, 0, wq, acc);
        else ell_steps<1>(V, ci, rot, X, 0, wq, acc);
    } else {
#pragma unroll 1
        for (int k = 0; k < tm; k += 4) ell_steps<4>(V + 128 * k, ci + 8 * k, rot, X, k, wq, acc);
    }
}

// ELL of an item whose widths are all <= N: N straight-line steps
template <int N>
__device__ __forceinline__ void half_ell_n(uint32_t P, int w, uint32_t X, int r, bool ok, double &acc) {
    ell_steps<N>(P + 8 * r, P + 128 * w + (r >> 1), (r & 1) ? 31u : 3u, X, 0, ok ? w : 0, acc);
}

// CSR2 (schedule.cu: two CSR tiles at adjacent tile columns merged, every
// merged row <= 3 entries): like CSR, but one column byte per entry (0..31)
// indexing the two x segments staged side by side from X
__device__ __forceinline__ void half_csr2_n3(uint32_t RP, int nz, uint32_t X, int r, bool ok, double &acc) {
    const int beg = (int)lds_u8(RP + r);
    const int end = r < 15 ? (int)lds_u8(RP + r + 1) : nz;
    const int len = ok ? end - beg : 0;
    const uint32_t ca = RP + 16 + beg, wa = ca & ~3u;
    const uint32_t u = funnel_r(lds_u32(wa), lds_u32(wa + 4), 8u * (ca & 3u));
    const uint32_t V = RP + 8 * (beg - nz);
    // byte j of u times 8: the entry's x offset from X (<= 248)
    const double x0 = lds_f64(X + ((u << 3) & 0xF8u)), x1 = lds_f64(X + ((u >> 5) & 0xF8u)),
                 x2 = lds_f64(X + ((u >> 13) & 0xF8u));
    const double v0 = lds_f64_lt(0, len, V), v1 = lds_f64_lt(1, len, V + 8), v2 = lds_f64_lt(2, len, V + 16);
    acc = fma(v0, x0, acc);
    acc = fma(v1, x1, acc);
    acc = fma(v2, x2, acc);
}

// ------------------------------------------ split routines (odd groups) ----
// A format group with an odd number of tiles ends in a pair whose second
// tile is a masked copy of the first.  That last tile then runs on BOTH
// halves: half h takes the tile's entries / slots / columns / full rows of
// parity h, and the halves' partial row sums meet in the final
// acc(r) + acc(r + 16) like every other pair's.  Which tiles split depends
// only on the item's content (the group's tile count), so every row's
// summation order stays content-defined.

// Dns: half h multiplies columns 8h .. 8h + 7
__device__ __forceinline__ void split_dns(uint32_t P, uint32_t X, int r, int h, double &acc) {
    const uint32_t V = P + 8 * r + 1024 * h, Xh = X + 64 * h;
    double a0 = 0.0, a1 = 0.0;
#pragma unroll
    for (int c = 0; c < 8; c += 2) {
        const double2 xc = lds_v2f64(Xh + 8 * c);
        a0 = fma(lds_f64(V + 128 * c), xc.x, a0);
        a1 = fma(lds_f64(V + 128 * c + 128), xc.y, a1);
    }
    acc += a0 + a1;
}

// CSR: half h takes entries h, h + 2, ... of row r (tm: the tile's longest row)
__device__ __forceinline__ void split_csr(uint32_t RP, int nz, int tm, uint32_t X, int r, int h, double &acc) {
    const int beg = (int)lds_u8(RP + r);
    const int end = r < 15 ? (int)lds_u8(RP + r + 1) : nz;
    const int len = end - beg;
    const uint32_t V = RP + 8 * (beg - nz);
#pragma unroll 1
    for (int j0 = h; j0 < tm; j0 += 4) {
        double v[2], xv[2];
#pragma unroll
        for (int q = 0; q < 2; ++q) {
            const int j = j0 + 2 * q, e = beg + j;
            const uint32_t b = lds_u8(RP + 16 + (min(e, 255) >> 1));
            xv[q] = lds_f64(X + 8 * ((b >> (4 * (e & 1))) & 15u));
            v[q] = lds_f64_lt(j, len, V + 8 * j);
        }
        acc = fma(v[0], xv[0], acc);
        acc = fma(v[1], xv[1], acc);
    }
}

// ELL: half h takes slots h, h + 2, ... (w: the width)
__device__ __forceinline__ void split_ell(uint32_t P, int w, uint32_t X, int r, int h, double &acc) {
    const uint32_t ci = P + 128 * w + (r >> 1), V = P + 8 * r;
    const uint32_t rot = (r & 1) ? 31u : 3u;
#pragma unroll 1
    for (int k = h; k < w; k += 2) {
        const uint32_t b = lds_u8(ci + 8 * k);
        acc = fma(lds_f64(V + 128 * k), lds_f64(xaddr(__funnelshift_l(b, b, rot), X)), acc);
    }
}

// DnsCol: half h takes full columns q = h, h + 2, ...
__device__ __forceinline__ void split_dnscol(uint32_t P, int nc, uint32_t X, int r, int h, double &acc) {
    const uint32_t cid = P + 128 * nc;
#pragma unroll 1
    for (int q = h; q < nc; q += 2)
        acc = fma(lds_f64(P + 8 * (16 * q + r)), lds_f64(X + 8 * (lds_u8(cid + q) & 15u)), acc);
}

// DnsRow (P:173's mapping): half h takes full rows q = h, h + 2, ..., lane c
// of the half multiplies value q*16 + c by x[c], a 16-lane tree sums the row
// and the lane of rowid[q] adds it
__device__ __forceinline__ void split_dnsrow(uint32_t P, int nr, uint32_t X, int r, int h, double &acc) {
    const uint32_t rid = P + 128 * nr;
    const double xc = lds_f64(X + 8 * r);
    const int trips = (nr + 1) >> 1;  // warp-uniform: both halves hold the same tile
#pragma unroll 1
    for (int t = 0; t < trips; ++t) {
        const int q = 2 * t + h;
        double s = lds_f64_lt(q, nr, P + 8 * (16 * q + r)) * xc;
        s += __shfl_xor_sync(FULL, s, 8);
        s += __shfl_xor_sync(FULL, s, 4);
        s += __shfl_xor_sync(FULL, s, 2);
        s += __shfl_xor_sync(FULL, s, 1);
        if (q < nr && (int)lds_u8(rid + q) == r) acc += s;
    }
}

}  // namespace tsp
