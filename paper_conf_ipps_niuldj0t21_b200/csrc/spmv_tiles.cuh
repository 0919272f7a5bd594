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
    // four entries per step (independent load chains, two FMA chains); the
    // first step is straight-line, longer rows (trips > 4) loop
    double a1 = 0.0;
    {
        const uint32_t c0 = (lds_u8(cb) >> s_even) & 15u;
        const uint32_t c1 = (lds_u8(b_odd) >> s_odd) & 15u;
        const uint32_t c2 = (lds_u8(cb + 1) >> s_even) & 15u;
        const uint32_t c3 = (lds_u8(b_odd + 1) >> s_odd) & 15u;
        const double v0 = lds_f64(V), v1 = lds_f64(V + 8), v2 = lds_f64(V + 16), v3 = lds_f64(V + 24);
        const double x0 = lds_f64(X + 8 * c0), x1 = lds_f64(X + 8 * c1);
        const double x2 = lds_f64(X + 8 * c2), x3 = lds_f64(X + 8 * c3);
        fma_if(0 < len, v0, x0, acc);
        fma_if(1 < len, v1, x1, a1);
        fma_if(2 < len, v2, x2, acc);
        fma_if(3 < len, v3, x3, a1);
    }
#pragma unroll 1
    for (int i = 4; i < trips; i += 4) {
        const uint32_t c0 = (lds_u8(cb + (i >> 1)) >> s_even) & 15u;
        const uint32_t c1 = (lds_u8(b_odd + (i >> 1)) >> s_odd) & 15u;
        const uint32_t c2 = (lds_u8(cb + (i >> 1) + 1) >> s_even) & 15u;
        const uint32_t c3 = (lds_u8(b_odd + (i >> 1) + 1) >> s_odd) & 15u;
        const double v0 = lds_f64(V + 8 * i), v1 = lds_f64(V + 8 * i + 8);
        const double v2 = lds_f64(V + 8 * i + 16), v3 = lds_f64(V + 8 * i + 24);
        const double x0 = lds_f64(X + 8 * c0), x1 = lds_f64(X + 8 * c1);
        const double x2 = lds_f64(X + 8 * c2), x3 = lds_f64(X + 8 * c3);
        fma_if(i < len, v0, x0, acc);
        fma_if(i + 1 < len, v1, x1, a1);
        fma_if(i + 2 < len, v2, x2, acc);
        fma_if(i + 3 < len, v3, x3, a1);
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
        fma_if(k < wq && (k == 0 || c != 0), v, xv, acc);
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
        fma_if(q < nq, v, xv, acc);
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
        fma_if(j < nq && (int)(b >> 4) == r, v, xv, acc);
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
        fma_if(k < wq, v, xv, acc);
    }
    half_coo(P + 128 * w, ei + 8 * w, kc, X, r, ok, acc);
}

// dispatch one descriptor-list entry pair (see k_dsc_write): half h runs entry 2q + h
__device__ __forceinline__ void run_pair(uint2 e, uint32_t pay, uint32_t xs, int r, double &acc) {
    const int f = (int)(e.x >> 29);  // same for both halves by construction
    const bool ok = (int)e.y >= 0;
    const uint32_t P = pay + (e.x & 0x3FFFu);
    const uint32_t X = xs + ((e.x >> 14) & 0x7FFu);
    switch (f) {
    case F_CSR: half_csr(P, (int)(e.y >> 8) & 511, X, r, ok, acc); break;
    case F_ELL: half_ell(P, (int)(e.y & 31u), X, r, ok, acc); break;
    case F_DNS: half_dns(P, X, r, ok, acc); break;
    case F_DNSCOL: half_dnscol(P, (int)(e.y & 31u), X, r, ok, acc); break;
    case F_DNSROW: half_dnsrow(P, (int)(e.y & 31u), X, r, ok, acc); break;
    case F_COO: {
        const int nz = (int)(e.y >> 8) & 511;
        half_coo(P, P + 8 * nz, nz, X, r, ok, acc);
        break;
    }
    case F_HYB: half_hyb(P, (int)(e.y & 31u), (int)(e.y >> 8) & 511, X, r, ok, acc); break;
    default: break;
    }
}

}  // namespace tsp
