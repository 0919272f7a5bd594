// tiler.cu -- GPU preprocessing: canonical CSR -> two-level 16x16 tiled
// storage (§III.B), per-tile format selection
// (TileSpMV_ADPT, §III.D) and the DeferredCOO extraction (P:177,
// P:201).  Every step is a data-parallel kernel or a CUB device-wide
// primitive; the host only reads back sizes to allocate.  The result must be
// bit-identical to the independent CPU reference tiler in oracle/ (it shares
// no code with it): same tiles, order, formats, widths and payload bytes.
//
// Steps (DESIGN.md §"GPU tiler"):
//   a1 validate   rowptr monotone 0..nnz, columns in range and increasing
//   a2 discover   key (I, J) per entry; stable radix sort by key; tile heads
//   a3 census     16 row bitmasks per tile (bit c of row r = entry (r,c))
//   a4 select     format + aux from the masks (integer-exact predicates),
//                 extraction flags for DEFERRED
//   a5 size/scan  held nnz, payload bytes, kept-tile compaction, tilePtr
//   a6 pack       payload bytes (values are bit copies) + remainder CSR
#include <cub/cub.cuh>

#include <algorithm>
#include <cstdio>
#include <vector>

#include "internal.cuh"

namespace tsp {

#define TSP_CK(call)                                                   \
    do {                                                               \
        cudaError_t e_ = (call);                                       \
        if (e_ != cudaSuccess) return cuda_status(e_, #call);          \
    } while (0)

namespace {

// stream-ordered temporary (cudaMallocAsync / cudaFreeAsync on the create
// stream: no device-wide synchronisation, other streams keep running)
template <class T>
struct DevBuf {
    T *p = nullptr;
    cudaStream_t st = nullptr;
    explicit DevBuf(cudaStream_t s) : st(s) {}
    DevBuf(const DevBuf &) = delete;
    ~DevBuf() { free(); }
    void free() {
        if (p) cudaFreeAsync(p, st);
        p = nullptr;
    }
    int alloc(size_t n) {
        free();
        cudaError_t e = cudaMallocAsync(&p, std::max<size_t>(n, 1) * sizeof(T), st);
        if (e != cudaSuccess) {
            cudaGetLastError();
            p = nullptr;
            return set_error(TILESPMV_OOM, "cudaMallocAsync of a tiler temporary failed");
        }
        return 0;
    }
};

inline unsigned blocks_for(int64_t n, int threads) {
    return (unsigned)std::max<int64_t>(1, (n + threads - 1) / threads);
}

inline int bits_for(int64_t v) {  // bits needed to represent values in [0, v)
    int b = 0;
    while ((int64_t(1) << b) < v) b++;
    return std::max(b, 1);
}

// ---------------------------------------------------------------- a1 ------
__global__ void k_check_rowptr(const int32_t *__restrict__ rowptr, int64_t m, int64_t nnz,
                               int *bad) {
    int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i > m) return;
    int32_t v = rowptr[i];
    bool b = (i == 0 && v != 0) || (i == m && v != nnz) || (i < m && rowptr[i + 1] < v);
    if (b) atomicOr(bad, 1);
}

__global__ void k_expand_rows(const int32_t *__restrict__ rowptr, int64_t m,
                              int32_t *__restrict__ rowOf) {
    int64_t w = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    int lane = threadIdx.x & 31;
    if (w >= m) return;
    int32_t b = rowptr[w], e = rowptr[w + 1];
    for (int32_t k = b + lane; k < e; k += 32) rowOf[k] = (int32_t)w;
}

__global__ void k_check_cols(const int32_t *__restrict__ rowptr, const int32_t *__restrict__ col,
                             const int32_t *__restrict__ rowOf, int64_t nnz, int64_t n, int *bad) {
    int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (k >= nnz) return;
    int32_t c = col[k];
    bool b = c < 0 || c >= n;
    if (!b && k > 0 && rowptr[rowOf[k]] < k && col[k - 1] >= c) b = true;
    if (b) atomicOr(bad, 1);
}

// ---------------------------------------------------------------- a2 ------
template <class K>
__global__ void k_make_keys(const int32_t *__restrict__ rowOf, const int32_t *__restrict__ col,
                            int64_t nnz, int jbits, K *__restrict__ key, int32_t *__restrict__ idx) {
    int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (k >= nnz) return;
    key[k] = ((K)(uint32_t)(rowOf[k] >> 4) << jbits) | (K)(uint32_t)(col[k] >> 4);
    idx[k] = (int32_t)k;
}

template <class K>
__global__ void k_heads(const K *__restrict__ key, int64_t nnz, int32_t *__restrict__ head) {
    int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (p >= nnz) return;
    head[p] = (p == 0 || key[p] != key[p - 1]) ? 1 : 0;
}

// tileId[p] = inclusive_scan(head)[p] - 1 ; tileStart[tileId] = p at heads
__global__ void k_tile_ids(const int32_t *__restrict__ head, int32_t *__restrict__ tid, int64_t nnz,
                           int32_t *__restrict__ tileStart) {
    int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (p >= nnz) return;
    int32_t t = tid[p] - 1;
    tid[p] = t;
    if (head[p]) tileStart[t] = (int32_t)p;
}

// ---------------------------------------------------------------- a3 ------
__global__ void k_masks(const int32_t *__restrict__ idx, const int32_t *__restrict__ tid,
                        const int32_t *__restrict__ rowOf, const int32_t *__restrict__ col,
                        int64_t nnz, uint32_t *__restrict__ mask32) {
    int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (p >= nnz) return;
    int32_t k = idx[p];
    int r = rowOf[k] & 15, c = col[k] & 15;
    atomicOr(&mask32[(int64_t)tid[p] * 8 + (r >> 1)], 1u << (c + 16 * (r & 1)));
}

__device__ __forceinline__ uint32_t row_mask(const uint32_t *m8, int r) {
    return (m8[r >> 1] >> (16 * (r & 1))) & 0xFFFFu;
}

// ---------------------------------------------------------------- a4 ------
// Stats layout: [0,7) selected tiles, [7,14) selected nnz, [14,21) kept
// tiles, [21,28) kept nnz (per format).
__global__ void k_select(const uint32_t *__restrict__ mask32, int64_t numtile, int mode,
                         uint8_t *__restrict__ fmt0, uint8_t *__restrict__ aux0,
                         uint8_t *__restrict__ sfmt, int32_t *__restrict__ held,
                         int64_t *__restrict__ size16, int32_t *__restrict__ keep,
                         unsigned long long *stats) {
    __shared__ unsigned long long s_stats[28];
    if (threadIdx.x < 28) s_stats[threadIdx.x] = 0;
    __syncthreads();
    int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (t < numtile) {
        uint32_t m8[8];
#pragma unroll
        for (int q = 0; q < 8; ++q) m8[q] = mask32[t * 8 + q];
        int n = 0, S2 = 0, maxl = 0, minl = 16, nfull = 0;
        bool rows_full = true, cols_same = true;
        uint32_t mk0 = row_mask(m8, 0);
#pragma unroll
        for (int r = 0; r < 16; ++r) {
            uint32_t mk = row_mask(m8, r);
            int L = __popc(mk);
            n += L;
            S2 += L * L;
            maxl = max(maxl, L);
            minl = min(minl, L);
            rows_full &= (L == 0 || L == 16);
            nfull += (L == 16);
            cols_same &= (mk == mk0);
        }
        // TileSpMV_ADPT rules.  With mean = n/16 and population
        // variance over the 16 rows, CV^2 = (16*S2 - n^2) / n^2, so
        //   CV <= te=0.2  <=>  400*S2 <= 26*n^2 ;  CV > th=1.0  <=>  8*S2 > n^2.
        int f, a = 0;
        if (mode == TILESPMV_MODE_BYTES) {
            // optional B200 byte-cost rule (not the paper's):
            // the eligible format with the smallest 16-rounded payload (§4
            // sizes), ties to the lower format code
            auto r16 = [](int v) { return (v + 15) & ~15; };
            int best = r16(8 * n + 16 + (n + 1) / 2);
            f = F_CSR;
            auto take = [&](int ff, int sz, int aa, bool ok) {
                if (ok && r16(sz) < best) {
                    best = r16(sz);
                    f = ff;
                    a = aa;
                }
            };
            take(F_COO, 9 * n, 0, true);
            take(F_ELL, 136 * maxl, maxl, minl >= 1);  // every row non-empty (R26)
            take(F_HYB, 136 * minl + 9 * (n - 16 * minl), minl, true);
            take(F_DNS, 2048, 0, true);
            take(F_DNSROW, 129 * nfull, nfull, rows_full);
            take(F_DNSCOL, 129 * __popc(mk0), __popc(mk0), cols_same);
        }
        else if (mode == TILESPMV_MODE_FORCE_CSR) f = F_CSR;
        else if (n < 12) f = F_COO;
        else if (n >= 128) f = F_DNS;
        else if (rows_full) { f = F_DNSROW; a = nfull; }
        else if (cols_same) { f = F_DNSCOL; a = __popc(mk0); }
        else if (400 * S2 <= 26 * n * n) { f = F_ELL; a = maxl; }
        else if (8 * S2 > n * n) { f = F_HYB; a = minl; }  // argmin of the P:105 scan
        else f = F_CSR;
        int sf = f, h = n;
        if (mode == TILESPMV_MODE_DEFERRED) {
            if (f == F_COO) h = 0;
            else if (f == F_HYB) { sf = F_ELL; h = 16 * a; }
        }
        int64_t sz;
        switch (sf) {
        case F_CSR: sz = 8 * h + 16 + (h + 1) / 2; break;
        case F_COO: sz = 9 * h; break;
        case F_ELL: sz = 136 * a; break;
        case F_HYB: sz = 136 * a + 9 * (h - 16 * a); break;
        case F_DNS: sz = 2048; break;
        default: sz = 129 * a; break;
        }
        fmt0[t] = (uint8_t)f;
        aux0[t] = (uint8_t)a;
        sfmt[t] = (uint8_t)sf;
        held[t] = h;
        keep[t] = h > 0 ? 1 : 0;
        size16[t] = h > 0 ? (sz + 15) / 16 : 0;
        atomicAdd(&s_stats[f], 1ull);
        atomicAdd(&s_stats[7 + f], (unsigned long long)n);
        if (h > 0) {
            atomicAdd(&s_stats[14 + sf], 1ull);
            atomicAdd(&s_stats[21 + sf], (unsigned long long)h);
        }
    }
    __syncthreads();
    if (threadIdx.x < 28 && s_stats[threadIdx.x]) atomicAdd(&stats[threadIdx.x], s_stats[threadIdx.x]);
}

// DEFERRED: entries of COO tiles and entries of HYB tiles beyond the first w
// of their row (the COO part) go to the remainder.
__global__ void k_extract_flags(const int32_t *__restrict__ idx, const int32_t *__restrict__ tid,
                                const int32_t *__restrict__ rowOf, const int32_t *__restrict__ col,
                                const uint32_t *__restrict__ mask32, const uint8_t *__restrict__ fmt0,
                                const uint8_t *__restrict__ aux0, int64_t nnz,
                                int32_t *__restrict__ ext) {
    int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (p >= nnz) return;
    int32_t k = idx[p];
    int64_t t = tid[p];
    int f = fmt0[t];
    int e = 0;
    if (f == F_COO) e = 1;
    else if (f == F_HYB) {
        int r = rowOf[k] & 15, c = col[k] & 15;
        uint32_t mk = (mask32[t * 8 + (r >> 1)] >> (16 * (r & 1))) & 0xFFFFu;
        e = __popc(mk & ((1u << c) - 1u)) >= aux0[t];
    }
    ext[k] = e;
}

__global__ void k_rem_rowptr(const int32_t *__restrict__ rowptr, const int32_t *__restrict__ pos,
                             int64_t m, int32_t *__restrict__ remRowPtr) {
    int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i > m) return;
    remRowPtr[i] = pos[rowptr[i]];
}

__global__ void k_rem_scatter(const int32_t *__restrict__ ext, const int32_t *__restrict__ pos,
                              const int32_t *__restrict__ col, const double *__restrict__ val,
                              int64_t nnz, int32_t *__restrict__ remCol, double *__restrict__ remVal) {
    int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (k >= nnz || !ext[k]) return;
    int32_t q = pos[k];
    remCol[q] = col[k];
    reinterpret_cast<unsigned long long *>(remVal)[q] =
        reinterpret_cast<const unsigned long long *>(val)[k];  // bit copy
}

// ---------------------------------------------------------------- a5 ------
template <class K>
__global__ void k_compact(const K *__restrict__ key, const int32_t *__restrict__ tileStart,
                          int jbits, int64_t numtile, const int32_t *__restrict__ keep,
                          const int32_t *__restrict__ newId, const uint8_t *__restrict__ sfmt,
                          const uint8_t *__restrict__ aux0, const int32_t *__restrict__ nnzOff,
                          const int64_t *__restrict__ off16, int32_t *__restrict__ tileColIdx,
                          uint8_t *__restrict__ tileFmt, uint8_t *__restrict__ tileAux,
                          int32_t *__restrict__ tileNnz, uint32_t *__restrict__ tileOff,
                          int32_t *__restrict__ rowCount) {
    int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (t >= numtile || !keep[t]) return;
    K kk = key[tileStart[t]];
    int32_t q = newId[t];
    tileColIdx[q] = (int32_t)(kk & (((K)1 << jbits) - 1));
    tileFmt[q] = sfmt[t];
    tileAux[q] = aux0[t];
    tileNnz[q] = nnzOff[t];
    tileOff[q] = (uint32_t)off16[t];
    atomicAdd(&rowCount[(int64_t)(kk >> jbits)], 1);
}

// ---------------------------------------------------------------- a6 ------
__device__ __forceinline__ void or_byte(uint8_t *addr, uint32_t v) {
    uintptr_t a = reinterpret_cast<uintptr_t>(addr);
    atomicOr(reinterpret_cast<unsigned int *>(a & ~uintptr_t(3)), v << (8 * (a & 3)));
}
__device__ __forceinline__ void or_nibble(uint8_t *base, int idx, uint32_t v) {
    or_byte(base + (idx >> 1), (v & 15u) << (4 * (idx & 1)));  // low nibble first
}

__global__ void k_pack_entries(const int32_t *__restrict__ idx, const int32_t *__restrict__ tid,
                               const int32_t *__restrict__ tileStart, const int32_t *__restrict__ rowOf,
                               const int32_t *__restrict__ col, const double *__restrict__ val,
                               const uint32_t *__restrict__ mask32, const uint8_t *__restrict__ fmt0,
                               const uint8_t *__restrict__ aux0, const uint8_t *__restrict__ sfmt,
                               const int32_t *__restrict__ held, const int64_t *__restrict__ off16,
                               int64_t nnz, uint8_t *__restrict__ payload) {
    int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (p >= nnz) return;
    int64_t t = tid[p];
    int h = held[t];
    if (h == 0) return;
    int32_t k = idx[p];
    int r = rowOf[k] & 15, c = col[k] & 15;
    unsigned long long bits = reinterpret_cast<const unsigned long long *>(val)[k];
    uint8_t *P = payload + off16[t] * 16;
    const uint32_t *m8 = mask32 + t * 8;
    uint32_t mk = row_mask(m8, r);
    int rank = __popc(mk & ((1u << c) - 1u));  // position of the entry in its row
    int w = aux0[t];
    auto put = [&](int64_t byte_off) { *reinterpret_cast<unsigned long long *>(P + byte_off) = bits; };
    switch (sfmt[t]) {
    case F_CSR: {  // csrVal row-major | rowptr[16] u8 | 4-bit columns
        int q = (int)(p - tileStart[t]);
        put(8 * q);
        or_nibble(P + 8 * h + 16, q, c);
        break;
    }
    case F_COO: {  // cooVal | (row << 4 | col)
        int q = (int)(p - tileStart[t]);
        put(8 * q);
        or_byte(P + 8 * h + q, (uint32_t)((r << 4) | c));
        break;
    }
    case F_ELL: {  // column-major slots k*16 + r | 4-bit columns
        if (rank >= w) return;  // HYB COO part extracted in DEFERRED mode
        int s = rank * 16 + r;
        put(8 * s);
        or_nibble(P + 128 * w, s, c);
        break;
    }
    case F_HYB: {  // ELL(w) values | COO values | ELL columns | COO (row,col)
        int kc = h - 16 * w;
        if (rank < w) {
            int s = rank * 16 + r;
            put(8 * s);
            or_nibble(P + 128 * w + 8 * kc, s, c);
        } else {
            int q = rank - w;
            for (int rr = 0; rr < r; ++rr) q += max(0, __popc(row_mask(m8, rr)) - w);
            put(128 * w + 8 * q);
            or_byte(P + 128 * w + 8 * kc + 8 * w + q, (uint32_t)((r << 4) | c));
        }
        break;
    }
    case F_DNS:  // column-major
        put(8 * (c * 16 + r));
        break;
    case F_DNSROW: {  // values of the full rows, in row order
        uint32_t full = 0;
        for (int rr = 0; rr < 16; ++rr) full |= (row_mask(m8, rr) == 0xFFFFu ? 1u : 0u) << rr;
        int q = __popc(full & ((1u << r) - 1u));
        put(8 * (q * 16 + c));
        break;
    }
    case F_DNSCOL: {  // values of the full columns, column by column
        int q = __popc(row_mask(m8, 0) & ((1u << c) - 1u));
        put(8 * (q * 16 + r));
        break;
    }
    }
}

__global__ void k_pack_tiles(const uint32_t *__restrict__ mask32, const uint8_t *__restrict__ sfmt,
                             const uint8_t *__restrict__ aux0, const int32_t *__restrict__ held,
                             const int64_t *__restrict__ off16, int64_t numtile,
                             uint8_t *__restrict__ payload) {
    int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (t >= numtile || held[t] == 0) return;
    const uint32_t *m8 = mask32 + t * 8;
    uint8_t *P = payload + off16[t] * 16;
    int f = sfmt[t], a = aux0[t], h = held[t];
    if (f == F_CSR) {  // rowptr[r] = entries in rows < r (<= 240)
        uint8_t rp[16];
        int acc = 0;
        for (int r = 0; r < 16; ++r) { rp[r] = (uint8_t)acc; acc += __popc(row_mask(m8, r)); }
        uint8_t *dst = P + 8 * h;
        for (int r = 0; r < 16; ++r) dst[r] = rp[r];
    } else if (f == F_DNSROW) {
        int q = 0;
        for (int r = 0; r < 16; ++r)
            if (row_mask(m8, r) == 0xFFFFu) P[128 * a + q++] = (uint8_t)r;
    } else if (f == F_DNSCOL) {
        uint32_t mk0 = row_mask(m8, 0);
        int q = 0;
        for (int c = 0; c < 16; ++c)
            if ((mk0 >> c) & 1u) P[128 * a + q++] = (uint8_t)c;
    }
}

template <class F>
int cub_call(F &&f, cudaStream_t stream) {
    size_t bytes = 0;
    TSP_CK(f((void *)nullptr, bytes));
    DevBuf<uint8_t> tmp(stream);
    if (int rc = tmp.alloc(bytes)) return rc;
    TSP_CK(f((void *)tmp.p, bytes));
    return 0;
}

template <class T>
int read_scalar(const T *d, T *h, cudaStream_t stream) {
    TSP_CK(cudaMemcpyAsync(h, d, sizeof(T), cudaMemcpyDeviceToHost, stream));
    TSP_CK(cudaStreamSynchronize(stream));
    return 0;
}

template <class K>
int build_tiled_k(Matrix &M, const int32_t *d_rowptr, const int32_t *d_colidx, const double *d_val,
                  const int32_t *rowOf, int jbits, cudaStream_t st) {
    const int TB = 256;
    const int64_t nnz = M.nnz;
    const int ibits = bits_for(M.tilem);
    // ---- a2: keys, stable radix sort (tiles by (I,J); entries stay row-major)
    DevBuf<K> keyA(st), keyB(st);
    DevBuf<int32_t> idxA(st), idxB(st);
    if (int rc = keyA.alloc(nnz)) return rc;
    if (int rc = keyB.alloc(nnz)) return rc;
    if (int rc = idxA.alloc(nnz)) return rc;
    if (int rc = idxB.alloc(nnz)) return rc;
    k_make_keys<K><<<blocks_for(nnz, TB), TB, 0, st>>>(rowOf, d_colidx, nnz, jbits, keyA.p, idxA.p);
    TSP_CK(cudaGetLastError());
    {
        cub::DoubleBuffer<K> kb(keyA.p, keyB.p);
        cub::DoubleBuffer<int32_t> vb(idxA.p, idxB.p);
        int rc = cub_call([&](void *tmp, size_t &bytes) {
            return cub::DeviceRadixSort::SortPairs(tmp, bytes, kb, vb, (int)nnz, 0, ibits + jbits, st);
        }, st);
        if (rc) return rc;
        if (kb.Current() != keyA.p) std::swap(keyA.p, keyB.p);
        if (vb.Current() != idxA.p) std::swap(idxA.p, idxB.p);
    }
    keyB.free();
    idxB.free();
    const K *key = keyA.p;
    const int32_t *idx = idxA.p;
    // ---- tile heads and ids
    DevBuf<int32_t> head(st), tid(st);
    if (int rc = head.alloc(nnz)) return rc;
    if (int rc = tid.alloc(nnz)) return rc;
    k_heads<K><<<blocks_for(nnz, TB), TB, 0, st>>>(key, nnz, head.p);
    if (int rc = cub_call([&](void *tmp, size_t &bytes) {
            return cub::DeviceScan::InclusiveSum(tmp, bytes, head.p, tid.p, (int)nnz, st);
        }, st)) return rc;
    int32_t numtile32 = 0;
    if (int rc = read_scalar(tid.p + nnz - 1, &numtile32, st)) return rc;
    const int64_t numtile = numtile32;
    DevBuf<int32_t> tileStart(st);
    if (int rc = tileStart.alloc(numtile + 1)) return rc;
    k_tile_ids<<<blocks_for(nnz, TB), TB, 0, st>>>(head.p, tid.p, nnz, tileStart.p);
    TSP_CK(cudaGetLastError());
    head.free();
    // ---- a3: census masks
    DevBuf<uint32_t> mask32(st);
    if (int rc = mask32.alloc(numtile * 8)) return rc;
    TSP_CK(cudaMemsetAsync(mask32.p, 0, numtile * 8 * sizeof(uint32_t), st));
    k_masks<<<blocks_for(nnz, TB), TB, 0, st>>>(idx, tid.p, rowOf, d_colidx, nnz, mask32.p);
    TSP_CK(cudaGetLastError());
    // ---- a4: selection
    DevBuf<uint8_t> fmt0(st), aux0(st), sfmt(st);
    DevBuf<int32_t> held(st), keep(st);
    DevBuf<int64_t> size16(st);
    DevBuf<unsigned long long> stats(st);
    if (int rc = fmt0.alloc(numtile)) return rc;
    if (int rc = aux0.alloc(numtile)) return rc;
    if (int rc = sfmt.alloc(numtile)) return rc;
    if (int rc = held.alloc(numtile + 1)) return rc;
    if (int rc = keep.alloc(numtile + 1)) return rc;
    if (int rc = size16.alloc(numtile + 1)) return rc;
    if (int rc = stats.alloc(28)) return rc;
    TSP_CK(cudaMemsetAsync(stats.p, 0, 28 * sizeof(unsigned long long), st));
    TSP_CK(cudaMemsetAsync(held.p + numtile, 0, sizeof(int32_t), st));
    TSP_CK(cudaMemsetAsync(keep.p + numtile, 0, sizeof(int32_t), st));
    TSP_CK(cudaMemsetAsync(size16.p + numtile, 0, sizeof(int64_t), st));
    k_select<<<blocks_for(numtile, TB), TB, 0, st>>>(mask32.p, numtile, M.mode, fmt0.p, aux0.p,
                                                     sfmt.p, held.p, size16.p, keep.p, stats.p);
    TSP_CK(cudaGetLastError());
    // ---- remainder (DEFERRED)
    if (M.mode == TILESPMV_MODE_DEFERRED) {
        DevBuf<int32_t> ext(st), pos(st);
        if (int rc = ext.alloc(nnz + 1)) return rc;
        if (int rc = pos.alloc(nnz + 1)) return rc;
        TSP_CK(cudaMemsetAsync(ext.p + nnz, 0, sizeof(int32_t), st));
        k_extract_flags<<<blocks_for(nnz, TB), TB, 0, st>>>(idx, tid.p, rowOf, d_colidx, mask32.p,
                                                            fmt0.p, aux0.p, nnz, ext.p);
        TSP_CK(cudaGetLastError());
        if (int rc = cub_call([&](void *tmp, size_t &bytes) {
                return cub::DeviceScan::ExclusiveSum(tmp, bytes, ext.p, pos.p, (int)(nnz + 1), st);
            }, st)) return rc;
        int32_t nrem = 0;
        if (int rc = read_scalar(pos.p + nnz, &nrem, st)) return rc;
        M.rem_nnz = nrem;
        if (nrem > 0) {
            TSP_CK(cudaMallocAsync(&M.remRowPtr, (M.m + 1 + 8) * sizeof(int32_t), st));  // + bulk-copy slack
            TSP_CK(cudaMallocAsync(&M.remCol, (nrem + 4) * sizeof(int32_t), st));
            TSP_CK(cudaMallocAsync(&M.remVal, (nrem + 2) * sizeof(double), st));
            k_rem_rowptr<<<blocks_for(M.m + 1, TB), TB, 0, st>>>(d_rowptr, pos.p, M.m, M.remRowPtr);
            k_rem_scatter<<<blocks_for(nnz, TB), TB, 0, st>>>(ext.p, pos.p, d_colidx, d_val, nnz,
                                                              M.remCol, M.remVal);
            TSP_CK(cudaGetLastError());
        }
    }
    // ---- a5: kept tiles, prefix sums, tilePtr
    DevBuf<int32_t> newId(st), nnzOff(st);
    DevBuf<int64_t> off16(st);
    if (int rc = newId.alloc(numtile + 1)) return rc;
    if (int rc = nnzOff.alloc(numtile + 1)) return rc;
    if (int rc = off16.alloc(numtile + 1)) return rc;
    if (int rc = cub_call([&](void *tmp, size_t &bytes) {
            return cub::DeviceScan::ExclusiveSum(tmp, bytes, keep.p, newId.p, (int)(numtile + 1), st);
        }, st)) return rc;
    if (int rc = cub_call([&](void *tmp, size_t &bytes) {
            return cub::DeviceScan::ExclusiveSum(tmp, bytes, held.p, nnzOff.p, (int)(numtile + 1), st);
        }, st)) return rc;
    if (int rc = cub_call([&](void *tmp, size_t &bytes) {
            return cub::DeviceScan::ExclusiveSum(tmp, bytes, size16.p, off16.p, (int)(numtile + 1), st);
        }, st)) return rc;
    int32_t nkept = 0;
    int64_t total16 = 0;
    if (int rc = read_scalar(newId.p + numtile, &nkept, st)) return rc;
    if (int rc = read_scalar(off16.p + numtile, &total16, st)) return rc;
    if (total16 >= (int64_t(1) << 32)) return set_error(TILESPMV_OVERFLOW, "payload >= 64 GiB");
    M.numtile = nkept;
    M.payload_bytes = total16 * 16;
    TSP_CK(cudaMallocAsync(&M.tilePtr, (M.tilem + 1) * sizeof(int32_t), st));
    TSP_CK(cudaMallocAsync(&M.tileColIdx, std::max<int64_t>(nkept, 1) * sizeof(int32_t), st));
    TSP_CK(cudaMallocAsync(&M.tileNnz, (nkept + 1) * sizeof(int32_t), st));
    TSP_CK(cudaMallocAsync(&M.tileFmt, std::max<int64_t>(nkept, 1), st));
    TSP_CK(cudaMallocAsync(&M.tileAux, std::max<int64_t>(nkept, 1), st));
    TSP_CK(cudaMallocAsync(&M.tileOff, (nkept + 1) * sizeof(uint32_t), st));
    // +64 bytes: the SpMV kernel never reads past the end, but keep a pad
    TSP_CK(cudaMallocAsync(&M.payload, M.payload_bytes + 64, st));
    DevBuf<int32_t> rowCount(st);
    if (int rc = rowCount.alloc(M.tilem + 1)) return rc;
    TSP_CK(cudaMemsetAsync(rowCount.p, 0, (M.tilem + 1) * sizeof(int32_t), st));
    k_compact<K><<<blocks_for(numtile, TB), TB, 0, st>>>(
        key, tileStart.p, jbits, numtile, keep.p, newId.p, sfmt.p, aux0.p, nnzOff.p, off16.p,
        M.tileColIdx, M.tileFmt, M.tileAux, M.tileNnz, M.tileOff, rowCount.p);
    TSP_CK(cudaGetLastError());
    // last entries of the prefix arrays
    TSP_CK(cudaMemcpyAsync(M.tileNnz + nkept, nnzOff.p + numtile, sizeof(int32_t),
                           cudaMemcpyDeviceToDevice, st));
    {
        uint32_t t16 = (uint32_t)total16;
        TSP_CK(cudaMemcpyAsync(M.tileOff + nkept, &t16, sizeof(uint32_t), cudaMemcpyHostToDevice, st));
        TSP_CK(cudaStreamSynchronize(st));  // t16 is a stack variable
    }
    if (int rc = cub_call([&](void *tmp, size_t &bytes) {
            return cub::DeviceScan::ExclusiveSum(tmp, bytes, rowCount.p, M.tilePtr, (int)(M.tilem + 1), st);
        }, st)) return rc;
    // ---- a6: pack the payload
    TSP_CK(cudaMemsetAsync(M.payload, 0, M.payload_bytes + 64, st));
    k_pack_entries<<<blocks_for(nnz, TB), TB, 0, st>>>(idx, tid.p, tileStart.p, rowOf, d_colidx, d_val,
                                                       mask32.p, fmt0.p, aux0.p, sfmt.p, held.p,
                                                       off16.p, nnz, M.payload);
    k_pack_tiles<<<blocks_for(numtile, TB), TB, 0, st>>>(mask32.p, sfmt.p, aux0.p, held.p, off16.p,
                                                         numtile, M.payload);
    TSP_CK(cudaGetLastError());
    unsigned long long hs[28];
    TSP_CK(cudaMemcpyAsync(hs, stats.p, sizeof hs, cudaMemcpyDeviceToHost, st));
    TSP_CK(cudaStreamSynchronize(st));
    for (int f = 0; f < 7; ++f) {
        M.sel_tiles[f] = (int64_t)hs[f];
        M.sel_nnz[f] = (int64_t)hs[7 + f];
        M.kept_tiles[f] = (int64_t)hs[14 + f];
        M.kept_nnz[f] = (int64_t)hs[21 + f];
    }
    return 0;
}

}  // namespace

int build_tiled(Matrix &M, const int32_t *d_rowptr, const int32_t *d_colidx, const double *d_val,
                int validate, cudaStream_t st) {
    const int TB = 256;
    M.tilem = (M.m + kTile - 1) / kTile;
    M.tilen = (M.n + kTile - 1) / kTile;
    // a1: validation
    if (validate && M.m > 0) {
        DevBuf<int> bad(st);
        if (int rc = bad.alloc(1)) return rc;
        TSP_CK(cudaMemsetAsync(bad.p, 0, sizeof(int), st));
        k_check_rowptr<<<blocks_for(M.m + 1, TB), TB, 0, st>>>(d_rowptr, M.m, M.nnz, bad.p);
        TSP_CK(cudaGetLastError());
        int hbad = 0;
        if (int rc = read_scalar(bad.p, &hbad, st)) return rc;
        if (hbad) return set_error(TILESPMV_NOT_CANONICAL, "rowptr is not a monotone 0..nnz sequence");
    }
    if (M.nnz == 0) {  // no tiles, empty remainder
        TSP_CK(cudaMallocAsync(&M.tilePtr, (M.tilem + 1) * sizeof(int32_t), st));
        TSP_CK(cudaMemsetAsync(M.tilePtr, 0, (M.tilem + 1) * sizeof(int32_t), st));
        TSP_CK(cudaMallocAsync(&M.tileNnz, sizeof(int32_t), st));
        TSP_CK(cudaMemsetAsync(M.tileNnz, 0, sizeof(int32_t), st));
        TSP_CK(cudaMallocAsync(&M.tileOff, sizeof(uint32_t), st));
        TSP_CK(cudaMemsetAsync(M.tileOff, 0, sizeof(uint32_t), st));
        TSP_CK(cudaMallocAsync(&M.payload, 64, st));
        TSP_CK(cudaStreamSynchronize(st));
        return 0;
    }
    DevBuf<int32_t> rowOf(st);
    if (int rc = rowOf.alloc(M.nnz)) return rc;
    k_expand_rows<<<blocks_for(M.m * 32, TB), TB, 0, st>>>(d_rowptr, M.m, rowOf.p);
    TSP_CK(cudaGetLastError());
    if (validate) {
        DevBuf<int> bad(st);
        if (int rc = bad.alloc(1)) return rc;
        TSP_CK(cudaMemsetAsync(bad.p, 0, sizeof(int), st));
        k_check_cols<<<blocks_for(M.nnz, TB), TB, 0, st>>>(d_rowptr, d_colidx, rowOf.p, M.nnz, M.n, bad.p);
        TSP_CK(cudaGetLastError());
        int hbad = 0;
        if (int rc = read_scalar(bad.p, &hbad, st)) return rc;
        if (hbad) return set_error(TILESPMV_NOT_CANONICAL,
                                   "column index out of range or not strictly increasing in a row");
    }
    const int jbits = bits_for(M.tilen);
    const int ibits = bits_for(M.tilem);
    if (ibits + jbits <= 32)
        return build_tiled_k<uint32_t>(M, d_rowptr, d_colidx, d_val, rowOf.p, jbits, st);
    return build_tiled_k<unsigned long long>(M, d_rowptr, d_colidx, d_val, rowOf.p, jbits, st);
}

}  // namespace tsp
