// schedule.cu -- create-time SpMV schedule and launch dispatch.
//   * work items: byte-bounded pieces of one tile row (internal.cuh), built
//     by one thread per tile row in two passes (count, scan, write);
//   * 8-byte tile descriptors derived from the canonical level-1 arrays, and
//     the per-item execution blobs the kernels stage with one TMA copy;
//   * kernel choice (tilespmv_opts_t.kernel) and the per-CTA / per-warp
//     work ranges.
// Everything runs on the caller's stream: temporaries are stream-ordered
// (cudaMallocAsync / cudaFreeAsync), and the only host waits are
// cudaStreamSynchronize(stream) for the sizes the next allocation needs.
#include <cub/cub.cuh>

#include <algorithm>

#include "spmv_common.cuh"

namespace tsp {

#define TSP_CK(call)                                                   \
    do {                                                               \
        cudaError_t e_ = (call);                                       \
        if (e_ != cudaSuccess) return cuda_status(e_, #call);          \
    } while (0)

namespace {

// The level-1 arrays the schedule reads, and whether items gather their COO
// data into a COO run (ADPT mode, see blob_parts).
struct TileView {
    const int32_t *tilePtr;
    const uint32_t *tileOff;
    const uint8_t *tileFmt, *tileAux;
    const int32_t *tileNnz;
    const int32_t *tileColIdx;
    int run;        // ADPT / BYTES: COO data as a COO run
    int local_rem;  // DEFERRED: remainders that fit the x stage as a local run (rem_local)
    const uint8_t *payload;  // canonical level-2 payload (CSR2 merge test and re-encoding)
};

// Bytes tile g occupies in its item's blob payload, and the entries it adds
// to the item's COO run: with a run, a COO tile moves wholly into the run and
// a HYB(w) tile keeps its ELL(w) part as an ELL tile (136 w bytes, no pads:
// every row holds >= w entries) and moves its COO part into the run.
__device__ __forceinline__ void tile_cost(const TileView &T, int g, uint32_t &pay, uint32_t &run) {
    pay = (T.tileOff[g + 1] - T.tileOff[g]) * 16u;
    run = 0;
    if (!T.run) return;
    const uint8_t f = T.tileFmt[g];
    const uint32_t nz = (uint32_t)(T.tileNnz[g + 1] - T.tileNnz[g]);
    if (f == F_COO) {
        pay = 0;
        run = nz;
    } else if (f == F_HYB) {
        const uint32_t w = T.tileAux[g];
        pay = up16(136u * w);
        run = nz - 16u * w;
    }
}

// Greedy split of tile row I into items whose staged bytes (blob_parts)
// never exceed the kernel's slot size (budget): tiles first (at most
// max_tiles), then the tile row's remainder entries.  Depends only on the
// tile row's own content.
template <bool WRITE>
__device__ int items_for_row(int64_t I, const TileView &T, const int32_t *remRowPtr, int64_t m, int budget,
                             int max_tiles, Item *out, int split, int nparts = 0, int lp = kLocalParts) {
    const int32_t *tilePtr = T.tilePtr;
    const uint32_t *tileOff = T.tileOff;
    const int tp0 = tilePtr[I], tp1 = tilePtr[I + 1];
    int k0 = 0, k1 = 0;
    if (remRowPtr) {
        k0 = remRowPtr[16 * I];
        k1 = remRowPtr[16 * I + 16 < m ? 16 * I + 16 : m];
    }
    const int64_t rows = imin64(16, m - 16 * I);
    const uint32_t rp_bytes = up16((uint32_t)(rows + 1) * 4u);
    int t = tp0, k = k0, cnt = 0;
    do {
        const int tb = t;
        uint32_t used = 0, pays = 0, rune = 0;
        while (t < tp1 && t - tb < max_tiles) {
            uint32_t pt, rt;
            tile_cost(T, t, pt, rt);
            // blob: descriptor list (<= ntiles + 7 pads) + J array + COO run (blob_parts)
            const uint32_t dsc = up16(8u * (uint32_t)(t - tb + 1 + 7)) + up16(4u * (uint32_t)(t - tb + 1));
            const uint32_t u = pays + pt + run_bytes(rune + rt) + dsc;
            if (u > (uint32_t)budget) break;
            used = u;
            pays += pt;
            rune += rt;
            t++;
        }
        if (t == tb && t < tp1) {  // unreachable: one tile (<= 2176 B) always fits
            tile_cost(T, t, pays, rune);
            used = pays + run_bytes(rune) + 80u;
            t++;
        }
        int kb = k, ke = k;
        if (t == tp1 && k < k1) {
            const int64_t avail = (int64_t)budget - used - rp_bytes - 64;  // 2 x 32 B skew slack
            const int64_t e = imin64(avail > 0 ? avail / 12 : 0, k1 - k);
            if (e > 0) {
                ke = k + (int)e;
                k = ke;
            }
        }
        if (WRITE) {
            Item it;
            it.I = (int32_t)I;
            it.tb = tb;
            it.kb = kb;
            it.ke = ke;
            it.offb = tileOff[tb];
            it.offe = tileOff[t];
            it.pay_bytes = pays;
            it.run_e = rune;
            it.xseg = (uint32_t)(t - tb);
            it.split = split;
            const bool local = split >= 0 && nparts <= lp;
            const bool last = split >= 0 && (cnt == nparts - 1 || cnt % lp == lp - 1);
            it.part_nt = (split >= 0 ? cnt : 0) | ((t - tb) << 24) | ((int)local << 29) | ((int)last << 30);
            it.dbeg = 0;
            it.ndsc = 0;
            it.blob16 = 0;
            it.blob_len = 0;
            it.ntr = 0;
            out[cnt] = it;
        }
        cnt++;
    } while (t < tp1 || k < k1);
    return cnt;
}

__global__ void k_items_count(TileView T, const int32_t *remRowPtr, int64_t m, int budget, int max_tiles, int64_t tilem,
                              int32_t *nitems, int32_t *nsplit, int32_t *parts) {
    int64_t I = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (I >= tilem) return;
    const int c = items_for_row<false>(I, T, remRowPtr, m, budget, max_tiles, nullptr, -1);
    nitems[I] = c;
    nsplit[I] = c > 1 ? 1 : 0;
    parts[I] = c > 1 ? c : 0;
}

// a tile row that may join a row-group item: no stored tile, one item
__device__ __forceinline__ bool groupable(int64_t I, const int32_t *tilePtr, const int32_t *nitems) {
    return tilePtr[I + 1] == tilePtr[I] && nitems[I] == 1;
}

// The items of window w (kGroupWindow tile rows) in tile-row order: ordinary
// tile rows give their items_for_row items; runs of groupable tile rows are
// packed greedily into row-group items (<= kGroupTileRows tile rows, blob
// within budget).  group = false: no row-group items (kernels without them).
template <bool WRITE>
__device__ int window_items(int64_t w, const TileView &T, const int32_t *remRowPtr, int64_t m, int budget,
                            int max_tiles, int64_t tilem, bool group, const int32_t *nitems, const int32_t *splitId,
                            Item *out, int lp) {
    const int32_t *tilePtr = T.tilePtr;
    const uint32_t *tileOff = T.tileOff;
    const int64_t I0 = w * kGroupWindow, I1 = imin64(I0 + kGroupWindow, tilem);
    int cnt = 0;
    int64_t I = I0;
    while (I < I1) {
        if (!group || !groupable(I, tilePtr, nitems)) {
            if (WRITE) items_for_row<true>(I, T, remRowPtr, m, budget, max_tiles, out + cnt,
                                           nitems[I] > 1 ? splitId[I] : -1, nitems[I], lp);
            cnt += nitems[I];
            ++I;
            continue;
        }
        int64_t J = I;
        int R = 0;
        while (J < I1 && R < kGroupTileRows && groupable(J, tilePtr, nitems)) {
            const int64_t rows = imin64(16 * (int64_t)(R + 1), m - 16 * I);
            const uint32_t e = remRowPtr ? (uint32_t)(remRowPtr[imin64(16 * (J + 1), m)] - remRowPtr[16 * I]) : 0u;
            const uint32_t bytes = e ? up16(4u * (uint32_t)(rows + 1)) + up16(4u * e) + up16(8u * e) : 0u;
            if (R > 0 && bytes + 64u > (uint32_t)budget) break;
            ++R;
            ++J;
        }
        if (WRITE) {
            Item it;
            it.I = (int32_t)I;
            it.tb = tilePtr[I];
            it.kb = remRowPtr ? remRowPtr[16 * I] : 0;
            it.ke = remRowPtr ? remRowPtr[imin64(16 * J, m)] : 0;
            it.offb = it.offe = tileOff[it.tb];
            it.pay_bytes = it.run_e = it.xseg = 0;
            it.split = -1;
            it.part_nt = 0;
            it.dbeg = it.ndsc = 0;
            it.blob16 = it.blob_len = 0;
            it.ntr = R;
            out[cnt] = it;
        }
        ++cnt;
        I = J;
    }
    return cnt;
}

__global__ void k_window_count(TileView T, const int32_t *remRowPtr, int64_t m, int budget, int max_tiles,
                               int64_t tilem, int group, const int32_t *nitems, int64_t nwin, int32_t *wcount) {
    const int64_t w = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (w >= nwin) return;
    wcount[w] = window_items<false>(w, T, remRowPtr, m, budget, max_tiles, tilem, group != 0, nitems, nullptr, nullptr,
                                    kLocalParts);
}

__global__ void k_window_write(TileView T, const int32_t *remRowPtr, int64_t m, int budget, int max_tiles, int64_t tilem,
                               int group,
                               const int32_t *nitems, int64_t nwin, const int32_t *wbase, const int32_t *splitId,
                               const int32_t *partBase, Item *items, int2 *split_info, int lp) {
    const int64_t w = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (w >= nwin) return;
    window_items<true>(w, T, remRowPtr, m, budget, max_tiles, tilem, group != 0, nitems, splitId, items + wbase[w], lp);
    const int64_t I1 = imin64((w + 1) * kGroupWindow, tilem);
    for (int64_t I = w * kGroupWindow; I < I1; ++I)
        if (nitems[I] > 1) split_info[splitId[I]] = make_int2(partBase[I], nitems[I]);
}

// Per-item tile-descriptor list: the item's tiles grouped by format (format
// order, tile order inside a group), every odd group padded with a copy of
// its last entry marked invalid, so a half-warp pair never mixes formats.
// Entry: x = payload byte offset inside the item | (t * 128) << 14 | fmt << 29
//        y = aux | nnz << 8 | invalid << 31          (t: tile index in the item;
// t * 128 is the byte offset of the tile's x segment in the warp's x scratch)
// With a COO run (tile_cost): COO tiles get no descriptor and a HYB(w)
// tile's descriptor is an ELL(w) one (none if w = 0).
__device__ __forceinline__ int dsc_format(const TileView &T, int g) {
    const int f = T.tileFmt[g];
    if (!T.run) return f;
    if (f == F_COO) return -1;
    if (f == F_HYB) return T.tileAux[g] ? F_ELL : -1;
    return f;
}

// CSR2 (execution copy only; the canonical tiling is untouched): two CSR
// tiles of an item at adjacent tile columns J, J + 1 whose merged rows hold
// at most 3 entries each -- the dy = +-1 half-bands of a 27-point stencil,
// where tile J holds rows 0..8 and tile J + 1 rows 7..15 -- run as ONE tile
// whose 5-bit columns index both x segments (staged side by side), so a lane
// does its row's 3 entries once instead of two half-empty tiles.  Encoding:
// val[nz] row-major (row r: tile J's entries, then tile J + 1's), rowptr[16]
// u8, one column byte per entry (0..31); never larger than the two tiles'
// canonical payloads (checked), written where they would be in the blob.
// Descriptor format code F_CSR2 = 1 (COO tiles never get descriptors:
// DEFERRED extracts them, ADPT/BYTES move them into the run).
__device__ __forceinline__ bool csr2_mergeable(const TileView &T, int g) {
    if (T.tileFmt[g] != F_CSR || T.tileFmt[g + 1] != F_CSR) return false;
    if (T.tileColIdx[g + 1] != T.tileColIdx[g] + 1) return false;
    const int na = T.tileNnz[g + 1] - T.tileNnz[g], nb = T.tileNnz[g + 2] - T.tileNnz[g + 1];
    if (up16(9u * (uint32_t)(na + nb) + 16u) > (T.tileOff[g + 2] - T.tileOff[g]) * 16u) return false;
    const uint8_t *ra = T.payload + (size_t)T.tileOff[g] * 16 + 8 * na;
    const uint8_t *rb = T.payload + (size_t)T.tileOff[g + 1] * 16 + 8 * nb;
    for (int r = 0; r < 16; ++r) {
        const int la = (r < 15 ? ra[r + 1] : na) - ra[r], lb = (r < 15 ? rb[r + 1] : nb) - rb[r];
        if (la + lb > 3) return false;
    }
    return true;
}

// the CSR2 encoding of tiles g, g + 1 at o (span: their canonical bytes,
// zeroed first); lane r < 16 writes row r
__device__ __forceinline__ void write_csr2(const TileView &T, int g, uint8_t *o, int lane) {
    const int na = T.tileNnz[g + 1] - T.tileNnz[g], nb = T.tileNnz[g + 2] - T.tileNnz[g + 1], nz = na + nb;
    const uint8_t *sa = T.payload + (size_t)T.tileOff[g] * 16, *sb = T.payload + (size_t)T.tileOff[g + 1] * 16;
    const uint8_t *ra = sa + 8 * na, *rb = sb + 8 * nb;
    const uint32_t span = (T.tileOff[g + 2] - T.tileOff[g]) * 16u;
    __syncwarp();
    for (uint32_t i = lane; i < span; i += 32) o[i] = 0;
    __syncwarp();
    if (lane < 16) {
        const int r = lane;
        const int ba = ra[r], ea = r < 15 ? ra[r + 1] : na, bb = rb[r], eb = r < 15 ? rb[r + 1] : nb;
        const int mp = ba + bb;  // merged row start
        o[8 * nz + r] = (uint8_t)mp;
        double *ov = reinterpret_cast<double *>(o);
        uint8_t *oc = o + 8 * nz + 16;
        int q = mp;
        for (int k = ba; k < ea; ++k, ++q) {
            ov[q] = reinterpret_cast<const double *>(sa)[k];
            oc[q] = (uint8_t)((sa[8 * na + 16 + (k >> 1)] >> (4 * (k & 1))) & 15);
        }
        for (int k = bb; k < eb; ++k, ++q) {
            ov[q] = reinterpret_cast<const double *>(sb)[k];
            oc[q] = (uint8_t)(16 + ((sb[8 * nb + 16 + (k >> 1)] >> (4 * (k & 1))) & 15));
        }
    }
    __syncwarp();
}

// execution format of every tile of the item (pairs merged greedily left to
// right): dsc_format, F_CSR2 for a merged pair's first tile, -1 for no descriptor
__device__ __forceinline__ void exec_formats(const Item &it, const TileView &T, int8_t *ef) {
    const int nt = item_nt(it);
    for (int t = 0; t < nt; ++t) {
        if (t + 1 < nt && csr2_mergeable(T, it.tb + t)) {
            ef[t] = F_CSR2;
            ef[t + 1] = -1;
            ++t;
        } else {
            ef[t] = (int8_t)dsc_format(T, it.tb + t);
        }
    }
}

__global__ void k_dsc_count(Item *items, int64_t n, TileView T, int32_t *ndsc) {
    int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (k >= n) return;
    const Item it = items[k];
    const int nt = item_nt(it);
    int cnt[8] = {0, 0, 0, 0, 0, 0, 0, 0};
    int8_t ef[kItemTiles];
    exec_formats(it, T, ef);
    for (int t = 0; t < nt; ++t) {
        const int f = ef[t];
        if (f >= 0) cnt[f]++;
    }
    int total = 0;
    for (int f = 0; f < 7; ++f) total += (cnt[f] + 1) & ~1;
    ndsc[k] = total;
}

__global__ void k_dsc_write(Item *items, int64_t n, const int32_t *dbeg, const int32_t *ndsc, TileView T, uint2 *dlist) {
    int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (k >= n) return;
    Item it = items[k];
    const int nt = item_nt(it);
    int pos = dbeg[k];
    it.dbeg = pos;
    it.ndsc = ndsc[k];
    items[k] = it;
    uint32_t off[kItemTiles];  // each tile's payload offset inside the item's blob payload
    {
        uint32_t o = 0;
        for (int t = 0; t < nt; ++t) {
            uint32_t pt, rt;
            tile_cost(T, it.tb + t, pt, rt);
            off[t] = o;
            o += pt;
        }
    }
    int8_t ef[kItemTiles];
    exec_formats(it, T, ef);
    for (int f = 0; f < 7; ++f) {
        uint2 last = make_uint2(0u, 0u);
        int c = 0;
        for (int t = 0; t < nt; ++t) {
            const int g = it.tb + t;
            if (ef[t] != f) continue;
            const bool hyb_ell = T.tileFmt[g] == F_HYB;  // (run) the ELL(w) part of a HYB tile
            uint2 d;
            d.x = off[t] | ((uint32_t)t << 21) | ((uint32_t)f << 29);
            d.y = f == F_CSR2 ? (uint32_t)(T.tileNnz[g + 2] - T.tileNnz[g]) << 8
                              : (uint32_t)T.tileAux[g] |
                                    ((hyb_ell ? 16u * T.tileAux[g] : (uint32_t)(T.tileNnz[g + 1] - T.tileNnz[g])) << 8);
            dlist[pos++] = d;
            last = d;
            c++;
        }
        if (c & 1) dlist[pos++] = make_uint2(last.x, last.y | (1u << 31));
    }
}

// blob length per item; *over is set if one exceeds the kernel's slot (a
// schedule bug: the kernel would stage past its shared-memory slot)
// DEFERRED, an ordinary item with remainder rows of <= 32 entries: the tile
// columns of its remainder entries that are not among its tiles' (ascending),
// if they fit the x stage beside the tiles' segments (returns their count,
// the list in extra[]), else -1.  Such an item runs its remainder as a local
// run (blob_parts): x from the staged segments through a one-byte x slot per
// entry instead of a global gather, the two-lanes-per-row sum of the
// remainder's short rows unchanged (coo_run), so y keeps every bit.
__device__ int rem_local(const Item &it, int64_t m, const TileView &T, const int32_t *remRowPtr, const int32_t *remCol,
                         int max_tiles, int32_t *extra) {
    if (!T.local_rem || it.ntr > 0 || it.ke <= it.kb) return -1;
    const int nt = item_nt(it);
    const int rows = (int)item_rows(it, m);
    for (int r = 0; r < rows; ++r) {  // the MED path's domain: every row <= 32 entries
        int b = remRowPtr[16 * (int64_t)it.I + r], e = remRowPtr[16 * (int64_t)it.I + r + 1];
        b = b < it.kb ? it.kb : (b > it.ke ? it.ke : b);
        e = e < it.kb ? it.kb : (e > it.ke ? it.ke : e);
        if (e - b > 32) return -1;
    }
    int nx = 0;
    for (int k = it.kb; k < it.ke; ++k) {
        const int J = remCol[k] >> 4;
        bool seen = false;
        for (int t = 0; t < nt && !seen; ++t) seen = T.tileColIdx[it.tb + t] == J;
        for (int q = 0; q < nx && !seen; ++q) seen = extra[q] == J;
        if (seen) continue;
        if (nt + nx >= max_tiles) return -1;
        int q = nx++;  // insertion keeps extra[] ascending
        while (q > 0 && extra[q - 1] > J) {
            extra[q] = extra[q - 1];
            --q;
        }
        extra[q] = J;
    }
    return nx;
}

// blob length per item (deciding the DEFERRED local runs first); *over is
// set if one exceeds the kernel's slot (a schedule bug: the kernel would
// stage past its shared-memory slot)
__global__ void k_blob_len(Item *items, int64_t n, int64_t m, uint32_t slot, TileView T, const int32_t *remRowPtr,
                           const int32_t *remCol, int max_tiles, int64_t *len16, int32_t *over) {
    int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (k >= n) return;
    Item it = items[k];
    int32_t extra[kItemTiles];
    const int nx = rem_local(it, m, T, remRowPtr, remCol, max_tiles, extra);
    if (nx >= 0) {
        it.run_e = (uint32_t)(it.ke - it.kb);
        it.xseg = (uint32_t)(item_nt(it) + nx);
        items[k] = it;
    }
    const uint32_t total = blob_parts(it, m).total;
    len16[k] = total / 16;
    if (total > slot) atomicOr(over, 1);
}

// one warp per item: copy descriptors, J, payload and the rebased remainder
__global__ void k_blob_fill(Item *items, int64_t nitems, int64_t m, int64_t n, const int64_t *start16, const uint2 *dlist,
                            const int32_t *tileColIdx, TileView T, const uint8_t *payload, const int32_t *remRowPtr,
                            const int32_t *remCol, const double *remVal, uint8_t *blob, WItem *witems,
                            int32_t *jcols, const int32_t *xc_slot) {
    const int64_t k = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    if (k >= nitems) return;
    Item it = items[k];
    const BlobParts b = blob_parts(it, m);
    const int nt = item_nt(it);
    uint8_t *dst = blob + start16[k] * 16;
    if (lane == 0) {
        it.blob16 = (uint32_t)start16[k];
        it.blob_len = b.total;
        items[k] = it;
        WItem w;
        w.blob16 = it.blob16;
        w.I = (uint32_t)it.I;
        w.split = it.split;
        w.part_nt = (it.part_nt & ~(31 << 24)) | (int32_t)(it.xseg << 24);  // x segments to stage
        const uint32_t rows = (uint32_t)item_rows(it, m);
        const uint32_t last = it.ntr > 0 ? rows - 16u * (uint32_t)(it.ntr - 1) : rows;
        w.jt_rows_pay = (uint32_t)it.ntr | (last << 8) | (b.pay << 16);
        w.rp_col = b.rp | (b.col << 16);
        w.val_tot = b.val | (b.total << 16);
        int cnt[7] = {0, 0, 0, 0, 0, 0, 0};
        int8_t ef[kItemTiles];
        exec_formats(it, T, ef);
        for (int t = 0; t < nt; ++t) {
            const int f = ef[t];
            if (f >= 0) cnt[f]++;
        }
        uint32_t g = 0;
        for (int f = 0; f < 7; ++f) g |= (uint32_t)((cnt[f] + 1) >> 1) << (4 * f);
        w.groups = g | (it.run_e > 0 ? 1u << 31 : 0u);  // a COO run or a local remainder run
        witems[k] = w;
    }
    for (uint32_t o = 4 * lane; o < b.total; o += 128) *reinterpret_cast<uint32_t *>(dst + o) = 0u;  // padding
    __syncwarp();
    uint2 *dd = reinterpret_cast<uint2 *>(dst);
    // kernel-native descriptors: x = distance from the descriptor itself to
    // the tile's payload (CSR: to its csrRowPtr, after the 8*nnz value bytes),
    // y = aux | t*128 | nnz << 11 | tm << 20 | invalid << 31, where tm is the
    // larger extent of the two tiles of the half-warp pair (2j, 2j+1): CSR the
    // longest row, ELL the width, COO the entry count (ndsc is even; the
    // loop is warp-uniform)
    uint32_t csr_max = 0, ell_max = 0;
    for (int i0 = 0; i0 < it.ndsc; i0 += 32) {
        const int i = i0 + lane;
        uint2 e = make_uint2(0u, 0u);
        uint32_t tm = 0;
        if (i < it.ndsc) {
            const uint2 d = dlist[it.dbeg + i];
            const uint32_t off = d.x & 0x1FFFFFu, t = (d.x >> 21) & 0xFFu, f = d.x >> 29;
            const uint32_t nz = (d.y >> 8) & 0x1FFu;
            e.x = b.pay + off + (f == F_CSR || f == F_CSR2 ? 8u * nz : 0u) - 8u * (uint32_t)i;
            e.y = (d.y & 0x1Fu) | (t << 7) | (nz << 11) | (d.y & 0x80000000u);
            if (f == F_CSR) {
                const uint8_t *rp = payload + (size_t)T.tileOff[it.tb + t] * 16 + 8u * nz;
                for (int r = 0; r < 16; ++r) {
                    const uint32_t len = (r < 15 ? rp[r + 1] : nz) - rp[r];
                    tm = len > tm ? len : tm;
                }
            } else if (f == F_ELL) {
                tm = d.y & 0x1Fu;
            } else if (f == F_CSR2) {
                tm = 3;  // merged rows hold <= 3 entries (csr2_mergeable)
            }
        }
        const uint32_t tmo = __shfl_xor_sync(0xFFFFFFFFu, tm, 1);
        tm = tmo > tm ? tmo : tm;
        if (i < it.ndsc) dd[i] = make_uint2(e.x, e.y | (tm << 20));
        const uint32_t fi = i < it.ndsc ? dlist[it.dbeg + i].x >> 29 : 7u;
        csr_max = max(csr_max, __reduce_max_sync(0xFFFFFFFFu, fi == F_CSR ? tm : 0u));
        ell_max = max(ell_max, __reduce_max_sync(0xFFFFFFFFu, fi == F_ELL ? tm : 0u));
    }
    // the x segments: the tiles' columns, then a DEFERRED local run's others
    const bool local = !T.run && it.run_e > 0;
    int32_t extra[kItemTiles];
    const int nx = local ? rem_local(it, m, T, remRowPtr, remCol, kItemTiles, extra) : 0;
    int jseg = 0;
    if (lane < 16) {
        jseg = lane < nt ? tileColIdx[it.tb + lane] : (lane < nt + nx ? extra[lane - nt] : 0);
        jcols[k * 16 + lane] = jseg;
    }
    // item-wide extents: the kernel runs such items' CSR / ELL groups with
    // straight-line 3-step routines and no per-pair dispatch; bit 30: some
    // staged segment reaches past x[n-1]
    const bool xtail = __any_sync(0xFFFFFFFFu, lane < nt + nx && 16 * (int64_t)jseg + 16 > n);
    if (lane == 0)
        witems[k].groups |= (csr_max <= 3 ? 1u << 28 : 0u) | (ell_max <= 3 ? 1u << 29 : 0u) | (xtail ? 1u << 30 : 0u);
    if (!T.run) {  // the canonical payload bytes of the item's tiles, in one piece
        const uint4 *ps = reinterpret_cast<const uint4 *>(payload + (size_t)it.offb * 16);
        uint4 *pd = reinterpret_cast<uint4 *>(dst + b.pay);
        for (uint32_t i = lane; i < it.offe - it.offb; i += 32) pd[i] = ps[i];
        __syncwarp();
        // CSR2 pairs re-encoded over their two tiles' bytes (lane r: row r)
        int8_t ef[kItemTiles];
        exec_formats(it, T, ef);
        for (int t = 0; t < nt; ++t)
            if (ef[t] == F_CSR2) write_csr2(T, it.tb + t, dst + b.pay + (T.tileOff[it.tb + t] - it.offb) * 16u, lane);
    } else {  // tile by tile: COO tiles left out, HYB(w) tiles as their ELL(w) part, CSR2 pairs merged
        uint32_t o = b.pay;
        int8_t ef[kItemTiles];
        exec_formats(it, T, ef);
        for (int t = 0; t < nt; ++t) {
            const int g = it.tb + t;
            uint32_t pt, rt;
            tile_cost(T, g, pt, rt);
            const uint8_t *src = payload + (size_t)T.tileOff[g] * 16;
            if (ef[t] == F_CSR2) {
                uint32_t pt1, rt1;
                tile_cost(T, g + 1, pt1, rt1);
                write_csr2(T, g, dst + o, lane);
                o += pt + pt1;
                ++t;
                continue;
            }
            if (T.tileFmt[g] == F_HYB) {
                const uint32_t w = T.tileAux[g], kc = rt;
                const uint2 *vs = reinterpret_cast<const uint2 *>(src);  // ELL values, 16 w
                uint2 *vd = reinterpret_cast<uint2 *>(dst + o);
                for (uint32_t i = lane; i < 16u * w; i += 32) vd[i] = vs[i];
                for (uint32_t i = lane; i < w; i += 32)  // ELL column nibbles, 8 w bytes
                    reinterpret_cast<uint2 *>(dst + o + 128u * w)[i] =
                        reinterpret_cast<const uint2 *>(src + 128u * w + 8u * kc)[i];
            } else if (pt) {
                const uint4 *ps = reinterpret_cast<const uint4 *>(src);
                uint4 *pd = reinterpret_cast<uint4 *>(dst + o);
                for (uint32_t i = lane; i < pt / 16u; i += 32) pd[i] = ps[i];
            }
            o += pt;
        }
        if (it.run_e > 0) {
            // the COO run: lane r < 16 gathers row r's COO entries, tile by tile
            const int r = lane & 15;
            int cnt = 0;
            for (int t = 0; t < nt; ++t) {
                const int g = it.tb + t;
                const uint8_t f = T.tileFmt[g];
                if (f != F_COO && f != F_HYB) continue;
                const uint32_t w = f == F_HYB ? T.tileAux[g] : 0u;
                const uint32_t kc = (uint32_t)(T.tileNnz[g + 1] - T.tileNnz[g]) - 16u * w;
                const uint8_t *rc = payload + (size_t)T.tileOff[g] * 16 + (f == F_HYB ? 136u * w + 8u * kc : 8u * kc);
                for (uint32_t j = 0; j < kc; ++j) cnt += (rc[j] >> 4) == (uint32_t)r;
            }
            int base = cnt;  // exclusive prefix over rows 0..15
            for (int d = 1; d < 16; d <<= 1) {
                const int v = __shfl_up_sync(0xFFFFFFFFu, base, d, 16);
                if (r >= d) base += v;
            }
            base -= cnt;
            int32_t *rp = reinterpret_cast<int32_t *>(dst + b.rp);
            uint8_t *xsl = dst + b.col;
            double *vv = reinterpret_cast<double *>(dst + b.val);
            if (lane < 16) {
                rp[r] = base;
                if (r == 15) rp[16] = base + cnt;
                int pos = base;
                for (int t = 0; t < nt; ++t) {
                    const int g = it.tb + t;
                    const uint8_t f = T.tileFmt[g];
                    if (f != F_COO && f != F_HYB) continue;
                    const uint32_t w = f == F_HYB ? T.tileAux[g] : 0u;
                    const uint32_t kc = (uint32_t)(T.tileNnz[g + 1] - T.tileNnz[g]) - 16u * w;
                    const uint8_t *src = payload + (size_t)T.tileOff[g] * 16;
                    const double *cv = reinterpret_cast<const double *>(src + 128u * w);  // COO values
                    const uint8_t *rc = src + (f == F_HYB ? 136u * w + 8u * kc : 8u * kc);
                    for (uint32_t j = 0; j < kc; ++j) {
                        if ((rc[j] >> 4) != (uint32_t)r) continue;
                        vv[pos] = cv[j];
                        xsl[pos] = (uint8_t)(16 * t + (rc[j] & 15));
                        ++pos;
                    }
                }
            }
        }
    }
    if (local) {  // the remainder as a local run: rows' pointers, x slots, values
        const int rows = (int)item_rows(it, m);
        int32_t *rp = reinterpret_cast<int32_t *>(dst + b.rp);
        for (int i = lane; i <= 16; i += 32) {
            int v = remRowPtr[16 * (int64_t)it.I + min(i, rows)];
            v = v < it.kb ? it.kb : (v > it.ke ? it.ke : v);
            rp[i] = v - it.kb;
        }
        uint8_t *xsl = dst + b.col;
        unsigned long long *vd = reinterpret_cast<unsigned long long *>(dst + b.val);
        const unsigned long long *vs = reinterpret_cast<const unsigned long long *>(remVal);
        for (int i = lane; i < it.ke - it.kb; i += 32) {
            const int c = remCol[it.kb + i], J = c >> 4;
            int s = 0;
            for (int t = 0; t < nt + nx; ++t)
                if ((t < nt ? tileColIdx[it.tb + t] : extra[t - nt]) == J) s = t;
            xsl[i] = (uint8_t)(16 * s + (c & 15));
            vd[i] = vs[it.kb + i];
        }
    } else if (it.ke > it.kb) {
        const int rows = (int)item_rows(it, m);
        int32_t *rp = reinterpret_cast<int32_t *>(dst + b.rp);
        for (int i = lane; i <= rows; i += 32) {
            int v = remRowPtr[16 * (int64_t)it.I + i];
            v = v < it.kb ? it.kb : (v > it.ke ? it.ke : v);
            rp[i] = v - it.kb;
        }
        int32_t *cd = reinterpret_cast<int32_t *>(dst + b.col);
        unsigned long long *vd = reinterpret_cast<unsigned long long *>(dst + b.val);
        const unsigned long long *vs = reinterpret_cast<const unsigned long long *>(remVal);
        for (int i = lane; i < it.ke - it.kb; i += 32) {
            const int32_t c = remCol[it.kb + i];
            const int32_t sl = xc_slot ? xc_slot[c] : -1;
            cd[i] = sl >= 0 ? ~sl : c;  // a cached column: ~(its x-cache slot)
            vd[i] = vs[it.kb + i];
        }
    }
}

// item cost for the CTA chunking: bytes staged + a fixed per-item overhead
__global__ void k_item_cost(const Item *items, int64_t n, int64_t m, int64_t fixed, int64_t group_row,
                            int64_t *cost) {
    int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (k >= n) return;
    const Item it = items[k];
    cost[k] = (int64_t)blob_parts(it, m).total + 40 * (item_nt(it)) + fixed + group_row * it.ntr;
}

__global__ void k_warp_first(const int64_t *begin, const WItem *witems, const int32_t *jcols, int W, WFirst *wf) {
    const int b = blockIdx.x * blockDim.x + threadIdx.x;
    if (b >= W) return;
    WFirst f;
    f.kbeg = (int32_t)begin[b];
    f.kend = (int32_t)begin[b + 1];
    f.pad0 = f.pad1 = 0;
    if (f.kbeg < f.kend) {
        f.w = witems[f.kbeg];
        for (int i = 0; i < 16; ++i) f.J[i] = jcols[(int64_t)f.kbeg * 16 + i];
    } else {
        f.w = WItem{};
        for (int i = 0; i < 16; ++i) f.J[i] = 0;
    }
    wf[b] = f;
}

__global__ void k_cta_begin(const int64_t *incl, const Item *items, int64_t n, int G, int lp, int64_t *cta_begin) {
    const int b = blockIdx.x * blockDim.x + threadIdx.x;
    if (b > G) return;
    if (b == G) {
        cta_begin[b] = n;
        return;
    }
    const int64_t total = n ? incl[n - 1] : 0;
    const int64_t target = total * b / G;  // first item whose prefix-before >= target
    int64_t lo = 0, hi = n;
    while (lo < hi) {
        const int64_t mid = (lo + hi) / 2;
        const int64_t before = mid ? incl[mid - 1] : 0;
        if (before < target) lo = mid + 1;
        else hi = mid;
    }
    // never start inside a group of parts of a split row (a group runs in one warp)
    while (lo < n && items[lo].split >= 0 && item_part(items[lo]) % lp != 0) lo++;
    cta_begin[b] = lo;
}

// units of the SM-queue kernel: an item that is not an inner part of a group
// of parts starts a unit
__global__ void k_unit_flags(const Item *items, int64_t n, int lp, int32_t *flag) {
    const int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (k >= n) return;
    const Item it = items[k];
    flag[k] = (it.split < 0 || item_part(it) % lp == 0) ? 1 : 0;
}

__global__ void k_unit_write(const int32_t *flag, const int32_t *pos, int64_t n, int32_t *units) {
    const int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (k > n) return;
    if (k == n) {
        units[pos[n]] = (int32_t)n;
        return;
    }
    if (flag[k]) units[pos[k]] = (int32_t)k;
}

// per-CTA unit ranges balanced by the inclusive item-cost prefix: CTA b
// starts at the first unit whose cost-before reaches total * b / G
__global__ void k_cta_units(const int64_t *incl, const int32_t *units, int64_t nu, int64_t n, int G,
                            int64_t *cta_begin) {
    const int b = blockIdx.x * blockDim.x + threadIdx.x;
    if (b > G) return;
    if (b == G) {
        cta_begin[b] = nu;
        return;
    }
    const int64_t total = n ? incl[n - 1] : 0;
    const int64_t target = total * b / G;
    int64_t lo = 0, hi = nu;
    while (lo < hi) {
        const int64_t mid = (lo + hi) / 2;
        const int64_t before = units[mid] ? incl[units[mid] - 1] : 0;
        if (before < target) lo = mid + 1;
        else hi = mid;
    }
    cta_begin[b] = lo;
}

// sort key of a unit for the per-CTA ordering: its cost (the items' costs);
// unless `all`, only units of at least twice the mean unit cost keep it and
// the others get 0 (they keep their tile-row order: on stencils and banded
// matrices neighbouring tile rows share x lines in L1/L2)
__global__ void k_unit_cost(const int64_t *incl, const int32_t *ustart, int64_t nu, int64_t n, int all,
                            int64_t *ucost, int32_t *uidx) {
    const int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (u >= nu) return;
    const int32_t a = ustart[u], b = ustart[u + 1];
    const int64_t c = incl[b - 1] - (a ? incl[a - 1] : 0);
    ucost[u] = all || c * nu >= 2 * incl[n - 1] ? c : 0;
    uidx[u] = (int32_t)u;
}

// the units in claim order: [first item, end item) of unit uidx[c]
__global__ void k_unit_bounds(const int32_t *ustart, const int32_t *uidx, int64_t nu, int2 *units) {
    const int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (c >= nu) return;
    const int32_t u = uidx[c];
    units[c] = make_int2(ustart[u], ustart[u + 1]);
}

// ADPT (and BYTES) mode gathers each item's COO data into a COO run (blob_parts)
TileView tile_view(const Matrix &M) {
    return {M.tilePtr, M.tileOff, M.tileFmt, M.tileAux, M.tileNnz, M.tileColIdx,
            M.mode == TILESPMV_MODE_ADPT || M.mode == TILESPMV_MODE_BYTES ? 1 : 0,
            M.mode == TILESPMV_MODE_DEFERRED ? 1 : 0, M.payload};
}

// stream-ordered temporary device buffer
struct Tmp {
    void *p = nullptr;
    cudaStream_t st;
    explicit Tmp(cudaStream_t s) : st(s) {}
    Tmp(const Tmp &) = delete;
    ~Tmp() { if (p) cudaFreeAsync(p, st); }
    int alloc(size_t bytes) {
        if (cudaMallocAsync(&p, bytes ? bytes : 1, st) != cudaSuccess) {
            p = nullptr;
            return cuda_status(cudaGetLastError(), "cudaMallocAsync(schedule temporary)");
        }
        return 0;
    }
    template <class T> T *as() const { return static_cast<T *>(p); }
};

// a CUB device-wide call with a stream-ordered temporary
template <class F>
int scan(F &&f, cudaStream_t st) {
    size_t bytes = 0;
    TSP_CK(f(nullptr, bytes));
    Tmp tmp(st);
    if (int rc = tmp.alloc(bytes)) return rc;
    TSP_CK(f(tmp.p, bytes));
    return 0;
}

}  // namespace

int build_schedule(Matrix &M, cudaStream_t st) {
    const int TB = 256;
    const int64_t T = M.tilem;
    if (T == 0) return 0;
    auto blocks = [&](int64_t n) { return (unsigned)std::max<int64_t>(1, (n + TB - 1) / TB); };
    const int64_t NW = (T + kGroupWindow - 1) / kGroupWindow;
    const int group = 1;  // both kernels run row-group items (compute_item)
    Tmp buf(st);
    if (int rc = buf.alloc((5 * (T + 1) + 2 * (NW + 1)) * sizeof(int32_t))) return rc;
    int32_t *nitems = buf.as<int32_t>(), *nsplit = nitems + (T + 1), *parts = nitems + 2 * (T + 1),
            *splitId = nitems + 3 * (T + 1), *partBase = nitems + 4 * (T + 1), *wcount = nitems + 5 * (T + 1),
            *wbase = wcount + (NW + 1);
    TSP_CK(cudaMemsetAsync(nitems, 0, 3 * (T + 1) * sizeof(int32_t), st));
    TSP_CK(cudaMemsetAsync(wcount, 0, (NW + 1) * sizeof(int32_t), st));
    const TileView TV = tile_view(M);
    k_items_count<<<blocks(T), TB, 0, st>>>(TV, M.remRowPtr, M.m, M.item_bytes, M.item_tiles, T, nitems, nsplit, parts);
    k_window_count<<<blocks(NW), TB, 0, st>>>(TV, M.remRowPtr, M.m, M.item_bytes, M.item_tiles, T, group, nitems, NW,
                                               wcount);
    TSP_CK(cudaGetLastError());
    if (int rc = scan([&](void *t, size_t &b) { return cub::DeviceScan::ExclusiveSum(t, b, wcount, wbase, (int)(NW + 1), st); }, st)) return rc;
    if (int rc = scan([&](void *t, size_t &b) { return cub::DeviceScan::ExclusiveSum(t, b, nsplit, splitId, (int)(T + 1), st); }, st)) return rc;
    if (int rc = scan([&](void *t, size_t &b) { return cub::DeviceScan::ExclusiveSum(t, b, parts, partBase, (int)(T + 1), st); }, st)) return rc;
    int32_t h[3];
    TSP_CK(cudaMemcpyAsync(&h[0], wbase + NW, 4, cudaMemcpyDeviceToHost, st));
    TSP_CK(cudaMemcpyAsync(&h[1], splitId + T, 4, cudaMemcpyDeviceToHost, st));
    TSP_CK(cudaMemcpyAsync(&h[2], partBase + T, 4, cudaMemcpyDeviceToHost, st));
    TSP_CK(cudaStreamSynchronize(st));
    M.num_items = h[0];
    M.num_split = h[1];
    const int64_t nparts = h[2];
    TSP_CK(cudaMalloc(&M.items, std::max<int64_t>(M.num_items, 1) * sizeof(Item)));
    TSP_CK(cudaMalloc(&M.split_info, std::max<int64_t>(M.num_split, 1) * sizeof(int2)));
    TSP_CK(cudaMalloc(&M.counters, std::max<int64_t>(M.num_split, 1) * sizeof(int32_t)));
    TSP_CK(cudaMalloc(&M.partials, std::max<int64_t>(nparts, 1) * 16 * sizeof(double)));
    M.device_bytes += M.num_split * 12 + nparts * 128;
    // whole records (padding included) are copied later: start from zeros
    TSP_CK(cudaMemsetAsync(M.items, 0, std::max<int64_t>(M.num_items, 1) * sizeof(Item), st));
    TSP_CK(cudaMemsetAsync(M.counters, 0, std::max<int64_t>(M.num_split, 1) * sizeof(int32_t), st));
    k_window_write<<<blocks(NW), TB, 0, st>>>(TV, M.remRowPtr, M.m, M.item_bytes, M.item_tiles, T,
                                               group, nitems, NW, wbase, splitId, partBase, M.items, M.split_info,
                                               kLocalParts);
    TSP_CK(cudaGetLastError());
    return 0;
}

__global__ void k_col_hist(const int32_t *col, int64_t nnz, int32_t *cnt, int32_t *iota, int64_t n) {
    const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i < n) iota[i] = (int32_t)i;
    if (i < nnz) atomicAdd(cnt + col[i], 1);
}
// the first k of the columns sorted by decreasing count, if gathered at least twice
__global__ void k_xc_mark(const int32_t *cnt_s, const int32_t *col_s, int64_t k, int32_t *flag) {
    const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i < k && cnt_s[i] >= 2) flag[col_s[i]] = 1;
}
// slots in column order: slot[c] = prefix of the flags, -1 if c is not cached
__global__ void k_xc_write(const int32_t *flag, const int32_t *pos, int64_t n, int32_t *slot, int32_t *cols) {
    const int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (c >= n) return;
    const int32_t f = flag[c], q = pos[c];
    slot[c] = f ? q : -1;
    if (f) cols[q] = (int32_t)c;
}

// GATHER kernel's x cache (spmv_warp.cu): the (at most) `slots` remainder
// columns gathered most often (ties: lower column first; only columns
// gathered at least twice), in column order.  slot[c] = its cache slot or -1.
// A property of the handle's own entries: it moves where x is read from, never
// a value or a summation order, so y is the same with or without it.
static int build_xcache(Matrix &M, int slots, int32_t *slot, cudaStream_t st) {
    const int64_t n = M.n;
    Tmp ab(st), bb(st);
    if (int rc = ab.alloc(4 * (size_t)(n + 1) * sizeof(int32_t))) return rc;
    int32_t *cnt = ab.as<int32_t>(), *iota = cnt + (n + 1), *cnt_s = iota + (n + 1), *col_s = cnt_s + (n + 1);
    TSP_CK(cudaMemsetAsync(cnt, 0, (n + 1) * sizeof(int32_t), st));
    const int64_t mx = std::max<int64_t>(n, M.rem_nnz);
    k_col_hist<<<(unsigned)((mx + 255) / 256), 256, 0, st>>>(M.remCol, M.rem_nnz, cnt, iota, n);
    if (int rc = scan([&](void *t, size_t &b) {
            return cub::DeviceRadixSort::SortPairsDescending(t, b, cnt, cnt_s, iota, col_s, (int)n, 0, 32, st);
        }, st)) return rc;
    // flags over columns (reusing cnt), then their exclusive prefix (in iota)
    int32_t *flag = cnt, *pos = iota;
    TSP_CK(cudaMemsetAsync(flag, 0, (n + 1) * sizeof(int32_t), st));
    const int64_t k = std::min<int64_t>(slots, n);
    k_xc_mark<<<(unsigned)((k + 255) / 256), 256, 0, st>>>(cnt_s, col_s, k, flag);
    if (int rc = scan([&](void *t, size_t &b) { return cub::DeviceScan::ExclusiveSum(t, b, flag, pos, (int)(n + 1), st); }, st)) return rc;
    int32_t nx = 0;
    TSP_CK(cudaMemcpyAsync(&nx, pos + n, 4, cudaMemcpyDeviceToHost, st));
    TSP_CK(cudaStreamSynchronize(st));
    TSP_CK(cudaMalloc(&M.xc_cols, std::max(nx, 1) * sizeof(int32_t)));
    M.device_bytes += std::max(nx, 1) * 4;
    M.xc_n = nx;
    k_xc_write<<<(unsigned)((n + 255) / 256), 256, 0, st>>>(flag, pos, n, slot, M.xc_cols);
    TSP_CK(cudaGetLastError());
    return 0;
}

int build_tdesc(Matrix &M, cudaStream_t st) {
    const int64_t n = M.num_items;
    if (n == 0) {
        TSP_CK(cudaMalloc(&M.blob, 256));
        TSP_CK(cudaMalloc(&M.witems, sizeof(WItem)));
        TSP_CK(cudaMalloc(&M.jcols, 16 * sizeof(int32_t)));
        M.device_bytes += 256 + sizeof(WItem) + 64;
        return 0;
    }
    Tmp cntb(st);
    if (int rc = cntb.alloc(2 * (n + 1) * sizeof(int32_t))) return rc;
    int32_t *cnt = cntb.as<int32_t>(), *beg = cnt + (n + 1);
    const unsigned nb = (unsigned)((n + 255) / 256);
    TSP_CK(cudaMemsetAsync(cnt + n, 0, sizeof(int32_t), st));
    const TileView TV = tile_view(M);
    k_dsc_count<<<nb, 256, 0, st>>>(M.items, n, TV, cnt);
    if (int rc = scan([&](void *t, size_t &b) { return cub::DeviceScan::ExclusiveSum(t, b, cnt, beg, (int)(n + 1), st); }, st)) return rc;
    int32_t total = 0;
    TSP_CK(cudaMemcpyAsync(&total, beg + n, 4, cudaMemcpyDeviceToHost, st));
    TSP_CK(cudaStreamSynchronize(st));
    M.num_dsc = total;
    TSP_CK(cudaMallocAsync(&M.tdesc, (total + 4) * sizeof(uint2), st));  // create-time only
    k_dsc_write<<<nb, 256, 0, st>>>(M.items, n, beg, cnt, TV, M.tdesc);
    TSP_CK(cudaGetLastError());
    // execution blobs
    Tmp lenb(st);
    if (int rc = lenb.alloc(2 * (n + 1) * sizeof(int64_t))) return rc;
    int64_t *len16 = lenb.as<int64_t>(), *start16 = len16 + (n + 1);
    TSP_CK(cudaMemsetAsync(len16 + n, 0, sizeof(int64_t), st));
    TSP_CK(cudaMemsetAsync(cnt + n, 0, sizeof(int32_t), st));  // cnt[n]: slot overflow flag
    k_blob_len<<<nb, 256, 0, st>>>(M.items, n, M.m, (uint32_t)M.item_bytes, TV, M.remRowPtr, M.remCol, M.item_tiles,
                                   len16, cnt + n);
    if (int rc = scan([&](void *t, size_t &b) { return cub::DeviceScan::ExclusiveSum(t, b, len16, start16, (int)(n + 1), st); }, st)) return rc;
    int64_t total16 = 0;
    int32_t over = 0;
    TSP_CK(cudaMemcpyAsync(&total16, start16 + n, 8, cudaMemcpyDeviceToHost, st));
    TSP_CK(cudaMemcpyAsync(&over, cnt + n, 4, cudaMemcpyDeviceToHost, st));
    TSP_CK(cudaStreamSynchronize(st));
    if (over) return set_error(TILESPMV_CUDA, "schedule: an item's blob exceeds the kernel's slot");
    if (total16 >= (int64_t(1) << 32)) return set_error(TILESPMV_OVERFLOW, "execution blob >= 64 GiB");
    M.blob_bytes = total16 * 16;
    // GATHER: the kernel's x cache holds the most-gathered remainder columns
    Tmp xcb(st);
    int32_t *xc_slot = nullptr;
    const int xcache = kernel_choice(M.kernel).xcache;
    if (xcache > 0 && M.rem_nnz > 0) {
        if (int rc = xcb.alloc((size_t)(M.n + 1) * sizeof(int32_t))) return rc;
        xc_slot = xcb.as<int32_t>();
        if (int rc = build_xcache(M, xcache, xc_slot, st)) return rc;
    }
    TSP_CK(cudaMalloc(&M.blob, M.blob_bytes + 256));
    M.device_bytes += M.blob_bytes + 256;
    TSP_CK(cudaMalloc(&M.witems, n * sizeof(WItem)));
    TSP_CK(cudaMalloc(&M.jcols, n * 16 * sizeof(int32_t)));
    M.device_bytes += n * (int64_t)(sizeof(WItem) + 64);
    k_blob_fill<<<(unsigned)((n * 32 + 255) / 256), 256, 0, st>>>(M.items, n, M.m, M.n, start16, M.tdesc, M.tileColIdx,
                                                                 TV, M.payload, M.remRowPtr, M.remCol, M.remVal,
                                                                 M.blob, M.witems, M.jcols, xc_slot);
    TSP_CK(cudaGetLastError());
    return 0;
}

int auto_kernel(int64_t payload_bytes, int64_t tilem, int64_t rem_nnz, int64_t alg) {
    // the remainder's bytes (12 per entry) are most of what the SpMV moves:
    // its x gathers need the L1 that the big-slot kernels give to shared memory
    if (2 * 12 * rem_nnz > alg) return TILESPMV_KERNEL_GATHER;
    // integer form of "mean payload per tile row > 6 KiB"
    return tilem > 0 && payload_bytes > 6144 * tilem ? TILESPMV_KERNEL_DENSE_ROWS : TILESPMV_KERNEL_SM_QUEUE;
}

int choose_kernel(Matrix &M, int requested) {
    // AUTO: the SM-queue kernel (one CTA of 32 warps per SM, 4.5 KB slots,
    // warps claim units from a shared-memory counter); matrices whose tile
    // rows average more than 6 KB of payload (dense, FEM-like) use the
    // dense-row kernel with 10.5 KB slots (16 warps/SM) so a tile row stays
    // one item.  Measured in round 1 (graph-replayed launches, profiles/):
    // C5 498 us (SM queue) vs 512 us (static chunks); R-MAT 145 vs 163 us;
    // mixed 113 vs 116 us; C2 6.9 us (dense-row) vs 7.5 us (SM queue, 10.5 KB).
    const int k = requested == TILESPMV_KERNEL_AUTO ? auto_kernel(M.payload_bytes, M.tilem, M.rem_nnz, alg_bytes(M))
                                                    : requested;
    const KernelChoice kc = kernel_choice(k);
    M.kernel = k;
    M.item_bytes = kc.slot_bytes;
    M.item_tiles = kc.item_tiles;
    return 0;
}

// SM-queue kernel: units (items, or whole groups of parts) and a
// contiguous, cost-balanced unit range per CTA
static int configure_sm_queue(Matrix &M, int G, cudaStream_t st) {
    M.grid = G;
    const int64_t n = M.num_items;
    TSP_CK(cudaMalloc(&M.cta_begin, (G + 1) * sizeof(int64_t)));
    if (n == 0) {
        TSP_CK(cudaMalloc(&M.units, sizeof(int2)));
        M.device_bytes += (G + 1) * 8 + 8;
        TSP_CK(cudaMemsetAsync(M.cta_begin, 0, (G + 1) * sizeof(int64_t), st));
        TSP_CK(cudaMemsetAsync(M.units, 0, sizeof(int2), st));
        M.num_units = 0;
        return 0;
    }
    Tmp costb(st), flagb(st), ub(st);
    if (int rc = costb.alloc(2 * n * sizeof(int64_t))) return rc;
    if (int rc = flagb.alloc(2 * (n + 1) * sizeof(int32_t))) return rc;
    if (int rc = ub.alloc((n + 1) * sizeof(int32_t))) return rc;
    int64_t *cost = costb.as<int64_t>(), *incl = cost + n;
    int32_t *flag = flagb.as<int32_t>(), *pos = flag + (n + 1), *ustart = ub.as<int32_t>();
    const unsigned nb = (unsigned)((n + 1 + 255) / 256);
    k_item_cost<<<nb, 256, 0, st>>>(M.items, n, M.m, kItemFixedCost,
                                    M.kernel == TILESPMV_KERNEL_GATHER ? kGroupRowCostPre : kGroupRowCost, cost);
    if (int rc = scan([&](void *t, size_t &b) { return cub::DeviceScan::InclusiveSum(t, b, cost, incl, (int)n, st); }, st)) return rc;
    TSP_CK(cudaMemsetAsync(flag + n, 0, sizeof(int32_t), st));
    k_unit_flags<<<nb, 256, 0, st>>>(M.items, n, kLocalParts, flag);
    if (int rc = scan([&](void *t, size_t &b) { return cub::DeviceScan::ExclusiveSum(t, b, flag, pos, (int)(n + 1), st); }, st)) return rc;
    int32_t nu = 0;
    TSP_CK(cudaMemcpyAsync(&nu, pos + n, 4, cudaMemcpyDeviceToHost, st));
    TSP_CK(cudaStreamSynchronize(st));
    M.num_units = nu;
    k_unit_write<<<nb, 256, 0, st>>>(flag, pos, n, ustart);
    k_cta_units<<<(G + 1 + 255) / 256, 256, 0, st>>>(incl, ustart, nu, n, G, M.cta_begin);
    // inside each CTA's range the warps claim units costliest first
    // (longest-processing-time order), so the SM's tail is made of its
    // smallest units: all units for GATHER (power-law remainders; R-MAT 99.4
    // -> 93.2 us), only the big ones (>= 2x the mean unit cost) for SM_QUEUE,
    // whose other units keep their tile-row order (sorting them all cost C5
    // 5%: neighbouring tile rows share x lines); stable sort
    TSP_CK(cudaMalloc(&M.units, (size_t)nu * sizeof(int2)));
    M.device_bytes += (G + 1) * 8 + (int64_t)nu * 8;
    {
        Tmp kb(st), vb(st);
        if (int rc = kb.alloc(2 * (size_t)nu * sizeof(int64_t))) return rc;
        if (int rc = vb.alloc(2 * (size_t)nu * sizeof(int32_t))) return rc;
        int64_t *ucost = kb.as<int64_t>(), *ucost_s = ucost + nu;
        int32_t *uidx = vb.as<int32_t>(), *uidx_s = uidx + nu;
        const unsigned nbu = (unsigned)((nu + 255) / 256);
        k_unit_cost<<<nbu, 256, 0, st>>>(incl, ustart, nu, n, M.kernel == TILESPMV_KERNEL_GATHER, ucost, uidx);
        if (int rc = scan([&](void *t, size_t &b) {
                return cub::DeviceSegmentedSort::StableSortPairsDescending(t, b, ucost, ucost_s, uidx, uidx_s, (int)nu, G,
                                                                           M.cta_begin, M.cta_begin + 1, st);
            }, st)) return rc;
        k_unit_bounds<<<nbu, 256, 0, st>>>(ustart, uidx_s, nu, M.units);
    }
    TSP_CK(cudaGetLastError());
    return 0;
}

int configure_launch(Matrix &M, cudaStream_t st) {
    const KernelChoice kc = kernel_choice(M.kernel);
    TSP_CK(cudaFuncSetAttribute(kc.fn, cudaFuncAttributeMaxDynamicSharedMemorySize, kc.smem));
    TSP_CK(cudaFuncSetAttribute(kc.fn_scatter, cudaFuncAttributeMaxDynamicSharedMemorySize, kc.smem));
    int sms = 0, per_sm = 0;
    TSP_CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, M.device));
    TSP_CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kc.fn, kc.threads, kc.smem));
    if (per_sm < 1) return set_error(TILESPMV_CUDA, "SpMV kernel does not fit on an SM");
    M.kernel_name = kc.name;
    M.block = kc.threads;
    M.smem = kc.smem;
    if (kc.sm_queue) return configure_sm_queue(M, sms * per_sm, st);
    // dense-row kernel: persistent grid, one contiguous, cost-balanced,
    // row-aligned item chunk per warp
    const int64_t warps = kc.threads / 32;
    const int64_t need = (M.num_items + warps - 1) / warps;
    M.grid = (int)std::max<int64_t>(1, std::min<int64_t>(need, (int64_t)sms * per_sm));
    const int W = (int)(M.grid * warps);
    TSP_CK(cudaMalloc(&M.cta_begin, (W + 1) * sizeof(int64_t)));
    M.device_bytes += (W + 1) * 8;
    if (M.num_items > 0) {
        Tmp costb(st);
        if (int rc = costb.alloc(2 * M.num_items * sizeof(int64_t))) return rc;
        int64_t *cost = costb.as<int64_t>(), *incl = cost + M.num_items;
        k_item_cost<<<(unsigned)((M.num_items + 255) / 256), 256, 0, st>>>(M.items, M.num_items, M.m, kItemFixedCost,
                                                                         kGroupRowCost, cost);
        if (int rc = scan([&](void *t, size_t &b) { return cub::DeviceScan::InclusiveSum(t, b, cost, incl, (int)M.num_items, st); }, st))
            return rc;
        k_cta_begin<<<(W + 1 + 255) / 256, 256, 0, st>>>(incl, M.items, M.num_items, W, kLocalParts, M.cta_begin);
        TSP_CK(cudaGetLastError());
    } else {
        TSP_CK(cudaMemsetAsync(M.cta_begin, 0, (W + 1) * sizeof(int64_t), st));
    }
    TSP_CK(cudaMalloc(&M.wfirst, W * sizeof(WFirst)));
    M.device_bytes += W * (int64_t)sizeof(WFirst);
    k_warp_first<<<(W + 255) / 256, 256, 0, st>>>(M.cta_begin, M.witems, M.jcols, W, M.wfirst);
    TSP_CK(cudaGetLastError());
    return 0;
}

// After the schedule is built: free what only create needed (items, the
// descriptor lists) and, unless the caller asked to keep the canonical
// layout (tilespmv_export), the canonical level-1/level-2 arrays and the
// remainder CSR, which the kernels never read (they read the blobs).
void release_create_time(Matrix &M, cudaStream_t st) {
    auto drop = [&](auto *&p) {
        if (p) cudaFreeAsync(p, st);
        p = nullptr;
    };
    drop(M.items);
    drop(M.tdesc);
    if (M.keep_layout) {
        M.device_bytes += (M.tilem + 1) * 4 + M.numtile * 14 + 8 + M.payload_bytes + 64;
        if (M.rem_nnz > 0) M.device_bytes += (M.m + 1 + 8) * 4 + (M.rem_nnz + 4) * 4 + (M.rem_nnz + 2) * 8;
        return;
    }
    drop(M.tilePtr);
    drop(M.tileColIdx);
    drop(M.tileNnz);
    drop(M.tileFmt);
    drop(M.tileAux);
    drop(M.tileOff);
    drop(M.payload);
    drop(M.remRowPtr);
    drop(M.remCol);
    drop(M.remVal);
}

int launch_spmv(const Matrix &M, const double *d_x, double *d_y, cudaStream_t st, double *const *yx, int nyx) {
    if (M.m == 0) return 0;
    Params p;
    p.nyx = nyx;
    for (int t = 0; t < kMaxScatter; ++t) p.yx[t] = t < nyx ? yx[t] : nullptr;
    p.blob = M.blob;
    p.witems = M.witems;
    p.jcols = M.jcols;
    p.wfirst = M.wfirst;
    p.cta_begin = M.cta_begin;
    p.units = M.units;
    p.xc_cols = M.xc_cols;
    p.xc_n = M.xc_n;
    p.split_info = M.split_info;
    p.partials = M.partials;
    p.counters = M.counters;
    p.x = d_x;
    p.y = d_y;
    p.m = M.m;
    p.n = M.n;
    p.x_vec = (reinterpret_cast<uintptr_t>(d_x) & 15u) == 0;
    p.blob_bytes = M.blob_bytes;
    p.num_items = M.num_items;
    p.slot_bytes = M.item_bytes;
    const KernelChoice kc = kernel_choice(M.kernel);
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(M.grid);
    cfg.blockDim = dim3(M.block);
    cfg.dynamicSmemBytes = M.smem;
    cfg.stream = st;
    // programmatic dependent launch: the kernel waits (griddepcontrol.wait)
    // before its first read of x or write of y
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    TSP_CK(cudaLaunchKernelEx(&cfg, nyx > 0 ? kc.fn_scatter : kc.fn, p));
    return 0;
}

}  // namespace tsp
