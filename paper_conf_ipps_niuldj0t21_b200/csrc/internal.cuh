// internal.cuh -- shared definitions of the CUDA product path (tiler, SpMV
// kernel, C ABI).  Nothing here is shared with oracle/.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <string>

#include "../../include/tilespmv.h"

namespace tsp {

constexpr int kTile = 16;  // P:20 "the size is always 16 by 16"
constexpr int kMaxScatter = 7;  // tilespmv_run_scatter: peers (the other 7 GPUs of one node)

// Format codes (same numbering as the ABI, P:96 order).
enum : uint8_t { F_CSR = 0, F_COO = 1, F_ELL = 2, F_HYB = 3, F_DNS = 4, F_DNSROW = 5, F_DNSCOL = 6 };
// execution-descriptor code of a merged CSR pair (schedule.cu, CSR2): COO
// tiles never get descriptors, so their code is free on the execution side
constexpr uint8_t F_CSR2 = F_COO;

// ---------------------------------------------------------------------------
// SpMV schedule.  A work item is a byte-bounded piece of one tile row: a run
// of at most kItemTiles (the kernel's item_tiles) consecutive tiles and/or a
// range of remainder entries of the tile row's 16 rows, such that everything
// the kernel stages for it (payloads, 8-byte tile descriptors, remainder
// rowptr/col/val) fits one shared-memory slot (the kernel's slot size,
// <= kItemBytesMax).  A tile row split over several items writes
// per-item partials that the last finishing item sums in item order
// (deterministic; replaces the atomic merge of tbalance).  Item
// boundaries depend only on the tile row's own content, so a tile-row-sharded
// run reproduces the 1-GPU y bitwise.
// ---------------------------------------------------------------------------
constexpr int kItemTiles = 16;
constexpr int kItemBytesMax = 12288;  // largest shared-memory slot of any kernel

struct __align__(16) Item {
    int32_t I;        // tile row
    int32_t tb;       // first tile
    int32_t kb, ke;   // remainder entry range
    uint32_t offb;    // payload offset of tile tb (16-byte units)
    uint32_t offe;    // payload offset one past the last tile
    uint32_t pay_bytes;  // bytes of the tiles in the blob payload (tile_cost; canonical unless a COO run)
    uint32_t run_e;      // entries of the item's COO run (ADPT: COO tiles + HYB COO parts; DEFERRED:
                         // a remainder whose x lies in the item's staged segments), 0 if none
    uint32_t xseg;       // x segments the kernel stages: the tiles' J, then (local remainder) the
                         // remainder's other tile columns
    int32_t split;    // split-row index, or -1 if the item covers its whole tile row
    int32_t part_nt;  // part index (bits 0-23) | tiles << 24 (5 bits) | local << 29 | last-of-group << 30
    int32_t dbeg;      // first entry of the item's tile-descriptor list (dlist)
    int32_t ndsc;      // entries: the item's tiles grouped by format, groups padded to even length
    uint32_t blob16;   // start of the item's execution blob (16-byte units)
    uint32_t blob_len; // bytes of the blob (blob_parts)
    int32_t ntr;       // row-group item: consecutive tile rows I..I+ntr-1 (0: ordinary item)
};

// Row-group items (warp kernel): consecutive tile rows that hold no stored
// tile and whose remainder rows fit one slot together (power-law matrices:
// most R-MAT tile rows hold a few dozen remainder entries, or none) share one
// item of up to kGroupTileRows tile rows, formed inside windows of
// kGroupWindow tile rows.  Every tile row of a group item is summed by the
// same flat pass whether it is grouped with its neighbours or alone, so the
// grouping never changes a bit of y (shard invariance).
constexpr int kGroupTileRows = 16;
constexpr int kGroupWindow = 64;

// Compact per-item record read by the warp kernel (built with the blobs):
// blob start, tile row, split bookkeeping, and the blob's part offsets.
struct __align__(16) WItem {
    uint32_t blob16;    // blob start (16-byte units)
    uint32_t I;         // tile row
    int32_t split;      // split-row index or -1
    int32_t part_nt;    // as Item::part_nt
    uint32_t jt_rows_pay;  // tile rows of a row-group item (8 bits, 0: ordinary) | rows in the (last) tile row (5 bits) << 8 | payload offset << 16
    uint32_t rp_col;       // rp offset | col offset << 16
    uint32_t val_tot;      // val offset | total bytes << 16
    uint32_t groups;       // tile pairs per format f, 4 bits at 4f (descriptor list order);
                           // bit 28: every CSR row of the item <= 3 entries, bit 29: every ELL width <= 3,
                           // bit 30: the last tile column's x segment passes x[n-1] (ragged tail),
                           // bit 31: the rp/col/val parts are a COO run (ADPT), not a CSR remainder
};

// Per-warp start record of the dense-row kernel: the warp's item chunk and a
// copy of its first item, so the prologue needs one round trip before the
// blob copy.
struct __align__(16) WFirst {
    int32_t kbeg, kend, pad0, pad1;
    WItem w;
    int32_t J[16];
};

// The parts of a split tile row form groups of kLocalParts consecutive parts.
// One warp runs a whole group in order, carrying the partial row sums in
// registers.  A row of one group ("local") writes y directly; a hub row of
// several groups writes one partial per group and the last group to finish
// sums the group partials in group order.  Everything depends only on the
// row's own content (deterministic, shard-invariant).
constexpr int kLocalParts = 4;
// per-item fixed cost (bytes-equivalent of an item's latency chain: record,
// blob, x gathers) used to balance the warps' item chunks; measured on R-MAT
// (power-law, many small items): 2048 gave 174 us against 188 us for 512,
// neutral on the stencil and mixed matrices (round 1)
constexpr int64_t kItemFixedCost = 2048;
// row-group items cost more per byte than their bytes say (two tile rows per
// step, one chain of gather round trips each): per-item traces of R-MAT
// (profiles/r02_ab/trace_items_rmat20.txt) put a row-group item at 5.99 us
// for 2,392 B against 5.12 us for a 3,071 B remainder-only item; charging
// 320 per tile row of a group moves R-MAT from 108.8 to 102.9 us
// (profiles/r02_ab/group_row_cost_rmat20.txt; 160: 104.1, 640: 104.0)
constexpr int64_t kGroupRowCost = 320;
// ... with the GATHER kernel's product pre-pass a row-group item costs close
// to what its bytes say (R-MAT traces: 4.71 us for 2,224 B against 5.47 us
// for a 2,911 B remainder-only item); 80 per tile row measured best (R-MAT
// 0 / 80 / 160 / 320: 90.8 / 86.5 / 86.9 / 88.4 us, profiles/r02_ab2)
constexpr int64_t kGroupRowCostPre = 80;
__host__ __device__ __forceinline__ int item_nt(const Item &it) { return (it.part_nt >> 24) & 31; }
__host__ __device__ __forceinline__ int item_part(const Item &it) { return it.part_nt & 0xFFFFFF; }
__host__ __device__ __forceinline__ bool item_local(const Item &it) { return (it.part_nt >> 29) & 1; }
__host__ __device__ __forceinline__ bool item_last(const Item &it) { return (it.part_nt >> 30) & 1; }

struct Matrix {
    int device = 0;
    int64_t m = 0, n = 0, nnz = 0, tilem = 0, tilen = 0, numtile = 0;
    int32_t mode = TILESPMV_MODE_DEFERRED;
    bool keep_layout = false;  // keep the canonical arrays after create (tilespmv_export)
    // level 1 + format bytes + payload offsets; create-time only
    // unless keep_layout
    int32_t *tilePtr = nullptr, *tileColIdx = nullptr, *tileNnz = nullptr;
    uint8_t *tileFmt = nullptr, *tileAux = nullptr;
    uint32_t *tileOff = nullptr;
    // level 2
    uint8_t *payload = nullptr;
    int64_t payload_bytes = 0;
    // DeferredCOO remainder
    int32_t *remRowPtr = nullptr, *remCol = nullptr;
    double *remVal = nullptr;
    int64_t rem_nnz = 0;
    // SpMV schedule (create-time: items, tdesc)
    Item *items = nullptr;
    int64_t num_items = 0;
    uint2 *tdesc = nullptr;        // per-item tile-descriptor lists (dlist)
    int64_t num_dsc = 0;
    int2 *split_info = nullptr;  // {first partial slot, number of parts}
    int64_t num_split = 0;
    double *partials = nullptr;
    int32_t *counters = nullptr;
    // what the kernels read
    uint8_t *blob = nullptr;       // per-item execution blobs (blob_parts)
    WItem *witems = nullptr;       // compact per-item records
    int32_t *jcols = nullptr;      // 16 tile columns per item
    WFirst *wfirst = nullptr;      // dense-row kernel: per-warp chunk + first item
    int64_t blob_bytes = 0;
    int64_t *cta_begin = nullptr;  // dense-row kernel: item chunk per warp (row-aligned, cost-balanced);
                                   // SM-queue kernel: unit range per CTA
    int2 *units = nullptr;         // SM-queue kernel: [first, end) items of each unit, in claim order
                                   // (inside each CTA's range: decreasing cost)
    int64_t num_units = 0;
    int32_t *xc_cols = nullptr;    // GATHER kernel: columns of the shared-memory x cache (slot order)
    int32_t xc_n = 0;
    // host-staging buffers for tilespmv_run_host
    double *xstage = nullptr, *ystage = nullptr;
    // statistics
    int64_t sel_tiles[7] = {0}, sel_nnz[7] = {0}, kept_tiles[7] = {0}, kept_nnz[7] = {0};
    int64_t device_bytes = 0;
    double create_ms = 0;
    // launch shape
    int kernel = TILESPMV_KERNEL_SM_QUEUE;  // resolved kernel (never AUTO)
    const char *kernel_name = "";
    int item_bytes = kItemBytesMax;  // slot size the schedule was built for
    int item_tiles = kItemTiles;     // tiles per item (the kernel's x stage)
    int grid = 0, block = 0, smem = 0;
};

// status helpers (thread-local last error)
int set_error(int status, const std::string &msg);
int cuda_status(cudaError_t e, const char *what);

// tiler.cu
int build_tiled(Matrix &M, const int32_t *d_rowptr, const int32_t *d_colidx, const double *d_val,
                int validate, cudaStream_t stream);
// schedule.cu
int auto_kernel(int64_t payload_bytes, int64_t tilem, int64_t rem_nnz, int64_t alg_bytes);
int64_t alg_bytes(const Matrix &M);  // abi.cu
int choose_kernel(Matrix &M, int requested);
int build_schedule(Matrix &M, cudaStream_t stream);
int build_tdesc(Matrix &M, cudaStream_t stream);
int configure_launch(Matrix &M, cudaStream_t stream);
void release_create_time(Matrix &M, cudaStream_t stream);
int launch_spmv(const Matrix &M, const double *d_x, double *d_y, cudaStream_t stream, double *const *yx = nullptr,
                int nyx = 0);
// cg.cu
int cg_solve(const Matrix &M, const double *d_b, double *d_x, double tol, int maxit, int *iters, double *relres,
             cudaStream_t stream);

}  // namespace tsp
