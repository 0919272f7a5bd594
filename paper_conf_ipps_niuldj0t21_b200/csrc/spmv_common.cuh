// spmv_common.cuh -- pieces shared by the SpMV kernels (spmv_warp.cu) and
// the schedule builder (schedule.cu).
#pragma once

#include "internal.cuh"

// TSP_CHECKED (scripts/checked_small.py only): device-side bounds checks of
// every blob copy, x read, x segment and unit index against the handle's
// sizes; a failed check is a device assert.  Off in the product build.
#ifdef TSP_CHECKED
#include <cassert>
#define TSP_CHECK(c) assert(c)
#else
#define TSP_CHECK(c) ((void)0)
#endif

namespace tsp {

constexpr unsigned FULL = 0xffffffffu;

// Everything a launch reads; passed by value in constant memory.  The
// kernels read only the schedule's execution records (schedule.cu), never the
// canonical level-1/level-2 arrays, which the handle may free after create.
struct Params {
    const uint8_t *blob;       // per-item execution blobs (blob_parts)
    const WItem *witems;       // compact per-item records
    const int32_t *jcols;      // tile column J of each item's tiles, 16 per item
    const WFirst *wfirst;      // warp kernel: per-warp chunk and first item
    const int64_t *cta_begin;  // SM-queue kernel: unit range of each CTA
    const int2 *units;         // SM-queue kernel: item range of each unit, in claim order
    const int2 *split_info;    // split tile rows: {first partial slot, parts}
    double *partials;
    int32_t *counters;
    const double *x;
    double *y;
    int64_t m, n;
    int x_vec;                 // x is 16-byte aligned: x segments load as double2
    int nyx;                   // tilespmv_run_scatter: peers' y copies (0: plain run)
    double *yx[kMaxScatter];   // each row of y is also stored to yx[t][row], t < nyx
    int64_t blob_bytes, num_items;  // sizes for the TSP_CHECKED build's bounds checks
    int slot_bytes;
    const int32_t *xc_cols;    // GATHER: the columns of the shared-memory x cache
    int xc_n;                  // (their number, <= the kernel's cache slots)
};

// ------------------------------------------------------------------ PTX ----
__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void fence_proxy_async() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint32_t bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint32_t bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ bool mbar_try_wait(uint32_t bar, uint32_t parity) {
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(ok)
        : "r"(bar), "r"(parity)
        : "memory");
    return ok != 0;
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
    while (!mbar_try_wait(bar, parity)) {
    }
}

__host__ __device__ __forceinline__ int64_t imin64(int64_t a, int64_t b) { return a < b ? a : b; }
__host__ __device__ __forceinline__ uint32_t up16(uint32_t v) { return (v + 15u) & ~15u; }

// rows the item's remainder row pointers cover
__host__ __device__ __forceinline__ int64_t item_rows(const Item &it, int64_t m) {
    return imin64(it.ntr > 0 ? 16 * (int64_t)it.ntr : 16, m - 16 * (int64_t)it.I);
}

// ---------------------------------------------- one item's execution blob --
// A create-time copy of everything one work item reads, contiguous and
// 16-byte aligned part by part, so a single TMA bulk copy stages it:
//   dsc : the descriptor list (k_dsc_write), ndsc x 8 B
//   pay : the tiles' payload bytes: canonical, except that with a
//         COO run a COO tile is absent and a HYB(w) tile is its ELL(w) part
//   rp  : remainder row pointers of the item's rows, rebased to the item's
//         entry range and clamped to it (rows + 1 ints)
//   col, val : the item's remainder entries
// ADPT mode instead gathers the item's COO data -- its COO tiles and the
// COO parts of its HYB tiles, at most 11 and 15 entries per tile (P:181,
// P:105) -- into one COO run in the same three parts: rp = the 16 row
// pointers (+ end) of the run, col = one byte per entry holding its x slot
// (tile index * 16 + column in the tile), val = the values, entries in row
// order and, within a row, in tile then column order.  The kernel sums the
// run two lanes per row from the staged x segments (coo_run) instead of
// running each 1..11-entry tile on its own half-warp.
__host__ __device__ __forceinline__ uint32_t run_bytes(uint32_t e) {
    return e ? 80u + up16(e) + up16(8u * e) : 0u;
}

struct BlobParts {
    uint32_t pay, rp, col, val, total;
};

__host__ __device__ __forceinline__ BlobParts blob_parts(const Item &it, int64_t m) {
    BlobParts b;
    b.pay = up16(8u * (uint32_t)it.ndsc);
    b.rp = b.pay + it.pay_bytes;
    if (it.run_e > 0) {
        b.col = b.rp + 80u;
        b.val = b.col + up16(it.run_e);
        b.total = b.val + up16(8u * it.run_e);
    } else if (it.ke > it.kb) {
        const uint32_t rows = (uint32_t)item_rows(it, m);
        const uint32_t e = (uint32_t)(it.ke - it.kb);
        b.col = b.rp + up16(4u * (rows + 1));
        b.val = b.col + up16(4u * e);
        b.total = b.val + up16(8u * e);
    } else {
        b.col = b.val = b.total = b.rp;
    }
    return b;
}

// L2 cache policies: the streamed blobs are read once (evict first), x is
// reused by neighbouring tile rows (evict last)
__device__ __forceinline__ uint64_t policy_evict_first() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ uint64_t policy_evict_last() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ void bulk_g2s_hint(uint32_t dst, const void *src, uint32_t bytes, uint32_t bar,
                                              uint64_t policy) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::"r"(dst),
        "l"(src), "r"(bytes), "r"(bar), "l"(policy)
        : "memory");
}
__device__ __forceinline__ double ldg_hint(const double *p, uint64_t policy) {
    double v;
    asm volatile("ld.global.nc.L2::cache_hint.f64 %0, [%1], %2;" : "=d"(v) : "l"(p), "l"(policy));
    return v;
}
__device__ __forceinline__ void sts_v2f64(uint32_t a, double2 v) {
    asm volatile("st.shared.v2.f64 [%0], {%1, %2};" ::"r"(a), "d"(v.x), "d"(v.y) : "memory");
}
// 16-byte async copy global -> shared; bytes beyond src_bytes (0..16) are zero-filled
__device__ __forceinline__ void cp_async16(uint32_t dst, const void *src, uint32_t src_bytes, uint64_t policy) {
    asm volatile("cp.async.cg.shared.global.L2::cache_hint [%0], [%1], 16, %2, %3;" ::"r"(dst), "l"(src),
                 "r"(src_bytes), "l"(policy)
                 : "memory");
}
// 8-byte async copy global -> shared (an x gather; .ca: the L1 may hold hot x lines)
__device__ __forceinline__ void cp_async8(uint32_t dst, const void *src, uint64_t policy) {
    asm volatile("cp.async.ca.shared.global.L2::cache_hint [%0], [%1], 8, %2;" ::"r"(dst), "l"(src), "l"(policy)
                 : "memory");
}
__device__ __forceinline__ void cp_async_wait_all() {
    asm volatile("cp.async.commit_group;\n\tcp.async.wait_group 0;" ::: "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
// counter += v with acquire-release semantics at gpu scope; returns the old value
__device__ __forceinline__ int atom_add_acq_rel_gpu(int32_t *a, int v) {
    int old;
    asm volatile("atom.acq_rel.gpu.global.add.s32 %0, [%1], %2;" : "=r"(old) : "l"(a), "r"(v) : "memory");
    return old;
}
// Programmatic dependent launch: let the next kernel in the stream start its
// prologue early / wait until the previous kernel's writes are visible
__device__ __forceinline__ void griddep_launch_dependents() {
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}
__device__ __forceinline__ void griddep_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
// acc += a * b only where pred holds (one predicated DFMA, no select)
__device__ __forceinline__ void fma_if(bool pred, double a, double b, double &acc) {
    asm("{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %3, 0;\n\t@q fma.rn.f64 %0, %1, %2, %0;\n\t}"
        : "+d"(acc)
        : "d"(a), "d"(b), "r"((unsigned)pred));
}

// the SpMV kernels (spmv_warp.cu)
struct KernelChoice {
    const char *name;
    void (*fn)(Params);
    void (*fn_scatter)(Params);  // the same kernel storing y to the peer copies too (tilespmv_run_scatter)
    int threads, smem;
    int slot_bytes;   // item budget the schedule must respect
    int item_tiles;   // tiles per item (x stage segments)
    bool sm_queue;    // one CTA per SM; its warps claim units from a shared-memory counter
    int xcache;       // slots of the shared-memory x cache (0: none)
};
// GATHER kernel: x cache slots (8 B each) and slot bytes, sized so the
// kernel's 131 KB of shared memory stays in the 132 KB carve-out step
// (R-MAT: 1,024 / 3,136 B 88.4 us; 4,096 / 3,328 B, 164 KB step, 93.0 us;
// 2,048 / 3,136 B once the COO-scan scratch went: 83.5 us)
constexpr int kXCache = 2048;
constexpr int kGatherSlot = 3136;
// TILESPMV_KERNEL_SM_QUEUE, _DENSE_ROWS or _GATHER
KernelChoice kernel_choice(int kernel);

}  // namespace tsp
