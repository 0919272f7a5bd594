// spmv_common.cuh -- pieces shared by the SpMV kernels (spmv_v1.cu,
// spmv_warp.cu) and the schedule builder (schedule.cu).
#pragma once

#include "internal.cuh"

namespace tsp {

constexpr unsigned FULL = 0xffffffffu;

// Everything a launch reads; passed by value in constant memory.
struct Params {
    const Item *items;
    int64_t num_items;
    const int32_t *tileColIdx;
    const uint8_t *tileFmt;
    const uint8_t *tileAux;
    const int32_t *tileNnz;
    const uint32_t *tileOff;
    const uint8_t *payload;
    const int32_t *remRowPtr;
    const int32_t *remCol;
    const double *remVal;
    const int2 *split_info;
    double *partials;
    int32_t *counters;
    const double *x;
    double *y;
    int64_t m, n;
    const uint2 *tdesc;        // per-item tile-descriptor lists (schedule.cu)
    const uint8_t *blob;       // per-item execution blobs (schedule.cu)
    const WItem *witems;       // compact per-item records (schedule.cu)
    const int32_t *jcols;      // tile column J of each item's tiles, 16 per item
    const WFirst *wfirst;      // per-warp chunk and first item (warp kernel)
    const int64_t *cta_begin;  // warp kernel: item chunk of each warp
    int x_vec;                 // x is 16-byte aligned: x segments load as double2
    const int32_t *units;      // SM-queue kernel: first item of each unit (+ end), see schedule.cu
    int local_parts;           // parts per group of a split tile row (Matrix::local_parts)
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
// 1-D TMA: global -> shared, completion counted on an mbarrier (bytes % 16 == 0)
__device__ __forceinline__ void bulk_g2s(uint32_t dst, const void *src, uint32_t bytes, uint32_t bar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
        "l"(src), "r"(bytes), "r"(bar)
        : "memory");
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

__device__ __forceinline__ int nib(const uint8_t *base, int idx) {
    return (base[idx >> 1] >> ((idx & 1) * 4)) & 15;
}

// ------------------------------------------------- one item's staged bytes --
// payload | tile descriptors | remRowPtr[16I..16I+rows] | remCol[kb..ke) | remVal[kb..ke)
// Each part is 16-byte aligned in shared memory; the unaligned arrays are
// copied as their enclosing 16-byte-aligned superset ("skew" = offset of the
// first wanted byte inside it).
struct ItemParts {
    uint32_t pay, dsc, rp, col, val, total;
    uint32_t dsc_skew, col_skew, val_skew;
};

// rows the item's remainder row pointers cover
__host__ __device__ __forceinline__ int64_t item_rows(const Item &it, int64_t m) {
    return imin64(it.ntr > 0 ? 16 * (int64_t)it.ntr : 16, m - 16 * (int64_t)it.I);
}

__host__ __device__ __forceinline__ ItemParts item_parts(const Item &it, int64_t m) {
    ItemParts r;
    r.pay = (it.offe - it.offb) * 16u;
    r.dsc_skew = (uint32_t)(it.dbeg & 1) * 8u;
    r.dsc = it.ndsc ? up16(r.dsc_skew + 8u * (uint32_t)it.ndsc) : 0u;
    if (it.ke > it.kb) {
        const int64_t rows = item_rows(it, m);
        r.rp = up16((uint32_t)(rows + 1) * 4u);
        r.col_skew = ((uint32_t)it.kb * 4u) & 15u;
        r.col = up16(r.col_skew + 4u * (uint32_t)(it.ke - it.kb));
        r.val_skew = ((uint32_t)it.kb * 8u) & 15u;
        r.val = up16(r.val_skew + 8u * (uint32_t)(it.ke - it.kb));
    } else {
        r.rp = r.col = r.val = r.col_skew = r.val_skew = 0u;
    }
    r.total = r.pay + r.dsc + r.rp + r.col + r.val;
    return r;
}

// ---------------------------------------------- one item's execution blob --
// A create-time copy of everything one work item reads, contiguous and
// 16-byte aligned part by part, so a single TMA bulk copy stages it:
//   dsc : the descriptor list (k_dsc_write), ndsc x 8 B
//   pay : the tiles' canonical payload bytes
//   rp  : remainder row pointers of the item's rows, rebased to the item's
//         entry range and clamped to it (rows + 1 ints)
//   col, val : the item's remainder entries
struct BlobParts {
    uint32_t pay, rp, col, val, total;
};

__host__ __device__ __forceinline__ BlobParts blob_parts(const Item &it, int64_t m) {
    BlobParts b;
    b.pay = up16(8u * (uint32_t)it.ndsc);
    b.rp = b.pay + (it.offe - it.offb) * 16u;
    if (it.ke > it.kb) {
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
__device__ __forceinline__ double2 ldg2_hint(const double *p, uint64_t policy) {
    double2 v;
    asm volatile("ld.global.nc.L2::cache_hint.v2.f64 {%0, %1}, [%2], %3;" : "=d"(v.x), "=d"(v.y) : "l"(p), "l"(policy));
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
__device__ __forceinline__ void cp_async_wait_all() {
    asm volatile("cp.async.commit_group;\n\tcp.async.wait_group 0;" ::: "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
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

// ----------------------------------------------------------- y output ------
// Lanes 0..15 hold the 16 row sums of the item.  A whole tile row writes y
// directly (one 128-byte store); a split tile row writes its partial and the
// last finishing part sums all parts in part order (deterministic).
__device__ __forceinline__ void write_rows(const Params &p, const Item &item, int lane, double acc) {
    const int64_t row = 16 * (int64_t)item.I + lane;
    if (item.split < 0) {
        if (lane < 16 && row < p.m) p.y[row] = acc;
        return;
    }
    const int2 si = p.split_info[item.split];
    const int part = item_part(item);
    if (lane < 16) __stcg(p.partials + (int64_t)(si.x + part) * 16 + lane, acc);
    __threadfence();
    __syncwarp();
    int old = 0;
    if (lane == 0) old = atomicAdd(p.counters + item.split, 1);
    old = __shfl_sync(FULL, old, 0);
    if (old == si.y - 1) {
        __threadfence();
        const int r = lane & 15, hh = lane >> 4;
        double s = 0.0;
        for (int q = hh; q < si.y; q += 2) s += __ldcg(p.partials + (int64_t)(si.x + q) * 16 + r);
        s += __shfl_xor_sync(FULL, s, 16);
        if (lane < 16 && row < p.m) p.y[row] = s;
        if (lane == 0) p.counters[item.split] = 0;  // ready for the next run
    }
}

// kernels (spmv_v1.cu, spmv_warp.cu)
struct KernelChoice {
    const char *name;
    void (*fn)(Params);
    int threads, smem, ctas_per_sm;
    bool ring;       // one CTA per SM with cta_begin chunks (no current kernel)
    int slot_bytes;  // item budget the schedule must respect
    bool pdl;        // launched with programmatic dependent launch (kernel waits on griddepcontrol)
    bool sm_queue;   // one CTA per SM; its warps claim units from a shared-memory counter
};
KernelChoice kernel_v1();
KernelChoice kernel_warp(int variant);

}  // namespace tsp
