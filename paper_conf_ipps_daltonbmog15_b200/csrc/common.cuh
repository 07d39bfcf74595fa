// common.cuh -- device helpers shared by the libmsp kernels (sm_100a only).
//
// * mbarrier + cp.async.bulk (TMA bulk copy, SASS UBLKCP) wrappers used to
//   stage CSR tiles in shared memory;
// * L2 cache-policy creation (evict_first for the streamed col/val arrays);
// * warp / CTA scans (plain and segmented) used by the segmented reductions
//   of all three operations ("CTA wide segmented scan").
#pragma once

#include <cstdint>
#include <cuda_runtime.h>

#if defined(__CUDA_ARCH__) && (__CUDA_ARCH__ < 1000)
#error "libmsp is written for sm_100a (B200); compile with -gencode arch=compute_100a,code=sm_100a"
#endif

namespace msp {

constexpr int kWarp = 32;

__host__ __device__ __forceinline__ int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }

// ------------------------------------------------------------------ PTX ---

__device__ __forceinline__ uint32_t smem_u32(const void *p)
{
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count)
{
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}

__device__ __forceinline__ void fence_mbar_init()
{
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}

__device__ __forceinline__ void mbar_arrive(uint64_t *bar)
{
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t *bar, uint32_t bytes)
{
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
}

__device__ __forceinline__ bool mbar_try_wait(uint64_t *bar, uint32_t parity)
{
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(ok)
        : "r"(smem_u32(bar)), "r"(parity)
        : "memory");
    return ok != 0;
}

// try_wait with a suspend-time hint: the waiting thread sleeps until the
// phase completes (or the hint expires) instead of re-issuing the test.
__device__ __forceinline__ bool mbar_try_wait_sleep(uint64_t *bar, uint32_t parity)
{
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(ok)
        : "r"(smem_u32(bar)), "r"(parity), "r"(1000000u)
        : "memory");
    return ok != 0;
}

__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity)
{
    while (!mbar_try_wait_sleep(bar, parity)) {
    }
}

// Read-only random gathers with a 64-byte L2 fill: a miss fetches 64
// instead of 128 DRAM bytes (tools/probe/gather_probe.py).  Used for the
// SpGEMM B-row and B-offset gathers; MSP_L2_64B=0 (experiment builds) gives
// plain __ldg.
#ifndef MSP_L2_64B
#define MSP_L2_64B 1
#endif
__device__ __forceinline__ int32_t ldg64(const int32_t *p)
{
#if MSP_L2_64B
    int32_t v;
    asm("ld.global.nc.L2::64B.s32 %0, [%1];" : "=r"(v) : "l"(p));
    return v;
#else
    return __ldg(p);
#endif
}
__device__ __forceinline__ float ldg64(const float *p)
{
#if MSP_L2_64B
    float v;
    asm("ld.global.nc.L2::64B.f32 %0, [%1];" : "=f"(v) : "l"(p));
    return v;
#else
    return __ldg(p);
#endif
}
__device__ __forceinline__ double ldg64(const double *p)
{
#if MSP_L2_64B
    double v;
    asm("ld.global.nc.L2::64B.f64 %0, [%1];" : "=d"(v) : "l"(p));
    return v;
#else
    return __ldg(p);
#endif
}

__device__ __forceinline__ uint64_t policy_evict_first()
{
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}

// 1-D bulk copy global -> shared (TMA engine), completion counted on `bar`.
// dst, src 16-byte aligned; bytes a positive multiple of 16.
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, uint32_t bytes, uint64_t *bar,
                                         uint64_t policy)
{
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint"
        " [%0], [%1], %2, [%3], %4;" ::"r"(smem_u32(dst)),
        "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(policy)
        : "memory");
}

// Ampere-style asynchronous global -> shared copies (SASS LDGSTS): many
// element copies in flight per thread without a register round trip.
template <int BYTES>
__device__ __forceinline__ void cp_async(void *smem_dst, const void *gmem_src)
{
    static_assert(BYTES == 4 || BYTES == 8 || BYTES == 16, "cp.async size");
    asm volatile("cp.async.ca.shared.global [%0], [%1], %2;" ::"r"(smem_u32(smem_dst)), "l"(gmem_src), "n"(BYTES)
                 : "memory");
}

__device__ __forceinline__ void cp_async_wait_all()
{
    asm volatile("cp.async.commit_group;\n\tcp.async.wait_group 0;" ::: "memory");
}

__device__ __forceinline__ void named_bar_sync(int id, int nthreads)
{
    asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}

// Plan of a TMA window copy of elements [lo, hi) of an array of `len`
// elements: each element keeps its address mod 16 in shared memory.  The
// window is widened to 16-byte boundaries (re-reading a few neighbouring
// elements of the same array is harmless) so that it normally goes through
// ONE bulk copy; only where widening would leave the array (a misaligned
// base, or the array's last bytes) are up to 15 bytes copied by hand.
struct WindowCopy {
    const char *bulk_src;  // null if no bulk part
    uint32_t bulk_bytes;
    uint32_t bulk_dst;     // byte offset from the window base
    uint32_t first;        // byte offset of element lo from the window base
    uint32_t head_elems;   // elements copied by hand at the head
    uint32_t tail_elems;   // ... and at the tail
    uint32_t span;         // bytes of window used (multiple of 16)
};

template <int ES>
__device__ __forceinline__ WindowCopy plan_window(const void *base, int64_t lo, int64_t hi, int64_t len)
{
    WindowCopy w;
    const uintptr_t b0 = reinterpret_cast<uintptr_t>(base);
    const uintptr_t s = b0 + uintptr_t(lo) * ES;
    const uintptr_t e = b0 + uintptr_t(hi) * ES;
    const uintptr_t end = b0 + uintptr_t(len) * ES;
    const uintptr_t a_lo = s & ~uintptr_t(15);
    w.first = uint32_t(s - a_lo);
    w.head_elems = 0;
    w.tail_elems = 0;
    if (hi <= lo) {
        w.bulk_src = nullptr; w.bulk_bytes = 0; w.bulk_dst = 0; w.span = 16;
        return w;
    }
    uintptr_t b_lo = a_lo, b_hi = (e + 15) & ~uintptr_t(15);
    if (b_lo < b0) {  // misaligned base: hand-copy up to the first aligned element
        b_lo = (s + 15) & ~uintptr_t(15);
        w.head_elems = uint32_t((b_lo < e ? b_lo - s : e - s) / ES);
    }
    if (b_hi > end) {  // array end: hand-copy the last partial 16 bytes
        b_hi = e & ~uintptr_t(15);
        if (b_hi < b_lo) b_hi = b_lo;
        w.tail_elems = uint32_t((e - (b_hi > s ? b_hi : s)) / ES) ;
        if (w.head_elems && b_hi <= b_lo) w.tail_elems = 0;  // head already covers [lo, hi)
    }
    if (b_hi > b_lo) {
        w.bulk_src = reinterpret_cast<const char *>(b_lo);
        w.bulk_bytes = uint32_t(b_hi - b_lo);
        w.bulk_dst = uint32_t(b_lo - a_lo);
    } else {
        w.bulk_src = nullptr; w.bulk_bytes = 0; w.bulk_dst = 0;
    }
    w.span = uint32_t((((e + 15) & ~uintptr_t(15)) - a_lo));
    return w;
}

// Hand-copy the ragged ends of a planned window; lane `l` copies manual
// element l (if any).  Returns the number of manual elements.
template <typename T>
__device__ __forceinline__ void window_manual(const WindowCopy &w, const T *base, int64_t lo, int64_t hi,
                                              char *dst_window, int lane_slot)
{
    const int nh = int(w.head_elems), nt = int(w.tail_elems);
    if (lane_slot < nh) {
        const int64_t e = lo + lane_slot;
        *reinterpret_cast<T *>(dst_window + w.first + size_t(lane_slot) * sizeof(T)) = base[e];
    } else if (lane_slot < nh + nt) {
        const int64_t e = hi - nt + (lane_slot - nh);
        *reinterpret_cast<T *>(dst_window + w.first + size_t(e - lo) * sizeof(T)) = base[e];
    }
}

// ------------------------------------------------------------ scans ------

template <typename T>
__device__ __forceinline__ T warp_inclusive_sum(T v, int lane)
{
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        T u = __shfl_up_sync(0xffffffffu, v, o);
        if (lane >= o) v = u + v;
    }
    return v;
}

// Segmented inclusive scan of (flag, value): flag marks "a segment starts
// inside this element's range" so earlier values are dropped.  Combining
// order is always earlier + later (deterministic).
template <typename T>
struct SegPair {
    int f;
    T v;
};

template <typename T>
__device__ __forceinline__ SegPair<T> seg_combine(SegPair<T> a, SegPair<T> b)
{
    SegPair<T> r;
    r.f = a.f | b.f;
    r.v = b.f ? b.v : (a.v + b.v);
    return r;
}

template <typename T>
__device__ __forceinline__ SegPair<T> warp_seg_inclusive(SegPair<T> x, int lane)
{
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        int uf = __shfl_up_sync(0xffffffffu, x.f, o);
        T uv = __shfl_up_sync(0xffffffffu, x.v, o);
        if (lane >= o) {
            if (!x.f) x.v = uv + x.v;
            x.f |= uf;
        }
    }
    return x;
}

// CTA-wide exclusive segmented scan over NW warps (all threads of the group
// must call; uses a named barrier `bar_id` over NW*32 threads).  `prefix` is
// combined in front of thread 0.  Returns this thread's exclusive value and
// writes the group total to *total.
template <typename T, int NW>
__device__ __forceinline__ SegPair<T> block_seg_exclusive(SegPair<T> x, SegPair<T> prefix, SegPair<T> *smem_w,
                                                          int bar_id, SegPair<T> *total)
{
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    SegPair<T> inc = warp_seg_inclusive(x, lane);
    if (lane == 31) smem_w[warp] = inc;
    named_bar_sync(bar_id, NW * 32);
    // prefix of the warps before this one
    SegPair<T> wp = prefix;
    for (int w = 0; w < warp; ++w) wp = seg_combine(wp, smem_w[w]);
    SegPair<T> tot = wp;
    for (int w = warp; w < NW; ++w) tot = seg_combine(tot, smem_w[w]);
    *total = tot;
    SegPair<T> ex;
    ex.f = __shfl_up_sync(0xffffffffu, inc.f, 1);
    ex.v = __shfl_up_sync(0xffffffffu, inc.v, 1);
    SegPair<T> r = (lane == 0) ? wp : seg_combine(wp, ex);
    named_bar_sync(bar_id, NW * 32);  // smem_w reusable afterwards
    return r;
}

// Plain CTA-wide exclusive sum over NW warps (named barrier).
template <typename T, int NW>
__device__ __forceinline__ T block_exclusive_sum(T v, T *smem_w, int bar_id, T *total)
{
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    T inc = warp_inclusive_sum(v, lane);
    if (lane == 31) smem_w[warp] = inc;
    named_bar_sync(bar_id, NW * 32);
    T wp = T(0), tot = T(0);
#pragma unroll
    for (int w = 0; w < NW; ++w) {
        T s = smem_w[w];
        if (w < warp) wp += s;
        tot += s;
    }
    *total = tot;
    T ex = __shfl_up_sync(0xffffffffu, inc, 1);
    named_bar_sync(bar_id, NW * 32);
    return lane == 0 ? wp : wp + ex;
}

// CTA-wide exclusive max over NW warps (named barrier); -1 before thread 0.
template <int NW>
__device__ __forceinline__ int block_exclusive_max(int v, int *smem_w, int bar_id)
{
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    int inc = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int u = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane >= o) inc = max(inc, u);
    }
    if (lane == 31) smem_w[warp] = inc;
    named_bar_sync(bar_id, NW * 32);
    int wp = -1;
#pragma unroll
    for (int w = 0; w < NW; ++w)
        if (w < warp) wp = max(wp, smem_w[w]);
    const int ex = __shfl_up_sync(0xffffffffu, inc, 1);
    named_bar_sync(bar_id, NW * 32);
    return lane == 0 ? wp : max(wp, ex);
}

}  // namespace msp
