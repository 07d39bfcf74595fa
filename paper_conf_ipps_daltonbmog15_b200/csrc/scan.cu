// scan.cu -- single-pass device-wide prefix sums (decoupled look-back).
//
// The method needs three scans: the row counts of C into
// C.row_offsets after SpAdd/SpGEMM symbolic ("space for C is allocated",
// P:820-822), and the SpGEMM product prefix S over the B row lengths
// referenced by A's columns (reading Z8: a flat int64 exclusive
// scan so that it can be binary-searched).  One pass: each CTA scans a
// 2048-item tile warp-striped (coalesced loads/stores), publishes its
// aggregate, and warp 0 looks back over its predecessors' published
// (flag, value) words to obtain the tile prefix.  Accumulation is int64.
#include "common.cuh"
#include "internal.h"

namespace msp {
namespace {

constexpr int SCAN_NT = 256;
#ifndef MSP_SCAN_ITEMS
#define MSP_SCAN_ITEMS 8  // 2,048-item tiles: C5 SpGEMM setup 14.9 -> 13.6 ms vs 16 (4-32 swept, profiles/r2/scan_items_sweep.txt)
#endif
constexpr int SCAN_ITEMS = MSP_SCAN_ITEMS;
constexpr int SCAN_TILE = SCAN_NT * SCAN_ITEMS;
constexpr unsigned long long FLAG_AGG = 1ull << 62;
constexpr unsigned long long FLAG_INC = 2ull << 62;
constexpr unsigned long long VAL_MASK = (1ull << 62) - 1;

struct LoadI32 {
    const int32_t *p;
    __device__ int64_t operator()(int64_t i) const { return p[i]; }
};
struct LoadI64 {
    const int64_t *p;
    __device__ int64_t operator()(int64_t i) const { return p[i]; }
};
struct LoadWidth {  // nnz of the B row referenced by A nonzero i
    const int32_t *acol, *brp;
    __device__ int64_t operator()(int64_t i) const
    {
        const int32_t k = acol[i];
        return int64_t(__ldg(brp + k + 1)) - __ldg(brp + k);
    }
};
struct LoadWidthStart {  // as LoadWidth, and records the B row start of A nonzero i
    const int32_t *acol, *brp;
    int32_t *bstart;
    __device__ int64_t operator()(int64_t i) const
    {
        const int32_t k = acol[i];
        const int32_t b0 = ldg64(brp + k);
        bstart[i] = b0;
        return int64_t(ldg64(brp + k + 1)) - b0;
    }
};
struct LoadNonEmpty {  // 1 if row i has nonzeros
    const int32_t *rp;
    __device__ int64_t operator()(int64_t i) const { return __ldg(rp + i + 1) > __ldg(rp + i) ? 1 : 0; }
};
struct StoreI64 {
    int64_t *p;
    __device__ void operator()(int64_t i, int64_t v) const { p[i] = v; }
};
struct StoreI32 {
    int32_t *p;
    __device__ void operator()(int64_t i, int64_t v) const { p[i] = int32_t(v); }
};

__device__ __forceinline__ unsigned long long ld_volatile(const unsigned long long *p)
{
    unsigned long long v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_volatile(unsigned long long *p, unsigned long long v)
{
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// EXCL: out(i) = sum_{k<i}, plus out(n) = total.  Otherwise out(i) = sum_{k<=i}.
template <class In, class Out, bool EXCL>
__global__ void __launch_bounds__(SCAN_NT)
scan_lookback(In in, Out out, int64_t n, unsigned long long *status, unsigned *tile_ctr, int64_t *total)
{
    __shared__ int tile_s;
    __shared__ int64_t warp_tot[SCAN_NT / 32];
    __shared__ int64_t tile_prefix_s;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    if (tid == 0) tile_s = int(atomicAdd(tile_ctr, 1u));
    __syncthreads();
    const int tile = tile_s;
    const int64_t base = int64_t(tile) * SCAN_TILE + int64_t(warp) * (32 * SCAN_ITEMS);

    int64_t v[SCAN_ITEMS], inc[SCAN_ITEMS];
#pragma unroll
    for (int k = 0; k < SCAN_ITEMS; ++k) {
        const int64_t i = base + k * 32 + lane;
        v[k] = (i < n) ? in(i) : 0;
    }
    int64_t acc = 0;
#pragma unroll
    for (int k = 0; k < SCAN_ITEMS; ++k) {
        const int64_t s = warp_inclusive_sum(v[k], lane);
        inc[k] = acc + s;
        acc += __shfl_sync(0xffffffffu, s, 31);
    }
    if (lane == 0) warp_tot[warp] = acc;
    __syncthreads();
    int64_t wpre = 0, agg = 0;
#pragma unroll
    for (int w = 0; w < SCAN_NT / 32; ++w) {
        if (w < warp) wpre += warp_tot[w];
        agg += warp_tot[w];
    }
    // ---- decoupled look-back (warp 0) ----
    if (warp == 0) {
        int64_t prefix = 0;
        if (tile == 0) {
            if (lane == 0) st_volatile(&status[0], FLAG_INC | (unsigned long long)agg);
        } else {
            if (lane == 0) st_volatile(&status[tile], FLAG_AGG | (unsigned long long)agg);
            int pos = tile - 1;  // look back window ends here
            while (true) {
                const int idx = pos - lane;
                unsigned long long w = 0;
                if (idx >= 0) {
                    do {
                        w = ld_volatile(&status[idx]);
                    } while ((w >> 62) == 0);
                } else {
                    w = FLAG_INC;  // virtual inclusive 0 before tile 0
                }
                const unsigned incmask = __ballot_sync(0xffffffffu, (w >> 62) == 2);
                // lanes up to (and including) the first inclusive one contribute
                const int stop = incmask ? (__ffs(incmask) - 1) : 32;
                int64_t contrib = (lane <= stop) ? int64_t(w & VAL_MASK) : 0;
#pragma unroll
                for (int o = 16; o > 0; o >>= 1) contrib += __shfl_xor_sync(0xffffffffu, contrib, o);
                prefix += contrib;
                if (incmask) break;
                pos -= 32;
            }
            if (lane == 0) st_volatile(&status[tile], FLAG_INC | (unsigned long long)(prefix + agg));
        }
        if (lane == 0) tile_prefix_s = prefix;
    }
    __syncthreads();
    const int64_t pre = tile_prefix_s + wpre;
#pragma unroll
    for (int k = 0; k < SCAN_ITEMS; ++k) {
        const int64_t i = base + k * 32 + lane;
        if (i < n) out(i, EXCL ? pre + inc[k] - v[k] : pre + inc[k]);
    }
    const int ntiles = int((n + SCAN_TILE - 1) / SCAN_TILE);
    if (tile == ntiles - 1 && tid == 0) {
        const int64_t t = tile_prefix_s + agg;
        if (total) *total = t;
        if (EXCL) out(n, t);
    }
}

__global__ void scan_empty(int64_t *total, int64_t *out0)
{
    if (total) *total = 0;
    if (out0) *out0 = 0;
}

template <class In, class Out, bool EXCL>
msp_status run_scan(In in, Out out, int64_t n, int64_t *total, int64_t *out0_if_empty, void *ws, size_t ws_bytes,
                    cudaStream_t s)
{
    if (n == 0) {
        scan_empty<<<1, 1, 0, s>>>(total, out0_if_empty);
        return last_launch("scan_empty");
    }
    const int64_t ntiles = ceil_div(n, SCAN_TILE);
    if (ntiles >= (int64_t(1) << 31)) return MSP_ERR_OVERFLOW;
    Carve cv(ws, ws_bytes);
    unsigned *ctr = cv.take<unsigned>(1);
    unsigned long long *status = cv.take<unsigned long long>(size_t(ntiles));
    if (!cv.ok()) return MSP_ERR_WORKSPACE;
    msp_status st = cuda_check(cudaMemsetAsync(ws, 0, cv.off, s), "scan: clear status");
    if (st != MSP_OK) return st;
    scan_lookback<In, Out, EXCL><<<unsigned(ntiles), SCAN_NT, 0, s>>>(in, out, n, status, ctr, total);
    return last_launch("scan_lookback");
}

}  // namespace

size_t scan_ws_bytes(int64_t n)
{
    return 512 + size_t(ceil_div(n > 0 ? n : 1, SCAN_TILE)) * 8 + 256;
}

msp_status scan_widths_to_S_bstart(const int32_t *Acol, const int32_t *Brp, int64_t nnzA, int64_t *S, int32_t *bstart,
                                   void *ws, size_t ws_bytes, cudaStream_t s)
{
    return run_scan<LoadWidthStart, StoreI64, true>(LoadWidthStart{Acol, Brp, bstart}, StoreI64{S}, nnzA, nullptr, S,
                                                    ws, ws_bytes, s);
}

msp_status scan_i32_to_i64(const int32_t *in, int64_t *out, int64_t n, void *ws, size_t ws_bytes, cudaStream_t s)
{
    return run_scan<LoadI32, StoreI64, true>(LoadI32{in}, StoreI64{out}, n, nullptr, out, ws, ws_bytes, s);
}

msp_status scan_counts_to_offsets_i32(int32_t *counts, int64_t n, int64_t *total_dev, void *ws, size_t ws_bytes,
                                      cudaStream_t s)
{
    // inclusive scan in place of counts[0..n) (the caller keeps offsets[0] = 0
    // just before `counts`); int64 accumulation, int32 store
    return run_scan<LoadI32, StoreI32, false>(LoadI32{counts}, StoreI32{counts}, n, total_dev, nullptr, ws,
                                              ws_bytes, s);
}

msp_status scan_i64_to_i64(const int64_t *in, int64_t *out, int64_t n, void *ws, size_t ws_bytes, cudaStream_t s)
{
    return run_scan<LoadI64, StoreI64, true>(LoadI64{in}, StoreI64{out}, n, nullptr, out, ws, ws_bytes, s);
}

msp_status scan_nonempty_rows(const int32_t *rp, int64_t m, int64_t *pos, void *ws, size_t ws_bytes, cudaStream_t s)
{
    return run_scan<LoadNonEmpty, StoreI64, true>(LoadNonEmpty{rp}, StoreI64{pos}, m, nullptr, pos, ws, ws_bytes, s);
}

msp_status scan_widths_to_S(const int32_t *Acol, const int32_t *Brp, int64_t nnzA, int64_t *S, void *ws,
                            size_t ws_bytes, cudaStream_t s)
{
    return run_scan<LoadWidth, StoreI64, true>(LoadWidth{Acol, Brp}, StoreI64{S}, nnzA, nullptr, S, ws, ws_bytes,
                                               s);
}

}  // namespace msp
