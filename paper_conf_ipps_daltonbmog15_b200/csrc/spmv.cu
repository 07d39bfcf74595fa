// spmv.cu -- merge-path SpMV y = A x for sm_100a.
//
// Paper: Section III-A.  The paper splits SpMV into three phases:
//   partition  one binary search per CTA over row_offsets,
//   reduction  load col/val, gather x, CTA segmented scan, write
//                           y at row discontinuities, carry the remainder,
//   update  add each CTA's carry to the next CTA's first row.
// B200 design: ONE persistent launch.
//   * The merge grid is the 2-D one of the north star (BJ:5): list A =
//     row_end = rp[1..m], list B = nonzero indices; row end r is consumed
//     before nonzero j iff rp[r+1] <= j.  CTA b owns the contiguous diagonal
//     range [b*total/G, (b+1)*total/G) (equal share of rows + nonzeros) and
//     walks it in tiles of T = NT*K items.
//   * Warp NT/32 is a producer: a 32-ary warp-cooperative diagonal search
//     (one ballot per round) finds each tile's end split, then one lane
//     issues TMA bulk copies (cp.async.bulk, L2 evict_first for col/val) of
//     the tile's row_end window, col window and val window into a STAGES-deep
//     shared-memory ring guarded by mbarriers.  No separate partition launch.
//   * NT consumer threads: phase A reads col/val coalesced from shared
//     memory, gathers x and writes the fp64 products to a swizzled product
//     buffer ("dereference entries from x ... scaled products");
//     phase B gives each thread K consecutive products (conflict-free 16-byte
//     reads through the XOR swizzle), reduces them by row against the staged
//     row_end window, and a CTA segmented scan supplies each
//     thread's carry-in.  Empty rows are zero-filled from the row_end window
//     (reading Z6), so the grid needs no compaction path.
//   * Carries between tiles of one CTA stay in registers; each CTA leaves one
//     (row, partial) carry plus the fp64 value of its first emitted row in the
//     workspace and the last CTA to finish applies them in CTA order (the
//     update phase with row ids, reading Z21) -- one rounding per y entry.
//   * fp32 inputs are promoted and accumulated in fp64 (reading Z4).
#include <climits>
#include <cstdio>
#include <cstdlib>
#include <algorithm>
#include <cmath>
#include <type_traits>

#include "common.cuh"
#include "internal.h"

#ifdef MSP_SPMV_TRACE
// Timeline instrumentation (experiment builds only): clock64 stamps per
// (CTA < 4, tile < 64, slot < 16), relative to the CTA's start.
__device__ long long g_spmv_trace[4][64][16];
extern "C" int msp_debug_spmv_trace(void *host)
{
    return int(cudaMemcpyFromSymbol(host, g_spmv_trace, sizeof(g_spmv_trace)));
}
#define TR(t, slot)                                                                                   \
    do {                                                                                              \
        if (blockIdx.x < 4 && (t) < 64) g_spmv_trace[blockIdx.x][(t)][(slot)] = clock64() - tr_t0;    \
    } while (0)
#else
#define TR(t, slot) \
    do {            \
    } while (0)
#endif

namespace msp {
namespace {

__device__ __forceinline__ int64_t max64(int64_t a, int64_t b) { return a > b ? a : b; }
__device__ __forceinline__ int64_t min64(int64_t a, int64_t b) { return a < b ? a : b; }

struct TileMeta {
    int32_t i_s, i_e, wr_end;  // rows [i_s, i_e) end in the tile; window rows [i_s, wr_end)
    int32_t j_s, j_e;          // nonzeros [j_s, j_e)
    uint32_t rp_first, col_first, val_first;  // byte offsets inside the stage
};

struct CtaRecord {  // one per CTA in the workspace
    int32_t carry_key;   // row holding the CTA's trailing partial (-1: none)
    int32_t head_row;    // first row emitted by this CTA (-1: none)
    double carry_val;    // trailing partial (fp64)
    double head_val;     // fp64 value written for head_row (before carries)
};

// NW worker warps of 32 lanes x K = 8 products each (one tile = NW * 256
// merge items), plus one producer warp and one row warp.
template <typename V, int NW_, int STAGES_, int RSLOTS_, int MINB_, bool EARLY_ = false, bool L1G_ = false>
struct Cfg {
    static constexpr bool ROWK = false;
    // L1G: x gathers allocate in L1 (ld.global.nc.L2::64B): R-MAT hub columns
    // are reused (C3 419 -> 407 us); else L2 only (ld.global.cg.L2::64B)
    static constexpr bool L1G = L1G_;
    // EARLY: a worker issues tile t+1's x gathers right after forming tile
    // t's products (they fly during t's walk, scan and look-back) instead of
    // after the walk
    static constexpr bool EARLY = EARLY_;
    static constexpr int NW = NW_;
    static constexpr int K = 8;
    static constexpr int WSPAN = 32 * K;                 // products per worker warp
    static constexpr int T = NW * WSPAN;                 // merge items (rows + nonzeros) per tile
    static constexpr int STAGES = STAGES_;
    static constexpr int MINB = MINB_;
    static constexpr int THREADS = (NW + 2) * 32;
    static constexpr int RING = 8;  // per-tile carry slots (power of 2; workers are in lockstep, skew <= 2 tiles)
    static constexpr int DATA_BYTES = int(((4 + sizeof(V)) * T + 64 + 15) / 16 * 16);  // rp, col, val windows
    static constexpr int FW = T / 32;                    // flag words per tile
    static constexpr int FLAG_BYTES = FW * 4;            // row-end bit per position
    static constexpr int RMAP_BYTES = T * 2;             // row (tile-relative, +1) ending at a position
    static constexpr int STAGE_BYTES = DATA_BYTES;       // TMA ring: released after phase A
    static constexpr int RSLOTS = RSLOTS_;               // row-map ring: released after the walk
    static constexpr int RSLOT_BYTES = FLAG_BYTES + RMAP_BYTES;
    static constexpr int PROD_BYTES = NW * WSPAN * 8;    // warp-private product buffers
    static constexpr int MISC_BYTES = 2048;
    static constexpr int SMEM = STAGES * STAGE_BYTES + RSLOTS * RSLOT_BYTES + PROD_BYTES + MISC_BYTES;
};

// Row-aligned variant (reading R2): every lane owns K
// consecutive products of the tile, K chosen per matrix from its mean row
// length (odd, so the lane-strided shared-memory reads of col/val are bank
// conflict free).  The products stay in registers (no transpose buffer), and
// when rows are about K long, gather u of the 32 lanes touches the same
// stencil position of 32 consecutive rows -- a few x cache lines per
// instruction instead of one per row.
template <typename V, int NW_, int K_, int STAGES_, int MINB_>
struct CfgK {
    static constexpr bool ROWK = true;
    static constexpr int NW = NW_;
    static constexpr int K = K_;
    static constexpr int WSPAN = 32 * K;
    static constexpr int T = NW * WSPAN;
    static constexpr int STAGES = STAGES_;
    static constexpr int MINB = MINB_;
    static constexpr int THREADS = (NW + 2) * 32;
    static constexpr int RING = 8;
    static constexpr int DATA_BYTES = int(((4 + sizeof(V)) * T + 64 + 15) / 16 * 16);
    static constexpr int FW = 1;
    static constexpr int STAGE_BYTES = DATA_BYTES;
    static constexpr int RSLOTS = 0;                     // no shared row map: each worker maps its own span
    static constexpr int RSLOT_BYTES = 0;
    // per worker warp: 32 lane masks of row-end bits + the tile-relative row
    // id at every row-end position of its span (WSPAN 16-bit entries)
    static constexpr int WMAP_BYTES = (32 * 4 + WSPAN * 2 + 15) / 16 * 16;
    static constexpr int PROD_BYTES = NW * WMAP_BYTES;
    static constexpr int MISC_BYTES = 2048;
    static constexpr int SMEM = STAGES * STAGE_BYTES + PROD_BYTES + MISC_BYTES;
    static constexpr bool EARLY = false;
    static_assert(K % 2 == 1 && K < 32, "K odd and < 32");
};

__device__ __forceinline__ int ld_volatile_s(const int *p) { return *reinterpret_cast<const volatile int *>(p); }
__device__ __forceinline__ void st_volatile_s(int *p, int v) { *reinterpret_cast<volatile int *>(p) = v; }

// 32-ary warp search on the CSR merge grid: smallest i in [lo, hi] with
// NOT(rp[i+1] <= d - i - 1) (i.e. the number of row ends consumed before
// diagonal d).  All lanes return the same value.
__device__ __forceinline__ int warp_grid_search(const int32_t *__restrict__ rp, int64_t d, int lo, int hi,
                                                int lane)
{
    while (hi - lo > 32) {
        const int64_t len = int64_t(hi) - lo;
        const int64_t step = (len + 31) / 32;
        const int64_t p = int64_t(lo) + (lane + 1) * step - 1;
        bool pred = false;
        if (p < hi) pred = int64_t(__ldg(rp + p + 1)) <= d - p - 1;
        const unsigned bal = __ballot_sync(0xffffffffu, pred);
        const int c = __popc(bal);
        const int64_t nlo = int64_t(lo) + int64_t(c) * step;
        const int64_t pc = int64_t(lo) + int64_t(c + 1) * step - 1;
        int nhi = hi;
        if (c < 32 && pc < hi) nhi = int(pc);
        lo = int(nlo);
        hi = nhi;
    }
    const int64_t p = int64_t(lo) + lane;
    bool pred = false;
    if (p < hi) pred = int64_t(__ldg(rp + p + 1)) <= d - p - 1;
    return lo + __popc(__ballot_sync(0xffffffffu, pred));
}

// x gathers as volatile asm: issued in program order ahead of the row-map
// wait (plain __ldg loads are sunk past it by the compiler, serialising each
// gather's latency with the multiply-add that uses it).
__device__ __forceinline__ double ldg_x(const double *p)
{
    double v;
    asm volatile("ld.global.f64 %0, [%1];" : "=d"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ double ldg_x(const float *p)
{
    float v;
    asm volatile("ld.global.f32 %0, [%1];" : "=f"(v) : "l"(p) : "memory");
    return double(v);
}

// x gather of the transpose walk: ld.global.cg.L2::64B -- L2 only (no L1
// line allocation: the walk serves irregular matrices, whose gathers rarely
// reuse an L1 line; 3-7 % faster than __ldg on C3/C4/C5), and a 64-byte
// L2 fill instead of the 128-byte line an L1 miss requests by default: a
// random 8-byte gather from a DRAM-resident x then costs 65 instead of
// 121 DRAM bytes (tools/probe/gather_probe.py; C5 13.0 -> 12.7 ms).
// (profiles/r2/spmv_irregular_shapes.txt)  Experiment builds:
// -DMSP_SPMV_GATHER=0 -> __ldg, 1 -> ld.global.cg, 2 -> ld.global.cs.
#ifndef MSP_SPMV_GATHER
#define MSP_SPMV_GATHER 3
#endif
template <typename T, bool L1G = false>
__device__ __forceinline__ T gather_x(const T *p)
{
    if constexpr (L1G) {
        T v;
        if constexpr (sizeof(T) == 8) {
            double d;
            asm volatile("ld.global.nc.L2::64B.f64 %0, [%1];" : "=d"(d) : "l"(p));
            v = T(d);
        } else {
            float f;
            asm volatile("ld.global.nc.L2::64B.f32 %0, [%1];" : "=f"(f) : "l"(p));
            v = T(f);
        }
        return v;
    }
#if MSP_SPMV_GATHER == 1
    return __ldcg(p);
#elif MSP_SPMV_GATHER == 2
    return __ldcs(p);
#elif MSP_SPMV_GATHER == 4
    T v;
    if constexpr (sizeof(T) == 8) {
        double d;
        asm volatile("ld.global.nc.L2::64B.f64 %0, [%1];" : "=d"(d) : "l"(p));
        v = T(d);
    } else {
        float f;
        asm volatile("ld.global.nc.L2::64B.f32 %0, [%1];" : "=f"(f) : "l"(p));
        v = T(f);
    }
    return v;
#elif MSP_SPMV_GATHER == 3
    T v;
    if constexpr (sizeof(T) == 8) {
        double d;
        asm volatile("ld.global.cg.L2::64B.f64 %0, [%1];" : "=d"(d) : "l"(p));
        v = T(d);
    } else {
        float f;
        asm volatile("ld.global.cg.L2::64B.f32 %0, [%1];" : "=f"(f) : "l"(p));
        v = T(f);
    }
    return v;
#else
    return __ldg(p);
#endif
}

// Predicated global store (keeps the walk straight-line code).
__device__ __forceinline__ void st_global_if(double *p, double v, bool pred)
{
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %2, 0;\n\t@p st.global.f64 [%0], %1;\n\t}" ::"l"(p), "d"(v),
                 "r"(int(pred)));
}
__device__ __forceinline__ void st_global_if(float *p, float v, bool pred)
{
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %2, 0;\n\t@p st.global.f32 [%0], %1;\n\t}" ::"l"(p), "f"(v),
                 "r"(int(pred)));
}

// The producer's wait for a free stage.  MSP_SPMV_PROD_SPIN=1 (experiment
// builds): a plain try_wait spin instead of the suspend-hinted wait.
#ifndef MSP_SPMV_PROD_SPIN
#define MSP_SPMV_PROD_SPIN 0
#endif
__device__ __forceinline__ void mbar_wait_backoff(uint64_t *bar, uint32_t parity)
{
#if MSP_SPMV_PROD_SPIN
    while (!mbar_try_wait(bar, parity)) {
    }
#else
    mbar_wait(bar, parity);
#endif
}

// Split search with a guess: probe the 32 consecutive rows around `g` first
// (one ballot round when the tile has about as many rows as the last one),
// and fall back to the 32-ary search on the remaining range.
__device__ __forceinline__ int warp_grid_search_guess(const int32_t *__restrict__ rp, int64_t d, int lo, int hi,
                                                      int g, int lane)
{
    if (hi - lo <= 32) return warp_grid_search(rp, d, lo, hi, lane);
    int base = g - 16;
    base = max(lo, min(base, hi - 32));
    const int64_t p = int64_t(base) + lane;
    const bool pred = int64_t(__ldg(rp + p + 1)) <= d - p - 1;
    const int c = __popc(__ballot_sync(0xffffffffu, pred));
    if (c > 0 && c < 32) return base + c;
    if (c == 0) return (base == lo) ? lo : warp_grid_search(rp, d, lo, base, lane);
    return warp_grid_search(rp, d, base + 32, hi, lane);
}

// Product buffer layout: logical position q (one fp64 product) lives in
// 16-byte chunk c = q/2 at physical chunk c ^ ((c >> 3) & (K/2 - 1)), so that
// both the strided writes of phase A and the K-consecutive reads of the walk
// are bank-conflict free.
template <int K>
__device__ __forceinline__ int swz(int q)
{
    const int c = q >> 1;
    return ((c ^ ((c >> 3) & (K / 2 - 1))) << 1) | (q & 1);
}

template <typename V, class C>
__global__ void __launch_bounds__(C::THREADS, C::MINB)
spmv_merge_kernel(int32_t m, int64_t nnz, const int32_t *__restrict__ rp, const int32_t *__restrict__ col,
                  const V *__restrict__ val, const V *__restrict__ x, V *__restrict__ y, int32_t n_cols,
                  CtaRecord *__restrict__ recs, unsigned *__restrict__ counter)
{
    constexpr int K = C::K, NW = C::NW, WSPAN = C::WSPAN, RING = C::RING;
    constexpr int FW = C::FW;
    extern __shared__ __align__(128) char smem[];
    char *stages = smem;
    char *rslots = smem + C::STAGES * C::STAGE_BYTES;                   // [RSLOTS] flags + row map
    double *prodbuf = reinterpret_cast<double *>(rslots + C::RSLOTS * C::RSLOT_BYTES);  // [NW][WSPAN]
    char *prodbuf_raw = reinterpret_cast<char *>(prodbuf);  // row-aligned variant: [NW] warp row maps
    char *misc = reinterpret_cast<char *>(prodbuf) + C::PROD_BYTES;
    uint64_t *full = reinterpret_cast<uint64_t *>(misc);               // [STAGES] TMA landed
    uint64_t *empty = full + C::STAGES;                                // [STAGES] stage free
    uint64_t *rowsrdy = empty + C::STAGES;                             // [RSLOTS] row map built
    uint64_t *rowsfree = rowsrdy + C::RSLOTS;                          // [RSLOTS] row map consumed
    TileMeta *meta = reinterpret_cast<TileMeta *>(rowsfree + C::RSLOTS);  // [STAGES]
    double *agg_v = reinterpret_cast<double *>(meta + C::STAGES);     // [RING][NW] warp trailing sums
    double *cta_v = agg_v + RING * NW;                                 // [RING] carry leaving each tile
    int *agg_f = reinterpret_cast<int *>(cta_v + RING);                // [RING][NW] warp had a row end
    int *agg_seq = agg_f + RING * NW;                                  // [RING][NW] tile tag (t+1) once published
    int *cta_f = agg_seq + RING * NW;                                  // [RING]
    int *cta_seq = cta_f + RING;                                       // [RING] tile tag once cta_v/f valid
    int *pub_cnt = cta_seq + RING;                                     // [RING] warps published
    __shared__ int s_carry_key, s_head_row, s_last;
    __shared__ double s_head_val;

    const int tid = threadIdx.x;
    const int lane = tid & 31;
    const int warp = tid >> 5;
    const int G = gridDim.x;
    const int64_t total = int64_t(m) + nnz;
#ifdef MSP_SPMV_TRACE
    const long long tr_t0 = clock64();
#endif
    const int64_t d_begin = int64_t(blockIdx.x) * total / G;
    const int64_t d_end = int64_t(blockIdx.x + 1) * total / G;
    const int ntiles = int((d_end - d_begin + C::T - 1) / C::T);

    if (tid == 0) {
        for (int s = 0; s < C::STAGES; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], NW + 1);
        }
        for (int s = 0; s < C::RSLOTS; ++s) {
            mbar_init(&rowsrdy[s], 1);
            mbar_init(&rowsfree[s], NW);
        }
        fence_mbar_init();
        s_carry_key = -1;
        s_head_row = -1;
        s_head_val = 0.0;
    }
    for (int i = tid; i < RING * NW; i += blockDim.x) agg_seq[i] = 0;
    for (int i = tid; i < RING; i += blockDim.x) {
        cta_seq[i] = 0;
        pub_cnt[i] = 0;
    }
    __syncthreads();

    if (warp == NW) {
        // ============================ producer warp ============================
        const uint64_t pol = policy_evict_first();
        int i_s = warp_grid_search(rp, d_begin, int(max64(0, d_begin - nnz)), int(min64(d_begin, m)), lane);
        int j_s = int(d_begin - i_s);
        int prev_rows = 0;
        for (int t = 0; t < ntiles; ++t) {
            const int stage = t % C::STAGES;
            const int64_t de = min64(d_begin + int64_t(t + 1) * C::T, d_end);
            const int lo = int(max64(i_s, de - nnz));
            const int hi = int(min64(m, de - j_s));
            const int i_e = warp_grid_search_guess(rp, de, lo, hi, i_s + prev_rows, lane);
            const int j_e = int(de - i_e);
            prev_rows = i_e - i_s;
            if (lane == 0) TR(t, 0);  // split searched
            if (t >= C::STAGES) mbar_wait_backoff(&empty[stage], ((t / C::STAGES) - 1) & 1);
            if (lane == 0) TR(t, 1);  // stage free: TMA issued
            char *sb = stages + size_t(stage) * C::STAGE_BYTES;
            const int wr_end = min(i_e + 1, m);
            // windows: rp[i_s .. wr_end] (inclusive), col/val[j_s .. j_e)
            const WindowCopy wr = plan_window<4>(rp, i_s, int64_t(wr_end) + 1, int64_t(m) + 1);
            const WindowCopy wc = plan_window<4>(col, j_s, j_e, nnz);
            const WindowCopy wv = plan_window<int(sizeof(V))>(val, j_s, j_e, nnz);
            const uint32_t off_r = 0, off_c = wr.span, off_v = wr.span + wc.span;
            const int nr = int(wr.head_elems + wr.tail_elems);
            const int nc = int(wc.head_elems + wc.tail_elems);
            const int nv = int(wv.head_elems + wv.tail_elems);
            if (nr + nc + nv) {  // rare: misaligned base or the arrays' last bytes
                if (lane < nr) window_manual<int32_t>(wr, rp, i_s, int64_t(wr_end) + 1, sb + off_r, lane);
                else if (lane < nr + nc) window_manual<int32_t>(wc, col, j_s, j_e, sb + off_c, lane - nr);
                else if (lane < nr + nc + nv) window_manual<V>(wv, val, j_s, j_e, sb + off_v, lane - nr - nc);
                __syncwarp();
            }
            if (lane == 0) {
                TileMeta &mt = meta[stage];
                mt.i_s = i_s; mt.i_e = i_e; mt.wr_end = wr_end;
                mt.j_s = j_s; mt.j_e = j_e;
                mt.rp_first = off_r + wr.first;
                mt.col_first = off_c + wc.first;
                mt.val_first = off_v + wv.first;
                mbar_arrive_expect_tx(&full[stage], wr.bulk_bytes + wc.bulk_bytes + wv.bulk_bytes);
                if (wr.bulk_bytes) bulk_g2s(sb + off_r + wr.bulk_dst, wr.bulk_src, wr.bulk_bytes, &full[stage], 0);
                if (wc.bulk_bytes) bulk_g2s(sb + off_c + wc.bulk_dst, wc.bulk_src, wc.bulk_bytes, &full[stage], pol);
                if (wv.bulk_bytes) bulk_g2s(sb + off_v + wv.bulk_dst, wv.bulk_src, wv.bulk_bytes, &full[stage], pol);
            }
            i_s = i_e;
            j_s = j_e;
        }
    } else if (warp == NW + 1) {
        // ============================ row warp =================================
        // Per tile: a row-end bit and the (tile-relative) row id at the
        // position of every nonempty row's last nonzero; empty rows whose
        // row-end item lies in the tile get y = +0.0 (Z6); the row holding the
        // tile's last nonzero is the CTA carry key.
        if constexpr (C::ROWK) {
            // row-aligned workers map their own spans' row ends: this warp only
            // zero-fills the tile's empty rows (Z6) and tracks the carry key
            for (int t = 0; t < ntiles; ++t) {
                const int stage = t % C::STAGES;
                mbar_wait(&full[stage], (t / C::STAGES) & 1);
                if (lane == 0) TR(t, 2);  // landed (row warp)
                const TileMeta mt = meta[stage];
                const int32_t *rps = reinterpret_cast<const int32_t *>(stages + size_t(stage) * C::STAGE_BYTES +
                                                                       mt.rp_first);
                const int z = mt.j_e - mt.j_s, i_s = mt.i_s, j_s = mt.j_s;
                for (int r = i_s + lane; r < mt.wr_end; r += 32) {
                    const int a = rps[r - i_s] - j_s;
                    const int b = rps[r - i_s + 1] - j_s;
                    if (a == b) {
                        if (r < mt.i_e) y[r] = V(0);
                    } else if (z > 0 && a < z && b >= z) {
                        s_carry_key = (b > z) ? r : -1;
                    }
                }
                __syncwarp();
                if (lane == 0) {
                    TR(t, 3);
                    mbar_arrive(&empty[stage]);  // this warp no longer reads the stage
                }
            }
        } else
        for (int t = 0; t < ntiles; ++t) {
            const int stage = t % C::STAGES;
            const int rs = t % C::RSLOTS;
            mbar_wait(&full[stage], (t / C::STAGES) & 1);
            if (lane == 0) TR(t, 2);  // landed (row warp)
            if (t >= C::RSLOTS) mbar_wait(&rowsfree[rs], ((t / C::RSLOTS) - 1) & 1);
            const TileMeta mt = meta[stage];
            char *sb = stages + size_t(stage) * C::STAGE_BYTES;
            const int32_t *rps = reinterpret_cast<const int32_t *>(sb + mt.rp_first);  // rps[r - i_s] = rp[r]
            uint32_t *flags = reinterpret_cast<uint32_t *>(rslots + size_t(rs) * C::RSLOT_BYTES);
            uint16_t *rmap = reinterpret_cast<uint16_t *>(rslots + size_t(rs) * C::RSLOT_BYTES + C::FLAG_BYTES);
            const int z = mt.j_e - mt.j_s, i_s = mt.i_s, j_s = mt.j_s;
            for (int i = lane; i < FW; i += 32) flags[i] = 0u;
            __syncwarp();
            {
#pragma unroll 4
                for (int r = i_s + lane; r < mt.wr_end; r += 32) {
                    const int a = rps[r - i_s] - j_s;
                    const int b = rps[r - i_s + 1] - j_s;
                    if (a == b) {
                        if (r < mt.i_e) y[r] = V(0);
                    } else {
                        if (b > 0 && b <= z) {
                            rmap[b - 1] = uint16_t(r - i_s + 1);
                            atomicOr(&flags[(b - 1) >> 5], 1u << ((b - 1) & 31));
                        }
                        if (z > 0 && a < z && b >= z) s_carry_key = (b > z) ? r : -1;
                    }
                }
            }
            __syncwarp();
            if (lane == 0) {
                TR(t, 3);  // row map built
                mbar_arrive(&rowsrdy[rs]);
                mbar_arrive(&empty[stage]);  // this warp no longer reads the stage
            }
        }
    } else if constexpr (C::ROWK) {
        // ===================== worker warps (row-aligned) =====================
        // Lane l of worker `warp` owns products [q0, q0 + K), q0 = warp*32K +
        // l*K, of every tile: it gathers their x entries (K loads in flight),
        // then walks them in order -- fp64 multiply-add into a running sum,
        // y written at each row end (its first row end waits for the carry of
        // earlier lanes); the warp segmented scan and the look-back across
        // warps / tiles are the same as in the transpose variant below.
        const int q0 = warp * WSPAN + lane * K;
        const int sp0 = warp * WSPAN;  // the warp's span of tile positions [sp0, sp0 + WSPAN)
        uint32_t *wmask = reinterpret_cast<uint32_t *>(prodbuf_raw + size_t(warp) * C::WMAP_BYTES);  // [32]
        uint16_t *wrow = reinterpret_cast<uint16_t *>(wmask + 32);  // [WSPAN] tile-relative row per row end
        auto finish_first = [&](int r, double v0, int tt) {
            const int sl = tt & (RING - 1);
            double c = 0.0;
            int f = 0;
            for (int w2 = warp - 1; w2 >= 0 && !f; --w2) {
                while (ld_volatile_s(&agg_seq[sl * NW + w2]) != tt + 1) {}
                __threadfence_block();
                c = reinterpret_cast<volatile double *>(agg_v)[sl * NW + w2] + c;
                f = reinterpret_cast<volatile int *>(agg_f)[sl * NW + w2];
            }
            if (!f && tt > 0) {
                const int ps = (tt - 1) & (RING - 1);
                while (ld_volatile_s(&cta_seq[ps]) != tt) {}
                __threadfence_block();
                c = reinterpret_cast<volatile double *>(cta_v)[ps] + c;
                f = reinterpret_cast<volatile int *>(cta_f)[ps];
            }
            const double v = v0 + c;
            y[r] = V(v);
            if (!f) {
                s_head_row = r;
                s_head_val = v;
            }
        };
        int pend_r = -1, pend_t = 0;
        double pend_v = 0.0;
        for (int t = 0; t < ntiles; ++t) {
            const int stage = t % C::STAGES;
            const int slot = t & (RING - 1);
            mbar_wait(&full[stage], (t / C::STAGES) & 1);
            if (lane == 0 && (warp == 0 || warp == NW - 1)) TR(t, warp ? 8 : 4);  // worker sees the stage
            const TileMeta mt = meta[stage];
            const int tile_is = mt.i_s;
            const int z = mt.j_e - mt.j_s;
            const char *sb = stages + size_t(stage) * C::STAGE_BYTES;
            const int32_t *cs = reinterpret_cast<const int32_t *>(sb + mt.col_first);
            const V *vs = reinterpret_cast<const V *>(sb + mt.val_first);
            const int32_t *rps = reinterpret_cast<const int32_t *>(sb + mt.rp_first);  // rps[k] = rp[i_s + k]
            // ---- gathers: K independent loads in flight per lane ----
            // all column reads first (plain shared loads, issued back to back),
            // then the K gathers: the volatile gathers keep program order, so
            // interleaving them with the column reads would serialise one
            // shared-memory latency per gather.  Positions >= z gather x[0]
            // (their products are masked in the walk).
            int cidx[K];
#pragma unroll
            for (int u = 0; u < K; ++u) cidx[u] = (q0 + u < z) ? cs[q0 + u] : 0;
            double xv[K];
#pragma unroll
            for (int u = 0; u < K; ++u) xv[u] = ldg_x(x + cidx[u]);
            // values into registers while the gathers fly (one burst of
            // conflict-free shared loads; the walk then reads registers only)
            double vv[K];
#pragma unroll
            for (int u = 0; u < K; ++u) vv[u] = double(vs[q0 + u]);
            if (lane == 0 && (warp == 0 || warp == NW - 1)) TR(t, warp ? 9 : 5);  // gathers issued
            // ---- this warp's row ends (no shared row warp: warps never wait
            //      on each other's maps) ----
            // Row k of the tile (global i_s + k) ends at tile position
            // e_k = rps[k+1] - j_s; a nonempty row is emitted at its last
            // nonzero e_k - 1 if that lies in [0, z) (empty rows: row warp).
            const int sp1 = min(sp0 + WSPAN, z);
            wmask[lane] = 0u;
            __syncwarp();
            if (sp0 < sp1) {
                const int nwin = mt.wr_end - mt.i_s;  // rows in the window
                const int j_s = mt.j_s;
                // first row ending after sp0: 32-ary search over the window
                int lo = 0, hi = nwin;
                while (hi - lo > 32) {
                    const int step = (hi - lo + 31) >> 5;
                    const int pp = lo + (lane + 1) * step - 1;
                    const bool pr = pp < hi && rps[pp + 1] - j_s <= sp0;
                    const int c = __popc(__ballot_sync(0xffffffffu, pr));
                    const int nhi = min(hi, lo + (c + 1) * step - 1);
                    lo = lo + c * step;
                    hi = c < 32 ? nhi : hi;
                }
                {
                    const int pp = lo + lane;
                    const bool pr = pp < hi && rps[pp + 1] - j_s <= sp0;
                    lo += __popc(__ballot_sync(0xffffffffu, pr));
                }
                for (int k = lo + lane;; k += 32) {
                    int e = INT_MAX, a = 0;
                    if (k < nwin) {
                        a = rps[k] - j_s;
                        e = rps[k + 1] - j_s;
                    }
                    if (e <= sp1 && a < e) {  // nonempty row ending in the span
                        const int pos = e - 1 - sp0;
                        const int ol = pos / K, bit = pos - ol * K;
                        atomicOr(&wmask[ol], 1u << bit);
                        wrow[pos] = uint16_t(k);
                    }
                    if (!__any_sync(0xffffffffu, e < sp1)) break;
                }
            }
            __syncwarp();
            const unsigned mask = wmask[lane];
            __syncwarp();
            if (lane == 0) {  // cols, vals and row offsets of this tile are in registers / the warp map now
                if (warp == 0 || warp == NW - 1) TR(t, warp ? 13 : 12);  // own map built
                mbar_arrive(&empty[stage]);
            }
#ifdef MSP_SPMV_TRACE
            asm volatile("" ::"d"(xv[K - 1]));
            if (lane == 0 && (warp == 0 || warp == NW - 1)) TR(t, warp ? 15 : 14);  // last gather returned
#endif
            // ---- walk (branch-free) ----
            // Every step is straight-line code: the multiply-add, the row-end
            // bit, a select that keeps the first row end's partial (it needs
            // the carry of earlier lanes, below), a predicated store for every
            // later row end, and a select that restarts the running sum.
            const int first_k = mask ? __ffs(mask) - 1 : K;
            V *ybase = y + tile_is;
            const uint16_t *lrow = wrow + lane * K;
            double run = 0.0, first_v = 0.0;
            auto walk = [&](auto tail) {
#pragma unroll
                for (int u = 0; u < K; ++u) {
                    double v = vv[u];
                    if constexpr (decltype(tail)::value) v = (q0 + u < z) ? v : 0.0;  // partial last tile
                    run = fma(v, xv[u], run);
                    const bool b = (mask >> u) & 1u;
                    first_v = (u == first_k) ? run : first_v;
                    const bool later = b && (u > first_k);
                    const int rr = later ? int(lrow[u]) : 0;
                    st_global_if(ybase + rr, V(run), later);
                    run = b ? 0.0 : run;
                }
            };
#ifdef MSP_SPMV_BRANCHY_WALK  // experiment: the round-1 walk (a branch per row end)
            (void)walk;
            {
                int fk = -1;
#pragma unroll
                for (int u = 0; u < K; ++u) {
                    if (q0 + u < z) run = fma(vv[u], xv[u], run);
                    if ((mask >> u) & 1u) {
                        if (fk < 0) {
                            fk = u;
                            first_v = run;
                        } else {
                            ybase[lrow[u]] = V(run);
                        }
                        run = 0.0;
                    }
                }
            }
#else
            if (q0 + K <= z) walk(std::false_type{});
            else walk(std::true_type{});
#endif
            const int first_r = mask ? tile_is + int(lrow[first_k]) : -1;
            if (lane == 0 && (warp == 0 || warp == NW - 1)) TR(t, warp ? 10 : 6);  // walk done
            const bool flagged = first_r >= 0;
            // ---- warp segmented scan ----
            const SegPair<double> inc = warp_seg_inclusive(SegPair<double>{flagged, run}, lane);
            const double exv = __shfl_up_sync(0xffffffffu, inc.v, 1);
            const unsigned fmask = __ballot_sync(0xffffffffu, flagged);
            const int flane = fmask ? __ffs(fmask) - 1 : 32;
            double pend_nv = 0.0;
            if (flagged) {
                const double v = lane ? first_v + exv : first_v;
                if (lane == flane) pend_nv = v;
                else y[first_r] = V(v);
            }
            // ---- publish the warp's trailing sum; the last warp forms the
            //      carry leaving the tile ----
            if (lane == 31) {
                // published through volatile stores, ordered before the tag by
                // the CTA fence (message passing; readers spin on the tag)
                reinterpret_cast<volatile double *>(agg_v)[slot * NW + warp] = inc.v;
                reinterpret_cast<volatile int *>(agg_f)[slot * NW + warp] = inc.f;
                __threadfence_block();
                st_volatile_s(&agg_seq[slot * NW + warp], t + 1);
                const int done = atomicAdd(&pub_cnt[slot], 1);
                if (done == NW - 1) {
                    __threadfence_block();
                    double c = 0.0;
                    int f = 0;
                    if (t > 0) {
                        const int ps = (t - 1) & (RING - 1);
                        while (ld_volatile_s(&cta_seq[ps]) != t) {}
                        __threadfence_block();
                        c = cta_v[ps];
                        f = cta_f[ps];
                    }
                    for (int w2 = 0; w2 < NW; ++w2) {
                        const int fw = reinterpret_cast<volatile int *>(agg_f)[slot * NW + w2];
                        const double vw = reinterpret_cast<volatile double *>(agg_v)[slot * NW + w2];
                        c = fw ? vw : c + vw;
                        f |= fw;
                    }
                    reinterpret_cast<volatile double *>(cta_v)[slot] = c;
                    reinterpret_cast<volatile int *>(cta_f)[slot] = f;
                    pub_cnt[slot] = 0;
                    __threadfence_block();
                    st_volatile_s(&cta_seq[slot], t + 1);
                }
            }
            if (pend_r >= 0) finish_first(pend_r, pend_v, pend_t);
            if (lane == 0 && (warp == 0 || warp == NW - 1)) TR(t, warp ? 11 : 7);  // tile finished
            pend_r = (lane == flane) ? first_r : -1;
            pend_v = pend_nv;
            pend_t = t;
        }
        if (pend_r >= 0) finish_first(pend_r, pend_v, pend_t);
    } else {
        // ============================ worker warps =============================
        // Worker `warp` owns products [warp*256, warp*256 + 256) of every tile.
        //   phase A: lane l computes products l, l+32, ... (coalesced col/val
        //            reads, x gathers of consecutive nonzeros) into a
        //            warp-private swizzled buffer (P:444-456 strided -> blocked);
        //   walk:    lane l sums products 8l .. 8l+7; at a row end it writes y
        //            (its first row waits for the carry of earlier lanes);
        //   scan:    warp segmented scan -> carry of earlier lanes; the warp's
        //            first row also needs the carry of earlier warps / tiles,
        //            read from their published trailing sums (look-back).
        double *wprod = prodbuf + warp * WSPAN;
        const int s_sw = (lane >> 1) & 3;
        const unsigned col_lim = unsigned(n_cols);
        const int wbase = warp * WSPAN;
        int cidx[K];
        V xv[K];
        // phase A issue: columns from the stage, x gathers into registers.
        // Positions >= z read other bytes of the stage (in bounds); their
        // columns are clamped and their products masked in the walk.
        V vv[K];
        int nx_is = 0, nx_z = 0;  // row window start and nonzero count of the issued tile
        auto a_issue = [&](int t) {
            const int stage = t % C::STAGES;
            mbar_wait(&full[stage], (t / C::STAGES) & 1);
            nx_is = meta[stage].i_s;
            nx_z = meta[stage].j_e - meta[stage].j_s;
            const char *sb = stages + size_t(stage) * C::STAGE_BYTES;
            const int32_t *cs = reinterpret_cast<const int32_t *>(sb + meta[stage].col_first) + wbase;
            const V *vs = reinterpret_cast<const V *>(sb + meta[stage].val_first) + wbase;
#pragma unroll
            for (int u = 0; u < K; ++u) {
                const unsigned c = unsigned(cs[lane + 32 * u]);
                cidx[u] = int(c < col_lim ? c : 0u);
            }
#pragma unroll
            for (int u = 0; u < K; ++u) xv[u] = gather_x<V, C::L1G>(x + cidx[u]);
#pragma unroll
            for (int u = 0; u < K; ++u) vv[u] = vs[lane + 32 * u];
        };
        auto finish_first = [&](int r, double v0, int tt) {
            const int sl = tt & (RING - 1);
            double c = 0.0;
            int f = 0;
            for (int w2 = warp - 1; w2 >= 0 && !f; --w2) {
                while (ld_volatile_s(&agg_seq[sl * NW + w2]) != tt + 1) {}
                __threadfence_block();
                c = reinterpret_cast<volatile double *>(agg_v)[sl * NW + w2] + c;
                f = reinterpret_cast<volatile int *>(agg_f)[sl * NW + w2];
            }
            if (!f && tt > 0) {
                const int ps = (tt - 1) & (RING - 1);
                while (ld_volatile_s(&cta_seq[ps]) != tt) {}
                __threadfence_block();
                c = reinterpret_cast<volatile double *>(cta_v)[ps] + c;
                f = reinterpret_cast<volatile int *>(cta_f)[ps];
            }
            const double v = v0 + c;
            y[r] = V(v);
            if (!f) {  // first row this CTA completes
                s_head_row = r;
                s_head_val = v;
            }
        };
        int pend_r = -1, pend_t = 0;
        double pend_v = 0.0;
        a_issue(0);
        for (int t = 0; t < ntiles; ++t) {
            const int stage = t % C::STAGES;
            const int slot = t & (RING - 1);
            const int rs = t % C::RSLOTS;
            const int tile_is = nx_is, z = nx_z;
            if (lane == 0 && (warp == 0 || warp == NW - 1)) TR(t, warp ? 8 : 4);  // tile's gathers issued earlier
            // ---- phase A finish: products -> warp-private buffer ----
#pragma unroll
            for (int u = 0; u < K; ++u) wprod[swz<K>(lane + 32 * u)] = double(vv[u]) * double(xv[u]);
            __syncwarp();
            // the stage is released once the products are formed (releasing it
            // right after the col/val loads measured slower: deeper TMA
            // run-ahead raised memory contention and per-CTA tail variance)
            // workers in lockstep: a warp that runs ahead would take issue slots from
            // the slowest one, whose lag then eats the ring's slack (measured)
            if (lane == 0 && (warp == 0 || warp == NW - 1)) TR(t, warp ? 9 : 5);  // products formed
            named_bar_sync(1, NW * 32);
            if (lane == 0) mbar_arrive(&empty[stage]);
            mbar_wait(&rowsrdy[rs], (t / C::RSLOTS) & 1);
            if (lane == 0 && (warp == 0 || warp == NW - 1)) TR(t, warp ? 13 : 12);  // lockstep + row map
            if constexpr (C::EARLY) {
                if (t + 1 < ntiles) a_issue(t + 1);
            }
            // ---- walk ----
            const uint32_t *flags = reinterpret_cast<const uint32_t *>(rslots + size_t(rs) * C::RSLOT_BYTES);
            const uint16_t *rmap =
                reinterpret_cast<const uint16_t *>(rslots + size_t(rs) * C::RSLOT_BYTES + C::FLAG_BYTES);
            const int qs = wbase + lane * K;  // tile position of this lane's first product
            const unsigned mask = reinterpret_cast<const uint8_t *>(flags)[qs >> 3];
            double run = 0.0, first_v = 0.0;
            int first_r = -1;
            if (qs < z) {
                double p[K];
                double *myp = wprod + lane * K;
                if (qs + K <= z) {
#pragma unroll
                    for (int i = 0; i < K / 2; ++i) {
                        const double2 d2 = reinterpret_cast<const double2 *>(myp)[i ^ s_sw];
                        p[2 * i] = d2.x;
                        p[2 * i + 1] = d2.y;
                    }
                } else {
#pragma unroll
                    for (int i = 0; i < K / 2; ++i) {
                        const double2 d2 = reinterpret_cast<const double2 *>(myp)[i ^ s_sw];
                        p[2 * i] = (qs + 2 * i < z) ? d2.x : 0.0;
                        p[2 * i + 1] = (qs + 2 * i + 1 < z) ? d2.y : 0.0;
                    }
                }
                // branch-free walk: predicated stores for every row end after
                // the lane's first (whose partial waits for the lane carry)
                const int k0 = mask ? __ffs(mask) - 1 : K;
#pragma unroll
                for (int k = 0; k < K; ++k) {
                    run += p[k];
                    const bool b = (mask >> k) & 1u;
                    first_v = (k == k0) ? run : first_v;
                    const bool later = b && (k > k0);
                    const int rr = later ? int(rmap[qs + k]) : 1;
                    st_global_if(y + tile_is + rr - 1, V(run), later);
                    run = b ? 0.0 : run;
                }
                if (mask) first_r = tile_is + int(rmap[qs + k0]) - 1;
            }
            const bool flagged = first_r >= 0;
            // ---- warp segmented scan ----
            const SegPair<double> inc = warp_seg_inclusive(SegPair<double>{flagged, run}, lane);
            const double exv = __shfl_up_sync(0xffffffffu, inc.v, 1);
            const unsigned fmask = __ballot_sync(0xffffffffu, flagged);
            const int flane = fmask ? __ffs(fmask) - 1 : 32;
            double pend_nv = 0.0;
            if (flagged) {
                const double v = lane ? first_v + exv : first_v;  // carry from earlier lanes
                if (lane == flane) pend_nv = v;                    // also needs earlier warps' carry
                else y[first_r] = V(v);
            }
            __syncwarp();
            if (lane == 0) mbar_arrive(&rowsfree[rs]);  // done with this tile's row map
            // ---- publish this warp's trailing sum; the last warp of the tile
            //      forms the carry leaving the tile ----
            if (lane == 31) {
                // published through volatile stores, ordered before the tag by
                // the CTA fence (message passing; readers spin on the tag)
                reinterpret_cast<volatile double *>(agg_v)[slot * NW + warp] = inc.v;
                reinterpret_cast<volatile int *>(agg_f)[slot * NW + warp] = inc.f;
                __threadfence_block();
                st_volatile_s(&agg_seq[slot * NW + warp], t + 1);
                const int done = atomicAdd(&pub_cnt[slot], 1);
                if (done == NW - 1) {
                    __threadfence_block();
                    double c = 0.0;
                    int f = 0;
                    if (t > 0) {
                        const int ps = (t - 1) & (RING - 1);
                        while (ld_volatile_s(&cta_seq[ps]) != t) {}
                        __threadfence_block();
                        c = cta_v[ps];
                        f = cta_f[ps];
                    }
                    for (int w2 = 0; w2 < NW; ++w2) {
                        const int fw = reinterpret_cast<volatile int *>(agg_f)[slot * NW + w2];
                        const double vw = reinterpret_cast<volatile double *>(agg_v)[slot * NW + w2];
                        c = fw ? vw : c + vw;
                        f |= fw;
                    }
                    reinterpret_cast<volatile double *>(cta_v)[slot] = c;
                    reinterpret_cast<volatile int *>(cta_f)[slot] = f;
                    pub_cnt[slot] = 0;
                    __threadfence_block();
                    st_volatile_s(&cta_seq[slot], t + 1);
                }
            }
            // next tile's gathers fly while the previous tile's first row is finished
            if (lane == 0 && (warp == 0 || warp == NW - 1)) TR(t, warp ? 10 : 6);  // walked + scanned
            if constexpr (!C::EARLY) {
                if (t + 1 < ntiles) a_issue(t + 1);
            }
            if (lane == 0 && (warp == 0 || warp == NW - 1)) TR(t, warp ? 11 : 7);  // next tile's gathers issued
            // ---- the warp's first row of tile t-1 (deferred one tile so that
            //      the look-back never waits): carry of earlier warps (nearest
            //      first), then of earlier tiles ----
            if (pend_r >= 0) finish_first(pend_r, pend_v, pend_t);
            pend_r = (lane == flane) ? first_r : -1;
            pend_v = pend_nv;
            pend_t = t;
        }
        if (pend_r >= 0) finish_first(pend_r, pend_v, pend_t);
    }
    __syncthreads();
    if (tid == 0) {
        CtaRecord rec;
        rec.carry_key = s_carry_key;
        rec.carry_val = ntiles > 0 ? cta_v[(ntiles - 1) & (RING - 1)] : 0.0;
        rec.head_row = s_head_row;
        rec.head_val = s_head_val;
        recs[blockIdx.x] = rec;
    }

    // ============================ update phase (last CTA) ======================
    __syncthreads();
    if (tid == 0) {
        __threadfence();
        const unsigned ticket = atomicAdd(counter, 1u);
        s_last = (ticket == unsigned(G - 1));
    }
    __syncthreads();
    if (!s_last) return;
    __threadfence();
    // A row spanning many CTAs (C4's 10^6-nonzero row crosses ~100 CTA ranges
    // at 8 CTAs/SM) is one run of equal carry keys: its head sums the run.
    // The carries are staged in shared memory (the tile buffers, free now;
    // the mbarrier words after them are not touched) so that the run sum
    // is a shared-memory loop, not a chain of dependent L2 round trips.
    constexpr int kStageBytes = C::SMEM - C::MISC_BYTES;
    const bool staged = size_t(G) * (sizeof(int) + sizeof(double)) <= size_t(kStageBytes);
    double *s_cv = reinterpret_cast<double *>(smem);
    int *s_ck = reinterpret_cast<int *>(s_cv + G);
    if (staged) {
        for (int k = tid; k < G; k += blockDim.x) {
            s_ck[k] = __ldcg(&recs[k].carry_key);
            s_cv[k] = __ldcg(&recs[k].carry_val);
        }
        __syncthreads();
    }
    for (int k = tid; k < G; k += blockDim.x) {
        const int key = staged ? s_ck[k] : __ldcg(&recs[k].carry_key);
        if (key < 0 || key >= m) continue;
        if (k > 0 && (staged ? s_ck[k - 1] : __ldcg(&recs[k - 1].carry_key)) == key) continue;  // not a run head
        double s = 0.0;
        int k2 = k;
        if (staged) {
            for (; k2 < G && s_ck[k2] == key; ++k2) s += s_cv[k2];
        } else {
            for (; k2 < G && __ldcg(&recs[k2].carry_key) == key; ++k2) s += __ldcg(&recs[k2].carry_val);
        }
        // the CTA after the run emits row `key` first (continuity of the path)
        if (k2 < G && __ldcg(&recs[k2].head_row) == key) y[key] = V(s + __ldcg(&recs[k2].head_val));
    }
    if (tid == 0) *counter = 0u;  // leave the workspace reusable
}

// Tile shapes (consumer threads, products per thread, stages, CTAs/SM).
// Configs 0 and 4 are the defaults (see launch()); MSP_SPMV_CFG=<n> forces one (tuning only).
template <typename V, int I> struct Shape;
template <typename V> struct Shape<V, 0> { using C = Cfg<V, 8, 2, 2, 2>; };
template <typename V> struct Shape<V, 1> { using C = Cfg<V, 8, 2, 2, 3>; };
template <typename V> struct Shape<V, 2> { using C = Cfg<V, 8, 3, 3, 2>; };
template <typename V> struct Shape<V, 3> { using C = Cfg<V, 8, 2, 4, 2>; };
template <typename V> struct Shape<V, 4> { using C = Cfg<V, 4, 2, 4, 4>; };
template <typename V> struct Shape<V, 5> { using C = Cfg<V, 4, 2, 4, 5>; };
template <typename V> struct Shape<V, 6> { using C = Cfg<V, 2, 2, 4, 8>; };
template <typename V> struct Shape<V, 7> { using C = Cfg<V, 2, 2, 4, 6>; };
template <typename V> struct Shape<V, 8> { using C = Cfg<V, 4, 2, 4, 4, true>; };
template <typename V> struct Shape<V, 9> { using C = Cfg<V, 2, 2, 4, 8, true, true>; };
template <typename V> struct Shape<V, 10> { using C = Cfg<V, 2, 3, 4, 8, true>; };
template <typename V> struct Shape<V, 11> { using C = Cfg<V, 2, 4, 4, 8, true>; };
constexpr int kNumShapes = 12;

template <typename V, class C>
msp_status launch_cfg(const msp_csr *A, const void *x, void *y, void *ws, size_t ws_bytes, cudaStream_t s)
{
    auto kern = spmv_merge_kernel<V, C>;
    int occ = 1;
    // the transpose walk's gathers need L1 lines for their in-flight misses:
    // carveout fitted to the occupancy (C3 534 -> 454 us, C4 103 -> 83 us,
    // C5 12.7 -> 9.0 ms; profiles/r2/spmv_irregular_shapes.txt)
    static const bool fit = !getenv("MSP_SPMV_FULL_CARVEOUT");
    msp_status st = set_smem_attr(reinterpret_cast<const void *>(kern), C::SMEM, "spmv: smem", C::THREADS, &occ,
                                  fit && !C::ROWK);
    if (st != MSP_OK) return st;
    if (occ > 8) occ = 8;
    static bool said = false;
    if (!said && getenv("MSP_VERBOSE")) {
        fprintf(stderr, "msp spmv: rowk=%d K=%d NW=%d T=%d stages=%d smem=%d occupancy=%d CTAs/SM\n", int(C::ROWK),
                C::K, C::NW, C::T, C::STAGES, C::SMEM, occ);
        said = true;
    }
    if (A->nrows == 0) return MSP_OK;
    if (A->nnz == 0)  // every row is empty: y = +0.0 (Z6)
        return cuda_check(cudaMemsetAsync(y, 0, size_t(A->nrows) * sizeof(V), s), "spmv: zero y");
    const int64_t total = int64_t(A->nrows) + A->nnz;
    const int64_t ntiles = ceil_div(total, C::T);
    // one persistent wave, no more CTAs than tiles
    int64_t g = int64_t(occ) * sm_count();
    if (g > ntiles) g = ntiles;
    const int grid = int(g);
    Carve cv(ws, ws_bytes);
    unsigned *counter = cv.take<unsigned>(1);
    CtaRecord *recs = cv.take<CtaRecord>(size_t(grid));
    if (!cv.ok()) return MSP_ERR_WORKSPACE;
    kern<<<grid, C::THREADS, C::SMEM, s>>>(A->nrows, A->nnz, A->row_offsets, A->col_idx,
                                           static_cast<const V *>(A->vals), static_cast<const V *>(x),
                                           static_cast<V *>(y), A->ncols, recs, counter);
    return last_launch("spmv_merge_kernel");
}

int shape_choice()
{
    static int c = -2;
    if (c == -2) {
        const char *e = getenv("MSP_SPMV_CFG");
        // -3: chosen per matrix (default), -1: row-aligned variant, 0..: transpose-walk shapes
        c = e ? atoi(e) : -3;
        if (c < -3 || c >= kNumShapes) c = -3;
    }
    return c;
}

// Row-aligned variant: K = the instantiated odd width nearest the mean row
// length (MSP_SPMV_K overrides, tuning only); NW worker warps per CTA.
constexpr int kKs[] = {7, 11, 15, 19, 23, 27, 31};

int k_choice(const msp_csr *A)
{
    const char *e = getenv("MSP_SPMV_K");
    const double avg = e ? atof(e) : (A->nrows > 0 ? double(A->nnz) / double(A->nrows) : 0.0);
    int best = kKs[0];
    for (int k : kKs)
        if (std::abs(double(k) - avg) < std::abs(double(best) - avg)) best = k;
    return best;
}

int nw_choice()
{
    static int nw = -1;
    if (nw < 0) {
        const char *e = getenv("MSP_SPMV_NW");
        nw = (e && atoi(e) == 4) ? 4 : 8;
    }
    return nw;
}

// Warp-tile kernel (spmv_wt.cu) for the row-aligned layout; MSP_SPMV_WT=0
// selects the CTA-tile kernel below (tuning / comparison only).
int wt_choice()
{
    static int v = -1;
    if (v < 0) {
        const char *e = getenv("MSP_SPMV_WT");
        v = e ? atoi(e) : 1;  // 0: CTA-tile kernel, 2: warp tiles for every K (tuning)
    }
    return v;
}

template <typename V, int NW>
msp_status launch_k(int K, const msp_csr *A, const void *x, void *y, void *ws, size_t ws_bytes, cudaStream_t s)
{
    constexpr int MB = NW == 4 ? 2 : 1;
    switch (K) {
    case 7: return launch_cfg<V, CfgK<V, NW, 7, 2, MB>>(A, x, y, ws, ws_bytes, s);
    case 11: return launch_cfg<V, CfgK<V, NW, 11, 2, MB>>(A, x, y, ws, ws_bytes, s);
    case 15: return launch_cfg<V, CfgK<V, NW, 15, 2, MB>>(A, x, y, ws, ws_bytes, s);
    case 19: return launch_cfg<V, CfgK<V, NW, 19, 2, MB>>(A, x, y, ws, ws_bytes, s);
    case 23: return launch_cfg<V, CfgK<V, NW, 23, 2, MB>>(A, x, y, ws, ws_bytes, s);
    case 27: return launch_cfg<V, CfgK<V, NW, 27, 2, MB>>(A, x, y, ws, ws_bytes, s);
    default: return launch_cfg<V, CfgK<V, NW, 31, 2, MB>>(A, x, y, ws, ws_bytes, s);
    }
}

template <typename V>
msp_status launch(const msp_csr *A, const void *x, void *y, void *ws, size_t ws_bytes, cudaStream_t s)
{
    int shape = shape_choice();
    if (shape == -3) {
        // default: row-aligned lanes for long regular rows; else the transpose
        // walk, with 4 small CTAs per SM (T = 1,024) while x fits in half of
        // L2 -- the x gathers are then L2-latency-bound and more resident
        // tiles hide it (C3 686 -> 534 us, C4 106 -> 103 us) -- and 2 large
        // CTAs per SM once x spills to DRAM, where more gathers in flight only
        // add DRAM contention (C5 13.0 vs 13.3 ms).
        // (profiles/r2/spmv_irregular_shapes.txt)
        // fp32 values with x in L2 (C3): 8 CTAs/SM of 2 workers that issue
        // tile t+1's gathers before walking tile t (C3 455 -> 419 us; fp64
        // spills at that size: C4 keeps shape 4, 83 vs 106 us)
        // (profiles/r2/spmv_irregular_shapes.txt)
        if (A->nrows > 0 && double(A->nnz) >= 20.0 * double(A->nrows)) shape = -1;
        else if (int64_t(A->ncols) * int64_t(sizeof(V)) <= l2_bytes() / 2) shape = sizeof(V) == 4 ? 9 : 4;
        else shape = 0;
    }
    switch (shape) {
    case -1: {
        const int K = k_choice(A);
        if (wt_choice() && (K >= 15 || wt_choice() == 2)) return spmv_wt_run(K, A, x, y, ws, ws_bytes, s);
        return nw_choice() == 8 ? launch_k<V, 8>(K, A, x, y, ws, ws_bytes, s)
                                : launch_k<V, 4>(K, A, x, y, ws, ws_bytes, s);
    }
    case 1: return launch_cfg<V, typename Shape<V, 1>::C>(A, x, y, ws, ws_bytes, s);
    case 2: return launch_cfg<V, typename Shape<V, 2>::C>(A, x, y, ws, ws_bytes, s);
    case 3: return launch_cfg<V, typename Shape<V, 3>::C>(A, x, y, ws, ws_bytes, s);
    case 4: return launch_cfg<V, typename Shape<V, 4>::C>(A, x, y, ws, ws_bytes, s);
    case 5: return launch_cfg<V, typename Shape<V, 5>::C>(A, x, y, ws, ws_bytes, s);
    case 6: return launch_cfg<V, typename Shape<V, 6>::C>(A, x, y, ws, ws_bytes, s);
    case 7: return launch_cfg<V, typename Shape<V, 7>::C>(A, x, y, ws, ws_bytes, s);
    case 8: return launch_cfg<V, typename Shape<V, 8>::C>(A, x, y, ws, ws_bytes, s);
    case 9: return launch_cfg<V, typename Shape<V, 9>::C>(A, x, y, ws, ws_bytes, s);
    case 10: return launch_cfg<V, typename Shape<V, 10>::C>(A, x, y, ws, ws_bytes, s);
    case 11: return launch_cfg<V, typename Shape<V, 11>::C>(A, x, y, ws, ws_bytes, s);
    default: return launch_cfg<V, typename Shape<V, 0>::C>(A, x, y, ws, ws_bytes, s);
    }
}

}  // namespace

size_t spmv_ws_bytes(const msp_csr *A)
{
    // counter + one record per CTA (grid <= max(8 per SM, tiles / tiles-per-CTA))
    const int64_t tiles = ceil_div(int64_t(A->nrows) + A->nnz, 1024);
    const int64_t g = std::max<int64_t>(int64_t(8) * sm_count(), ceil_div(tiles, 2));
    return 512 + size_t(g) * sizeof(CtaRecord);
}

msp_status spmv_run(const msp_csr *A, const void *x, void *y, void *ws, size_t ws_bytes, cudaStream_t s)
{
    if (A->dtype == MSP_F64) return launch<double>(A, x, y, ws, ws_bytes, s);
    return launch<float>(A, x, y, ws, ws_bytes, s);
}

}  // namespace msp

