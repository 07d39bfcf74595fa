// spgemm.cu -- C = A B by expansion, sorting and compression (sm_100a).
//
// Paper: Section III-C.  Work is measured in products, Nprods
// (P:888-896).  Setup forms the prefix sum S of the B row lengths referenced
// by A's column indices (reading Z8: flat int64 exclusive scan);
// products are split over CTAs with a search over S (reading Z7);
// every CTA expands its products, sorts them so duplicates become adjacent
// and reduces them; what straddles CTAs is
// ordered and reduced in a global phase.
//
// B200 design:
//   * Merge grid = A nonzero ends + products (items), so a tile of T items
//     holds at most T products and at most T nonzeros whatever the widths.
//     Tile boundaries are merge-path splits moved to the nearest row
//     boundary when they fall inside a short row (<= T/4 items), so short
//     rows never straddle tiles; rows with more than T/4 items ("long rows")
//     are masked out of the tiles and handled by the global phase.
//   * Tile kernel (512 threads x 16 products): merge-path expansion from
//     S (each thread finds its split once, then walks), keys (row, col)
//     packed in 64 bits, stable block merge sort (sort.cuh), then
//     compression: symbolic adds each row's unique count into
//     C.row_offsets; numeric writes each unique (col, sum) at
//     C.row_offsets[row] + rank of the key in its row (the tile's short
//     rows are complete).  Duplicates are summed in product order (k
//     ascending, as Gustavson's oracle), fp64 accumulation (Z4).
//   * Long rows (global phase): each is cut into chunks of T products, each
//     chunk expanded and sorted by column into a run; runs are merged pairwise
//     (merge path per thread, stable) until one run per row remains; a head-
//     flag pass reduces equal columns (counts, or scan + sums for numeric).
#include <algorithm>
#include <cstdlib>
#include <climits>
#include <cstdint>
#include <cstdio>

#include "common.cuh"
#include "internal.h"
#include "sort.cuh"

namespace msp {
namespace {

constexpr int GM_NT = 512;
constexpr int GM_IPT = 16;
constexpr int GM_T = GM_NT * GM_IPT;  // items (nonzero ends + products) per tile
constexpr int GM_LONG = GM_T / 4;     // rows with more items than this are long
// Partition step: snapping a split to the nearest short-row boundary moves
// it by at most GM_LONG / 2, so tiles of GM_TP nominal items never exceed GM_T.
constexpr int GM_TP = GM_T - GM_LONG;
constexpr int GM_TL = GM_T;           // products per long-row chunk
constexpr uint64_t KEY_MASKED = ~0ull;

__device__ __forceinline__ int64_t dmin(int64_t a, int64_t b) { return a < b ? a : b; }
__device__ __forceinline__ int64_t dmax(int64_t a, int64_t b) { return a > b ? a : b; }

// ================================================================ setup ===

// COO row of every A nonzero, merge-based (equal rows + nonzeros per thread).
constexpr int AROW_ITEMS = 16;
__global__ void arow_kernel(int32_t m, int64_t nnz, const int32_t *__restrict__ rp, int32_t *__restrict__ arow)
{
    const int64_t total = int64_t(m) + nnz;
    const int64_t d = (int64_t(blockIdx.x) * blockDim.x + threadIdx.x) * AROW_ITEMS;
    if (d >= total) return;
    int64_t lo = dmax(0, d - nnz), hi = dmin(d, m);
    while (lo < hi) {
        const int64_t mid = (lo + hi) >> 1;
        if (int64_t(rp[mid + 1]) <= d - mid - 1) lo = mid + 1;
        else hi = mid;
    }
    int64_t i = lo, j = d - lo;
    const int64_t end = dmin(d + AROW_ITEMS, total);
    for (int64_t q = d; q < end; ++q) {
        if (i < m && rp[i + 1] <= j) ++i;  // row end
        else arow[j++] = int32_t(i);
    }
}

// Per row: products P_r = S[rp[r+1]] - S[rp[r]]; long iff nnz_r + P_r > GM_LONG.
__global__ void rowclass_kernel(int32_t m, const int32_t *__restrict__ rp, const int64_t *__restrict__ S,
                                uint8_t *__restrict__ rowlong, int32_t *__restrict__ longflag,
                                int64_t *__restrict__ longP, unsigned long long *__restrict__ maxP)
{
    unsigned long long mx = 0, nl = 0;
    for (int64_t r = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; r < m; r += int64_t(gridDim.x) * blockDim.x) {
        const int32_t a = rp[r], b = rp[r + 1];
        const int64_t P = S[b] - S[a];
        const bool lg = (int64_t(b - a) + P) > GM_LONG;
        rowlong[r] = lg ? 1 : 0;
        longflag[r] = lg ? 1 : 0;
        longP[r] = 0;
        mx = max(mx, (unsigned long long)P);
        nl += lg;
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
        nl += __shfl_xor_sync(0xffffffffu, nl, o);
    }
    if ((threadIdx.x & 31) == 0 && mx) atomicMax(maxP, mx);
    if ((threadIdx.x & 31) == 0 && nl) atomicAdd(maxP + 12, nl);  // stats[12]: long rows
}

__global__ void long_scatter_kernel(int32_t m, const int32_t *__restrict__ rp, const int64_t *__restrict__ S,
                                    const int32_t *__restrict__ longflag, const int64_t *__restrict__ longpos,
                                    int32_t *__restrict__ longrow, int64_t *__restrict__ longP,
                                    int64_t *__restrict__ longC)
{
    for (int64_t r = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; r < m; r += int64_t(gridDim.x) * blockDim.x) {
        if (!longflag[r]) continue;
        const int64_t idx = longpos[r];
        const int64_t P = S[rp[r + 1]] - S[rp[r]];
        longrow[idx] = int32_t(r);
        longP[idx] = P;
        longC[idx] = (P + GM_TL - 1) / GM_TL;
    }
}

// ---------------------------------------------------- segmented path (f3)
// The paper's future work: "adaptively introducing segmented
// approaches when necessary" for rows where sorting the expanded products
// gains little -- its failure case is Dense, whose rows produce few
// duplicates per CTA but need huge temporary storage in the global pass
// (P:1648-1660).  A long row whose output columns span at most SPA_W
// columns, with at least one product per 4 columns of that span, is instead
// accumulated row-wise in a shared-memory dense accumulator (one CTA per
// row): no expanded product is stored, and the sum runs over k in A's
// column order -- the order of Gustavson's oracle -- with separate multiply
// and add roundings.
constexpr int SPA_W = 12288;    // accumulator columns (96 KB fp64 + a bit per column)
constexpr int SPA_NT = 256;

// (long rows only: the warp-row path's classification has written the
// BITMAP rows' spans already)
__global__ void span_init_kernel(int32_t m, const uint8_t *__restrict__ rowlong, int32_t *__restrict__ lo,
                                 int32_t *__restrict__ hi)
{
    for (int64_t r = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; r < m; r += int64_t(gridDim.x) * blockDim.x) {
        if (!rowlong[r]) continue;
        lo[r] = INT_MAX;
        hi[r] = -1;
    }
}

// column span of every long row: min / max over its products' columns
__global__ void span_kernel(int64_t nnzA, const int32_t *__restrict__ Acol, const int32_t *__restrict__ arow,
                            const uint8_t *__restrict__ rowlong, const int32_t *__restrict__ Brp,
                            const int32_t *__restrict__ Bcol, int32_t *__restrict__ lo, int32_t *__restrict__ hi)
{
    // grid-stride with whole warps, so that a warp whose 32 nonzeros all
    // belong to one long row (C4's dense row: 10^6 of them) reduces them
    // first and issues ONE atomic pair instead of 32
    const int64_t stride = int64_t(gridDim.x) * blockDim.x;
    for (int64_t j0 = int64_t(blockIdx.x) * blockDim.x; j0 < nnzA; j0 += stride) {
        const int64_t j = j0 + threadIdx.x;
        int32_t r = -1, cl = INT_MAX, ch = -1;
        if (j < nnzA) {
            r = arow[j];
            if (rowlong[r]) {
                const int32_t k = Acol[j], b0 = Brp[k], b1 = Brp[k + 1];
                if (b1 > b0) {
                    cl = Bcol[b0];
                    ch = Bcol[b1 - 1];
                }
            } else {
                r = -1;
            }
        }
        const int32_t r0 = __shfl_sync(0xffffffffu, r, 0);
        if (__all_sync(0xffffffffu, r == r0)) {
            const int32_t wl = __reduce_min_sync(0xffffffffu, cl), wh = __reduce_max_sync(0xffffffffu, ch);
            if ((threadIdx.x & 31) == 0 && r0 >= 0 && wh >= 0) {
                atomicMin(&lo[r0], wl);
                atomicMax(&hi[r0], wh);
            }
        } else if (r >= 0 && ch >= 0) {
            atomicMin(&lo[r], cl);
            atomicMax(&hi[r], ch);
        }
    }
}

// Cost model: a long row is segmented iff its products cover at least one
// column in four of its output span (P_r >= span / 4).  A span wider than
// SPA_W is cut into windows of SPA_W columns, one CTA each (every window CTA
// walks all of the row's A nonzeros and binary-searches each B row for its
// window), taken only while those searches stay below the product work:
// windows * nnz_r <= P_r (C4's rows through the dense row: 163 windows x ~10
// A nonzeros for 4.75e6 products; the dense row itself, 10^6 A nonzeros,
// stays on the ESC long-row pass).  spaflag[r] = the row's window count.
__global__ void spa_classify_kernel(int32_t m, const int32_t *__restrict__ rp, const int64_t *__restrict__ S,
                                    const int32_t *__restrict__ lo, const int32_t *__restrict__ hi,
                                    uint8_t *__restrict__ rowlong, int32_t *__restrict__ longflag,
                                    int32_t *__restrict__ spaflag)
{
    for (int64_t r = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; r < m; r += int64_t(gridDim.x) * blockDim.x) {
        int f = 0;
        if (rowlong[r]) {
            const int64_t span = int64_t(hi[r]) - lo[r] + 1;
            const int64_t P = S[rp[r + 1]] - S[rp[r]];
            const int64_t nwin = (span + SPA_W - 1) / SPA_W;
            if (span >= 1 && 4 * P >= span && (nwin == 1 || nwin * int64_t(rp[r + 1] - rp[r]) <= P)) {
                f = int(nwin);
                rowlong[r] = 2;   // masked in tiles like a long row
                longflag[r] = 0;  // not in the ESC long-row pass
            }
        }
        spaflag[r] = f;
    }
}

// The segmented rows' windows are numbered in row order by the exclusive
// scan spapos of spaflag: item i belongs to the row r with spapos[r] <= i <
// spapos[r+1] and is its window i - spapos[r].

// One CTA per window of a segmented row (rows with span <= SPA_W: one
// window).  Symbolic marks the window's output columns (no ordering needed),
// counts them into C.rp[r+1] (atomic: integers, order-free) and keeps the
// window's count in wcnt[item]; numeric accumulates a_ik * b_kj for k in A's
// column order (a barrier per A nonzero keeps every column's sum in that
// order), then writes the marked columns ascending at C.rp[r] + the counts
// of the row's earlier windows.
template <typename V, bool NUM>
__global__ void __launch_bounds__(SPA_NT)
spa_row_kernel(int32_t m, const int64_t *__restrict__ spapos, const int32_t *__restrict__ Arp,
               const int32_t *__restrict__ Acol, const V *__restrict__ Aval, const int32_t *__restrict__ Brp,
               const int32_t *__restrict__ Bcol, const V *__restrict__ Bval, const int32_t *__restrict__ spanlo,
               const int32_t *__restrict__ spanhi, int32_t *__restrict__ Crp_counts, const int32_t *__restrict__ Crp,
               int32_t *__restrict__ wcnt, int32_t *__restrict__ Ccol, V *__restrict__ Cval)
{
    extern __shared__ __align__(16) char spa_smem[];
    double *acc = reinterpret_cast<double *>(spa_smem);                       // [SPA_W] (numeric)
    uint32_t *mark = reinterpret_cast<uint32_t *>(spa_smem + (NUM ? SPA_W * 8 : 0));  // [SPA_W / 32]
    __shared__ int32_t wsum[SPA_NT / 32];
    __shared__ int32_t s_r;
    __shared__ int32_t s_qlo[SPA_NT], s_qhi[SPA_NT];  // each A nonzero's B entries inside the window
    const int tid = threadIdx.x;
    const int64_t item = blockIdx.x;
    if (tid == 0) {  // the row owning this item: last r with spapos[r] <= item
        int64_t lo = 0, hi = m;
        while (hi - lo > 1) {
            const int64_t mid = (lo + hi) >> 1;
            if (spapos[mid] <= item) lo = mid;
            else hi = mid;
        }
        while (lo + 1 < m && spapos[lo + 1] <= item) ++lo;  // rows without windows share the offset
        s_r = int32_t(lo);
    }
    __syncthreads();
    const int32_t r = s_r;
    const int64_t win = item - spapos[r];
    const int32_t c0 = int32_t(int64_t(spanlo[r]) + win * SPA_W);
    const int span = int((int64_t(spanhi[r]) - c0 + 1 < SPA_W ? int64_t(spanhi[r]) - c0 + 1 : int64_t(SPA_W)));
    const bool whole = (win == 0) && (int64_t(spanhi[r]) - spanlo[r] + 1 <= SPA_W);  // one window: no searches
    const int nw = (span + 31) >> 5;
    for (int i = tid; i < nw; i += SPA_NT) mark[i] = 0u;
    __syncthreads();
    const int32_t a0 = Arp[r], a1 = Arp[r + 1];
    for (int32_t jc = a0; jc < a1; jc += SPA_NT) {
        // this chunk's A nonzeros: their B row ranges clipped to the window
        if (jc + tid < a1) {
            const int32_t k = Acol[jc + tid];
            int32_t b0 = Brp[k], b1 = Brp[k + 1];
            if (!whole) {
                int32_t lo = b0, hi = b1;  // first entry >= c0
                while (lo < hi) {
                    const int32_t mid = (lo + hi) >> 1;
                    if (Bcol[mid] < c0) lo = mid + 1;
                    else hi = mid;
                }
                b0 = lo;
                hi = b1;  // first entry >= c0 + span
                while (lo < hi) {
                    const int32_t mid = (lo + hi) >> 1;
                    if (Bcol[mid] < c0 + span) lo = mid + 1;
                    else hi = mid;
                }
                b1 = lo;
            }
            s_qlo[tid] = b0;
            s_qhi[tid] = b1;
        }
        __syncthreads();
        const int nj = min(SPA_NT, a1 - jc);
    for (int32_t jj = 0; jj < nj; ++jj) {
        const int32_t j = jc + jj;
        const int32_t b0 = s_qlo[jj], b1 = s_qhi[jj];
        double a = 0.0;
        if constexpr (NUM) a = double(Aval[j]);
        for (int32_t q = b0 + tid; q < b1; q += SPA_NT) {
            const int c = Bcol[q] - c0;
            if constexpr (NUM) {
                const double p = __dmul_rn(a, double(Bval[q]));
                const uint32_t bit = 1u << (c & 31);
                const bool seen = (mark[c >> 5] & bit) != 0;
                acc[c] = seen ? __dadd_rn(acc[c], p) : p;
                if (!seen) atomicOr(&mark[c >> 5], bit);
            } else {
                atomicOr(&mark[c >> 5], 1u << (c & 31));
            }
        }
        if constexpr (NUM) __syncthreads();  // column sums advance in k order
    }
        __syncthreads();  // the range buffers are refilled by the next chunk
    }
    __syncthreads();
    // marked columns, ascending: thread t owns words [t*WPT, (t+1)*WPT)
    constexpr int WPT = (SPA_W / 32 + SPA_NT - 1) / SPA_NT;
    int cnt = 0;
#pragma unroll
    for (int u = 0; u < WPT; ++u) {
        const int w = tid * WPT + u;
        if (w < nw) cnt += __popc(mark[w]);
    }
    int tot;
    int o = block_exclusive_sum<int, SPA_NT / 32>(cnt, wsum, 1, &tot);
    if constexpr (!NUM) {
        if (tid == 0) {
            wcnt[item] = tot;
            atomicAdd(&Crp_counts[r], tot);
        }
    } else {
        // output offset of this window: the row's earlier windows' counts
        int pre = 0;
        for (int64_t i = spapos[r] + tid; i < item; i += SPA_NT) pre += wcnt[i];
        int pre_tot;
        (void)block_exclusive_sum<int, SPA_NT / 32>(pre, wsum, 1, &pre_tot);
        const int64_t base = int64_t(Crp[r]) + pre_tot + o;
        int64_t p = base;
#pragma unroll
        for (int u = 0; u < WPT; ++u) {
            const int w = tid * WPT + u;
            if (w < nw) {
                uint32_t bits = mark[w];
                while (bits) {
                    const int b = __ffs(bits) - 1;
                    bits &= bits - 1;
                    const int c = w * 32 + b;
                    Ccol[p] = c0 + c;
                    Cval[p] = V(acc[c]);
                    ++p;
                }
            }
        }
    }
}

// ------------------------------------------ row accumulator for short rows
// The same idea as the segmented path, for SHORT rows (a B200 addition in
// the direction of the paper's future work): when every short
// row's output columns span at most WR_SPAN columns, the whole short-row
// product set skips expansion + sort.  One warp owns one row:
//   symbolic: marks the row's output columns in a warp-private bitmap over
//             its span, counts them and writes them ascending into a
//             scratch list at the row's product offset S[rp[r]] (at most P_r
//             entries);
//   numeric:  reads that list (ranks by binary search in shared memory),
//             zero-free accumulates a_ik * b_kj into a shared-memory
//             accumulator for k in A's column order (one k per step, a
//             __syncwarp between steps: a B row has distinct columns, so the
//             lanes of a step never collide), and writes the row of C.
// Every column sums its products in Gustavson's order with separate multiply
// and add roundings, as the oracle does.  The choice is global (all short
// rows or none) so that the tile pass is either skipped or untouched.
constexpr int WR_SPAN = 65536;            // widest short-row span the bitmaps cover (8 KB per warp)
#ifndef MSP_WR_SYM_WARPS  // tuning builds
#define MSP_WR_SYM_WARPS 8
#endif
#ifndef MSP_WR_NUM_WARPS
#define MSP_WR_NUM_WARPS 8
#endif
#ifndef MSP_WR_NUM_MINB
#define MSP_WR_NUM_MINB 3
#endif
constexpr int WR_SYM_WARPS = MSP_WR_SYM_WARPS;
#ifndef WR_EMIT_SERIAL
#define WR_EMIT_SERIAL 0  // experiment: per-lane serial emission of the column list (C2 symbolic 2.25 -> 3.12 ms: slower)
#endif           // 64 KB of bitmaps per CTA
#ifndef MSP_WR_UMAX
#define MSP_WR_UMAX 512
#endif
constexpr int WR_UMAX = MSP_WR_UMAX;      // accumulator entries per warp per pass (6 KB with the column list)
constexpr int WR_NUM_WARPS = MSP_WR_NUM_WARPS;

__device__ __forceinline__ int warp_excl_sum(int v, int lane, int *total)
{
    const int inc = warp_inclusive_sum(v, lane);
    *total = __shfl_sync(0xffffffffu, inc, 31);
    return inc - v;
}

// Short-row modes of the warp-row path (wmode[r]).  WM_NONE: long, or no
// products (C.row_offsets is cleared before symbolic, so nothing to do);
// WM_BITMAP: the bitmap / hash accumulator below (output span <= WR_SPAN);
// WM_SMALL: the compare-count path (ws_small_kernel).
enum : uint8_t { WM_NONE = 0, WM_BITMAP = 1, WM_SMALL = 2 };
constexpr int WS_ALWAYS = 64;    // rows with at most this many products take the small path
constexpr int WS_PMAX = 256;     // ... and wider-than-WR_SPAN rows with at most this many
constexpr int WS_BATCH = 256;    // products (and A nonzeros) per warp batch of small rows
constexpr int WS_PPL = WS_BATCH / 32;

// Row classification for the warp-row path, 32 rows per warp round (lane per
// row): P_r = S[rp[r+1]] - S[rp[r]], nnz_r = rp[r+1] - rp[r].  Rows with
// 1 <= P_r <= WS_ALWAYS (and nnz_r <= WS_BATCH) are SMALL without a span;
// the others get their output span (warp-cooperative, one row at a time):
// span <= WR_SPAN -> BITMAP; wider and P_r, nnz_r <= WS_PMAX -> SMALL;
// wider still -> promoted to a long row (rowlong / longflag set: the global
// phase takes it).  With the small path off (MSP_SPGEMM_SMALL=0, the v5
// behaviour) every row with products needs the bitmap and a too-wide one is
// counted in stats[7], which turns the warp-row path off.  stats: [7]
// too-wide rows (small path off), [8] widest BITMAP span, [9] SMALL rows,
// [10] BITMAP rows, [11] rows promoted to long.
__global__ void wr_class_kernel(int32_t m, const int32_t *__restrict__ Arp, const int32_t *__restrict__ Acol,
                                const int32_t *__restrict__ Brp, const int32_t *__restrict__ Bcol,
                                const int64_t *__restrict__ S, uint8_t *__restrict__ rowlong,
                                int32_t *__restrict__ longflag, int32_t *__restrict__ lo_out,
                                int32_t *__restrict__ hi_out, uint8_t *__restrict__ wmode,
                                unsigned long long *__restrict__ stats, int small_on)
{
    const int lane = threadIdx.x & 31;
    const int64_t nwarps = int64_t(gridDim.x) * (blockDim.x >> 5);
    unsigned long long nwide = 0, mxspan = 0, nsmall = 0, nbitmap = 0, npromo = 0;
    for (int64_t r0 = (int64_t(blockIdx.x) * (blockDim.x >> 5) + (threadIdx.x >> 5)) * 32; r0 < m;
         r0 += nwarps * 32) {
        const int64_t r = r0 + lane;
        int mode = WM_NONE;
        int32_t a0 = 0, a1 = 0;
        bool need = false, fit = false;
        if (r < m && !rowlong[r]) {
            a0 = Arp[r];
            a1 = Arp[r + 1];
            const int64_t P = S[a1] - S[a0];
            fit = small_on && P <= WS_PMAX && a1 - a0 <= WS_BATCH;
            if (P > 0) {
                if (fit && P <= WS_ALWAYS) mode = WM_SMALL;
                else need = true;
            }
        }
        unsigned nb = __ballot_sync(0xffffffffu, need);
        while (nb) {
            const int src = __ffs(nb) - 1;
            nb &= nb - 1;
            const int32_t b_a0 = __shfl_sync(0xffffffffu, a0, src), b_a1 = __shfl_sync(0xffffffffu, a1, src);
            int32_t lo = INT_MAX, hi = -1;
            for (int32_t j = b_a0 + lane; j < b_a1; j += 32) {
                const int32_t k = Acol[j], b0 = Brp[k], b1 = Brp[k + 1];
                if (b1 > b0) {
                    lo = min(lo, Bcol[b0]);
                    hi = max(hi, Bcol[b1 - 1]);
                }
            }
            lo = __reduce_min_sync(0xffffffffu, lo);
            hi = __reduce_max_sync(0xffffffffu, hi);
            if (lane == src) {
                lo_out[r] = lo;
                hi_out[r] = hi;
                const unsigned long long sp = (unsigned long long)(int64_t(hi) - lo + 1);
                if (sp <= WR_SPAN) {
                    mode = WM_BITMAP;
                    mxspan = sp > mxspan ? sp : mxspan;
                } else if (fit) {
                    mode = WM_SMALL;
                } else if (small_on) {
                    rowlong[r] = 1;
                    longflag[r] = 1;
                    ++npromo;
                } else {
                    ++nwide;
                }
            }
        }
        if (r < m) wmode[r] = uint8_t(mode);
        nsmall += mode == WM_SMALL;
        nbitmap += mode == WM_BITMAP;
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        nwide += __shfl_xor_sync(0xffffffffu, nwide, o);
        mxspan = max(mxspan, __shfl_xor_sync(0xffffffffu, mxspan, o));
        nsmall += __shfl_xor_sync(0xffffffffu, nsmall, o);
        nbitmap += __shfl_xor_sync(0xffffffffu, nbitmap, o);
        npromo += __shfl_xor_sync(0xffffffffu, npromo, o);
    }
    if (lane == 0) {
        if (nwide) atomicAdd(stats + 7, nwide);
        if (mxspan) atomicMax(stats + 8, mxspan);
        if (nsmall) atomicAdd(stats + 9, nsmall);
        if (nbitmap) atomicAdd(stats + 10, nbitmap);
        if (npromo) atomicAdd(stats + 11, npromo);
    }
}

// ------------------------------------------------ small rows
// Rows with few products (C5's random rows: ~16; the uniform rows of C4) are
// too small for a warp each and too wide for a bitmap.  ESC in
// two passes per phase, so that the random B gathers and the per-row work
// never wait on each other:
//   expand (ws_expand_kernel): a thread per A nonzero j of a SMALL row
//     copies its B row's columns (symbolic) or the fp64 products
//     a_ik * b_kj, one rounding (numeric) to the product positions
//     [S[j], S[j+1]) of a staging array in main_ws -- positions follow
//     Gustavson's order (k ascending, then B's order); millions of
//     independent threads keep the B-row gathers in flight (setup recorded
//     each A nonzero's B row start, bstart[j], so no B offset is gathered);
//   compress (ws_small_kernel): a warp takes 32 rows (lane per row: mode,
//     offsets) and processes runs of consecutive SMALL rows with at most
//     WS_BATCH products together: their staged products come in with
//     coalesced loads (8 per lane in flight); then lane per product, rounds
//     of 32 positions.  Symbolic: a shared-memory hash set of (row, column)
//     counts each row's distinct columns (an insert that finds its own key is
//     a duplicate).  Numeric: a row whose C length equals P_r has no
//     duplicates and a product's rank is the number of smaller columns in its
//     row; otherwise first occurrences (no equal column earlier in the row)
//     are marked, each ranks among the marked columns and sums its column's
//     products in position (= k) order -- the oracle's order, separate
//     roundings -- and (c, sum) goes to C.rp[r] + rank.
// O(P_r) work per product, cheap for small rows; no sort.
#ifndef MSP_WS_WARPS
#define MSP_WS_WARPS 4
#endif
constexpr int WS_WARPS = MSP_WS_WARPS;
// WS_RANKS=1 (experiment): symbolic computes every product's rank in its row
// (smaller columns, one loop) and stores it as a byte next to the staged
// products, so numeric writes duplicate-free rows without a loop.  Measured on
// C5: symbolic compress 12.7 -> 24.2 ms, numeric 17.9 -> 12.1 ms (net slower);
// default 0: the symbolic hash count and the numeric rank loop.
#ifndef WS_RANKS
#define WS_RANKS 0
#endif
#ifndef WS_PAD
#define WS_PAD 0
#endif
constexpr int WS_HASH_BITS = 9;  // symbolic: 512-slot (row, column) hash set per warp (load <= 1/2)
constexpr int WS_HASH = 1 << WS_HASH_BITS;
constexpr unsigned long long WS_EMPTY = ~0ull;
// expand: product position S[j] + q of A nonzero j (in a SMALL row) gets
// B's column (symbolic) or the fp64 product a_ij * b_jq (numeric).
template <typename V, bool NUM>
__global__ void __launch_bounds__(256)
ws_expand_kernel(int64_t nnzA, const int32_t *__restrict__ arow, const uint8_t *__restrict__ wmode,
                 const int64_t *__restrict__ S, const int32_t *__restrict__ bstart, const V *__restrict__ Aval,
                 const int32_t *__restrict__ Bcol, const V *__restrict__ Bval, int32_t *__restrict__ X,
                 double *__restrict__ XV, int all_small)
{
    const int64_t stride = int64_t(gridDim.x) * blockDim.x;
    for (int64_t j = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; j < nnzA; j += stride) {
        // (every row with products small -- C5 -- needs no row lookup: the
        // nonzeros of other rows expand to nothing)
        if (!all_small && wmode[arow[j]] != WM_SMALL) continue;
        const int64_t s0 = S[j];
        const int len = int(S[j + 1] - s0);
        const int32_t b0 = bstart[j];
        if constexpr (!NUM) {
            for (int q = 0; q < len; q += 4) {
                int32_t c[4];
#pragma unroll
                for (int u = 0; u < 4; ++u) c[u] = (q + u < len) ? ldg64(Bcol + b0 + q + u) : 0;
#pragma unroll
                for (int u = 0; u < 4; ++u)
                    if (q + u < len) X[s0 + q + u] = c[u];
            }
        } else {
            const double a = double(Aval[j]);
            for (int q = 0; q < len; q += 4) {
                double v[4];
#pragma unroll
                for (int u = 0; u < 4; ++u) v[u] = (q + u < len) ? double(ldg64(Bval + b0 + q + u)) : 0.0;
#pragma unroll
                for (int u = 0; u < 4; ++u)
                    if (q + u < len) XV[s0 + q + u] = __dmul_rn(a, v[u]);
            }
        }
    }
}

template <typename V, bool NUM>
__global__ void __launch_bounds__(WS_WARPS * 32, (NUM && WS_PAD) ? 6 : 8)
ws_small_kernel(int32_t m, const int32_t *__restrict__ Arp, const uint8_t *__restrict__ wmode,
                const int64_t *__restrict__ S, const int32_t *__restrict__ X, const double *__restrict__ XV,
                uint8_t *__restrict__ XR, int32_t *__restrict__ Crp, int32_t *__restrict__ Ccol,
                V *__restrict__ Cval)
{
    constexpr unsigned FULL = 0xffffffffu;
    // WS_PAD (experiment): numeric stores each row at a 4-aligned start padded
    // with INT_MAX, so the rank loop reads 4 columns per shared load -- measured
    // slower on C5 (22.0 vs 18.6 ms: 80 registers, fewer warps), off
    constexpr bool PADDED = NUM && WS_PAD;
    constexpr int KCAP = PADDED ? WS_BATCH + 3 * 32 : WS_BATCH;
    __shared__ __align__(16) int32_t s_key_all[WS_WARPS][KCAP];  // column by (padded) batch position
    __shared__ __align__(16) uint8_t s_row_all[WS_WARPS][WS_BATCH];  // row lane of each batch position
    __shared__ int16_t s_slot_all[NUM ? 1 : WS_WARPS][NUM ? 1 : WS_BATCH];  // symbolic: hash slot of each product
    __shared__ unsigned s_first_all[NUM ? WS_WARPS : 1][KCAP / 32];         // numeric: first-occurrence bits
    __shared__ int s_cnt_all[WS_WARPS][32];                                   // symbolic: duplicates per row
    __shared__ unsigned long long s_hash_all[(NUM || WS_RANKS) ? 1 : WS_WARPS][(NUM || WS_RANKS) ? 1 : WS_HASH];
    __shared__ double s_val_all[NUM ? WS_WARPS : 1][NUM ? KCAP : 1];
    __shared__ uint8_t s_rank_all[(NUM && WS_RANKS) ? WS_WARPS : 1][(NUM && WS_RANKS) ? WS_BATCH : 1];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    int32_t *s_key = s_key_all[warp];
    uint8_t *s_row = s_row_all[warp];
    int16_t *s_slot = s_slot_all[NUM ? 0 : warp];
    unsigned long long *s_hash = s_hash_all[(NUM || WS_RANKS) ? 0 : warp];
    unsigned *s_first = s_first_all[NUM ? warp : 0];
    int *s_cnt = s_cnt_all[warp];
    double *s_val = s_val_all[NUM ? warp : 0];
    uint8_t *s_rank = s_rank_all[(NUM && WS_RANKS) ? warp : 0];
    const int64_t nwarps = int64_t(gridDim.x) * WS_WARPS;
    s_cnt[lane] = 0;
    reinterpret_cast<uint2 *>(s_row)[lane] = make_uint2(0u, 0u);
    if constexpr (!NUM && !WS_RANKS)
        for (int i = lane; i < WS_HASH; i += 32) s_hash[i] = WS_EMPTY;
    for (int64_t r0 = (int64_t(blockIdx.x) * WS_WARPS + warp) * 32; r0 < m; r0 += nwarps * 32) {
        const int64_t r = r0 + lane;
        bool sm = false;
        int32_t cb = 0;
        int64_t p0 = 0;
        int P = 0, U = 0;
        if (r < m && wmode[r] == WM_SMALL) {
            sm = true;
            p0 = S[Arp[r]];
            P = int(S[Arp[r + 1]] - p0);
            if (NUM) {
                cb = Crp[r];
                U = Crp[r + 1] - cb;  // == P: no duplicate columns in the row
            }
        }
        unsigned todo = __ballot_sync(FULL, sm);
        while (todo) {
            // batch: the run of consecutive SMALL lanes from s whose products fit
            const int s = __ffs(todo) - 1;
            const int64_t base = __shfl_sync(FULL, p0, s);
            const bool fits = sm && lane >= s && (p0 + P - base) <= WS_BATCH;
            const unsigned fm = __ballot_sync(FULL, fits) >> s;
            const int run = (~fm) ? __ffs(~fm) - 1 : 32 - s;
            const int e = s + run;  // lanes [s, e)
            todo &= ~unsigned(((1ull << run) - 1ull) << s);
            const int np = int(__shfl_sync(FULL, p0, e - 1) - base) + __shfl_sync(FULL, P, e - 1);
            const int prel = int(p0 - base);  // this lane's row start in the batch (lanes in [s, e))
            const bool inb = lane >= s && lane < e;
            // ---- the batch's staged products: coalesced, all loads in flight ----
            int32_t ck[WS_PPL];
            double cv[WS_PPL];
            uint32_t crk[WS_PPL];
#pragma unroll
            for (int u = 0; u < WS_PPL; ++u) {
                const int p = u * 32 + lane;
                ck[u] = p < np ? X[base + p] : 0;
                if constexpr (NUM) cv[u] = p < np ? XV[base + p] : 0.0;
                if constexpr (NUM && WS_RANKS) crk[u] = p < np ? XR[base + p] : 0u;
            }
            // ---- row lane of every position: start marks, blocked max-scan ----
            if (inb) s_row[prel] = uint8_t(lane + 1);
            __syncwarp();
            {
                const uint2 mk = reinterpret_cast<const uint2 *>(s_row)[lane];
                int v[8];
#pragma unroll
                for (int q = 0; q < 8; ++q) v[q] = int(((q < 4 ? mk.x : mk.y) >> (8 * (q & 3))) & 0xffu);
#pragma unroll
                for (int q = 1; q < 8; ++q) v[q] = max(v[q], v[q - 1]);
                int carry = v[7];
#pragma unroll
                for (int o = 1; o < 32; o <<= 1) {
                    const int t2 = __shfl_up_sync(FULL, carry, o);
                    if (lane >= o) carry = max(carry, t2);
                }
                int prev = __shfl_up_sync(FULL, carry, 1);
                if (lane == 0) prev = 0;
                uint32_t w0 = 0, w1 = 0;
#pragma unroll
                for (int q = 0; q < 8; ++q) {
                    const uint32_t b = uint32_t(max(v[q], prev) - 1) & 0xffu;  // 0-based row lane
                    if (q < 4) w0 |= b << (8 * q);
                    else w1 |= b << (8 * (q - 4));
                }
                __syncwarp();
                reinterpret_cast<uint2 *>(s_row)[lane] = make_uint2(w0, w1);
            }
            __syncwarp();
            // numeric: rows at 4-aligned starts (pstart), padded with INT_MAX
            int pstart = prel;
            if constexpr (PADDED) {
                const int pad = inb ? ((4 - (P & 3)) & 3) : 0;
                pstart = prel + warp_inclusive_sum(pad, lane) - pad;
                if (inb)
                    for (int q = 0; q < pad; ++q) s_key[pstart + P + q] = INT_MAX;
            }
#pragma unroll
            for (int u = 0; u < WS_PPL; ++u) {
                const int p = u * 32 + lane;
                const int t = p < np ? int(s_row[p]) : s;
                const int pp = PADDED ? __shfl_sync(FULL, pstart, t) + (p - __shfl_sync(FULL, prel, t)) : p;
                if (p < np) {
                    s_key[pp] = ck[u];
                    if constexpr (NUM) s_val[pp] = cv[u];
                    if constexpr (NUM && WS_RANKS) s_rank[p] = uint8_t(crk[u]);
                }
            }
            __syncwarp();
            // ---- C: compression, lane per product, rounds of 32 positions ----
            bool anydup = false;
            for (int pr = 0; pr < np; pr += 32) {
                const int p = pr + lane;
                const bool act = p < np;
                const int t = act ? int(s_row[p]) : s;  // the product's row lane
                if constexpr (!NUM && WS_RANKS) {
                    // one loop over the row: the product's rank (smaller
                    // columns) for numeric, and whether an earlier product of
                    // the row has the same column (a duplicate, not counted)
                    const int seg = __shfl_sync(FULL, prel, t);
                    const int len = __shfl_sync(FULL, P, t);
                    if (act) {
                        const int32_t c = s_key[p];
                        int less = 0;
                        bool dup = false;
                        for (int q = seg; q < seg + len; ++q) {
                            const int32_t kq = s_key[q];
                            less += kq < c ? 1 : 0;
                            dup = dup || (kq == c && q < p);
                        }
                        XR[base + p] = uint8_t(less);
                        if (dup) atomicAdd(&s_cnt[t], 1);
                    }
                } else if constexpr (!NUM) {
                    // distinct (row, column) pairs: insert into the warp's hash
                    // set; an insert that finds its own key is a duplicate
                    if (act) {
                        const int32_t c = s_key[p];
                        const unsigned long long key = (static_cast<unsigned long long>(t) << 32) | uint32_t(c);
                        uint32_t h = ((uint32_t(c) * 0x9E3779B1u) ^ (uint32_t(t) * 0x85EBCA77u)) >> (32 - WS_HASH_BITS);
                        while (true) {
                            const unsigned long long old = atomicCAS(&s_hash[h], WS_EMPTY, key);
                            if (old == WS_EMPTY) break;
                            if (old == key) {
                                atomicAdd(&s_cnt[t], 1);
                                break;
                            }
                            h = (h + 1) & (WS_HASH - 1);
                        }
                        s_slot[p] = int16_t(h);
                    }
                } else {
                    const int seg = __shfl_sync(FULL, pstart, t);
                    const int len = __shfl_sync(FULL, P, t);
                    const int32_t rowc = __shfl_sync(FULL, cb, t);
                    const int pp = seg + (p - __shfl_sync(FULL, prel, t));
                    const bool dupfree = __shfl_sync(FULL, U, t) == len;
                    anydup |= act && !dupfree;
                    if (act && dupfree) {
                        // rank = smaller columns in the row (4 per shared load; pads never count)
                        const int32_t c = s_key[pp];
                        int rk = 0;
                        if constexpr (WS_RANKS) {
                            rk = s_rank[p];  // from symbolic
                        } else if constexpr (PADDED) {
                            for (int q = seg; q < seg + len; q += 4) {
                                const int4 w = *reinterpret_cast<const int4 *>(s_key + q);
                                rk += int(w.x < c) + int(w.y < c) + int(w.z < c) + int(w.w < c);
                            }
                        } else {
                            for (int q = seg; q < seg + len; ++q) rk += s_key[q] < c ? 1 : 0;
                        }
                        Ccol[rowc + rk] = c;
                        Cval[rowc + rk] = V(s_val[pp]);
                    }
                }
            }
            if constexpr (!NUM && !WS_RANKS) {
                // clear the slots this batch used (a duplicate's probe ends on
                // its first occurrence's slot: cleared twice, harmlessly)
                __syncwarp();
                for (int p = lane; p < np; p += 32) s_hash[s_slot[p]] = WS_EMPTY;
            }
            if constexpr (NUM) {
                // rows with duplicate columns: mark first occurrences, then rank
                // among marked columns and sum each column's run in order
                if (__any_sync(FULL, anydup)) {
                    for (int i = lane; i < KCAP / 32; i += 32) s_first[i] = 0u;
                    __syncwarp();
                    for (int pr = 0; pr < np; pr += 32) {
                        const int p = pr + lane;
                        const int t = p < np ? int(s_row[p]) : s;
                        const int seg = __shfl_sync(FULL, pstart, t);
                        const int pp = seg + (p - __shfl_sync(FULL, prel, t));
                        const bool dup = __shfl_sync(FULL, U, t) != __shfl_sync(FULL, P, t);
                        if (p < np && dup) {
                            const int32_t c = s_key[pp];
                            bool first = true;
                            for (int q = seg; q < pp; ++q) first = first && (s_key[q] != c);
                            if (first) atomicOr(&s_first[pp >> 5], 1u << (pp & 31));
                        }
                    }
                    __syncwarp();
                    for (int pr = 0; pr < np; pr += 32) {
                        const int p = pr + lane;
                        const int t = p < np ? int(s_row[p]) : s;
                        const int seg = __shfl_sync(FULL, pstart, t);
                        const int len = __shfl_sync(FULL, P, t);
                        const int32_t rowc = __shfl_sync(FULL, cb, t);
                        const int pp = seg + (p - __shfl_sync(FULL, prel, t));
                        const bool dup = __shfl_sync(FULL, U, t) != len;
                        if (p < np && dup && ((s_first[pp >> 5] >> (pp & 31)) & 1u)) {
                            const int32_t c = s_key[pp];
                            int rk = 0;
                            double sum = s_val[pp];
                            for (int q = seg; q < seg + len; ++q) {
                                const int32_t kq = s_key[q];
                                const bool fq = (s_first[q >> 5] >> (q & 31)) & 1u;
                                rk += (fq && kq < c) ? 1 : 0;
                                if (kq == c && q > pp) sum = __dadd_rn(sum, s_val[q]);
                            }
                            Ccol[rowc + rk] = c;
                            Cval[rowc + rk] = V(sum);
                        }
                    }
                }
            }
            __syncwarp();
            reinterpret_cast<uint2 *>(s_row)[lane] = make_uint2(0u, 0u);  // marks of the next batch start clean
            __syncwarp();
        }
        if constexpr (!NUM) {
            __syncwarp();
            if (sm) Crp[r + 1] = P - s_cnt[lane];  // Crp holds the row offsets: row r's count goes to Crp[r + 1]
            s_cnt[lane] = 0;
            __syncwarp();
        }
    }
}

// One step per A nonzero of a chunk of <= 32 (lane l holds nonzero l's B
// row start b0 and length): f(step, c[u], v[u]) for 8 steps at a time, the
// 8 steps' B entries loaded up front (lane q holds entry q of the step's B
// row; rows longer than a warp take the per-step loop).  f runs in step
// order; `sync` adds a __syncwarp after every step (numeric ordering).
template <bool VALS, typename V, class F>
__device__ __forceinline__ void wr_steps(int nl, int lane, int32_t b0, int32_t len, const int32_t *__restrict__ Bcol,
                                         const V *__restrict__ Bval, bool sync, F &&f)
{
    if (__all_sync(0xffffffffu, len <= 32)) {
        for (int s0 = 0; s0 < nl; s0 += 8) {
            int32_t c[8];
            V v[8];
#pragma unroll
            for (int u = 0; u < 8; ++u) {
                const int sidx = (s0 + u) & 31;
                const int32_t bb = __shfl_sync(0xffffffffu, b0, sidx);
                const int32_t ll = __shfl_sync(0xffffffffu, len, sidx);
                const bool ok = s0 + u < nl && lane < ll;
                c[u] = ok ? Bcol[bb + lane] : -1;
                if constexpr (VALS) v[u] = ok ? Bval[bb + lane] : V(0);
            }
#pragma unroll
            for (int u = 0; u < 8; ++u) {
                f(s0 + u, c[u], VALS ? v[u] : V(0));
                if (sync) __syncwarp();
            }
        }
    } else {
        for (int sidx = 0; sidx < nl; ++sidx) {
            const int32_t bb = __shfl_sync(0xffffffffu, b0, sidx);
            const int32_t ll = __shfl_sync(0xffffffffu, len, sidx);
            for (int q0 = 0; q0 < ll; q0 += 32) {
                const bool ok = q0 + lane < ll;
                const int32_t c = ok ? Bcol[bb + q0 + lane] : -1;
                V v = V(0);
                if constexpr (VALS) v = ok ? Bval[bb + q0 + lane] : V(0);
                f(sidx, c, v);
            }
            if (sync) __syncwarp();
        }
    }
}

// Position of the n-th (0-based) set bit of w (w has more than n set bits).
__device__ __forceinline__ int nth_set_bit(uint32_t w, int n)
{
    int pos = 0;
#pragma unroll
    for (int sh = 16; sh >= 1; sh >>= 1) {
        const int c = __popc(w & ((1u << sh) - 1u));
        if (n >= c) {
            n -= c;
            w >>= sh;
            pos += sh;
        }
    }
    return pos;
}

// Symbolic: bitmap mark, then ONE pass over the bitmap (4 words per lane per
// round) counts the columns and writes them ascending at ucol + S[rp[r]].
__global__ void __launch_bounds__(WR_SYM_WARPS * 32, 1)
wr_symbolic_kernel(int32_t m, int nw_max, const int32_t *__restrict__ Arp, const int32_t *__restrict__ Acol,
                   const int32_t *__restrict__ Brp, const int32_t *__restrict__ Bcol,
                   const uint8_t *__restrict__ wmode, const int64_t *__restrict__ S,
                   const int32_t *__restrict__ spanlo, const int32_t *__restrict__ spanhi,
                   int32_t *__restrict__ Crp_counts, int32_t *__restrict__ ucol)
{
    extern __shared__ __align__(16) uint32_t wr_bm_all[];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    uint32_t *bm = wr_bm_all + size_t(warp) * nw_max;  // nw_max: a multiple of 128 words
    const int64_t nwarps = int64_t(gridDim.x) * WR_SYM_WARPS;
    for (int64_t r = int64_t(blockIdx.x) * WR_SYM_WARPS + warp; r < m; r += nwarps) {
        if (wmode[r] != WM_BITMAP) continue;  // long, small or without products (counts cleared)
        const int32_t lo = spanlo[r], hi = spanhi[r];
        const int nw = (hi - lo + 32) >> 5;
        const int nq = (nw + 127) >> 7;  // rounds of 4 words per lane
        for (int q = 0; q < nq; ++q) reinterpret_cast<uint4 *>(bm)[q * 32 + lane] = make_uint4(0u, 0u, 0u, 0u);
        __syncwarp();
        const int32_t a0 = Arp[r], a1 = Arp[r + 1];
        for (int32_t jc = a0; jc < a1; jc += 32) {
            const int32_t j = jc + lane;
            int32_t b0 = 0, len = 0;
            if (j < a1) {
                const int32_t k = Acol[j];
                b0 = Brp[k];
                len = Brp[k + 1] - b0;
            }
            wr_steps<false, float>(min(32, a1 - jc), lane, b0, len, Bcol, nullptr, false, [&](int, int32_t c, float) {
                if (c >= 0) {
                    const int x = c - lo;
                    atomicOr(&bm[x >> 5], 1u << (x & 31));
                }
            });
        }
        __syncwarp();
        int32_t *dst = ucol + S[a0];
        int run = 0;
        for (int q = 0; q < nq; ++q) {
            const uint4 w4 = reinterpret_cast<const uint4 *>(bm)[q * 32 + lane];
            const int p0 = __popc(w4.x), p1 = __popc(w4.y), p2 = __popc(w4.z), p3 = __popc(w4.w);
            int tot;
            const int ex = warp_excl_sum(p0 + p1 + p2 + p3, lane, &tot);
#if WR_EMIT_SERIAL
            // each lane emits its own words' set bits in order at ex + i
            // (lanes' runs are adjacent: the stores stay within a few lines)
            {
                int pos = run + ex;
                const uint32_t wv[4] = {w4.x, w4.y, w4.z, w4.w};
#pragma unroll
                for (int e = 0; e < 4; ++e) {
                    uint32_t bits = wv[e];
                    const int cbase = lo + (q * 128 + lane * 4 + e) * 32;
                    while (bits) {
                        const int bt = __ffs(bits) - 1;
                        bits &= bits - 1;
                        dst[pos++] = cbase + bt;
                    }
                }
            }
#else
            // the round's tot columns go out converged and coalesced: output o
            // (o = lane, lane + 32, ...) finds the lane owning it (last lane
            // with ex <= o), the word within that lane's four, and the bit
            for (int o0 = 0; o0 < tot; o0 += 32) {
                const int o = o0 + lane;
                int src_l = 0;
#pragma unroll
                for (int step = 16; step >= 1; step >>= 1) {
                    const int cand = src_l + step;
                    if (__shfl_sync(0xffffffffu, ex, cand) <= o) src_l = cand;
                }
                const int rel = o - __shfl_sync(0xffffffffu, ex, src_l);
                const uint32_t x0 = __shfl_sync(0xffffffffu, w4.x, src_l), x1 = __shfl_sync(0xffffffffu, w4.y, src_l);
                const uint32_t x2 = __shfl_sync(0xffffffffu, w4.z, src_l), x3 = __shfl_sync(0xffffffffu, w4.w, src_l);
                const int c0 = __popc(x0), c1 = c0 + __popc(x1), c2 = c1 + __popc(x2);
                int e, nth;
                uint32_t word;
                if (rel < c0) { e = 0; nth = rel; word = x0; }
                else if (rel < c1) { e = 1; nth = rel - c0; word = x1; }
                else if (rel < c2) { e = 2; nth = rel - c1; word = x2; }
                else { e = 3; nth = rel - c2; word = x3; }
                const int b = nth_set_bit(word, nth);
                if (o < tot) dst[run + o] = lo + (q * 128 + src_l * 4 + e) * 32 + b;
            }
#endif
            run += tot;
        }
        if (lane == 0) Crp_counts[r] = run;
        __syncwarp();  // the bitmap is reused by the warp's next row
    }
}

// Numeric: a hash of the row's column list (16-bit column offset | 16-bit
// rank per 32-bit slot, linear probing) gives each product's rank in one or
// two shared-memory probes; products accumulate into shared memory in k
// order.  WR_UMAX columns per pass.
constexpr int WR_HSLOTS = 1024;  // hash slots per warp (load <= 1/2 at WR_UMAX = 512)
constexpr uint32_t WR_EMPTY = 0xffffffffu;
constexpr int WR_NUM_SMEM = WR_NUM_WARPS * (WR_UMAX * 8 + WR_HSLOTS * 4);

__device__ __forceinline__ uint32_t wr_hash(uint32_t x) { return (x * 0x9E3779B1u) >> (32 - 10); }
static_assert(WR_HSLOTS == 1024, "wr_hash yields 10 bits");

template <typename V>
__global__ void __launch_bounds__(WR_NUM_WARPS * 32, MSP_WR_NUM_MINB)
wr_numeric_kernel(int32_t m, const int32_t *__restrict__ Arp, const int32_t *__restrict__ Acol,
                  const V *__restrict__ Aval, const int32_t *__restrict__ Brp, const int32_t *__restrict__ Bcol,
                  const V *__restrict__ Bval, const uint8_t *__restrict__ wmode, const int64_t *__restrict__ S,
                  const int32_t *__restrict__ spanlo, const int32_t *__restrict__ ucol,
                  const int32_t *__restrict__ Crp, int32_t *__restrict__ Ccol, V *__restrict__ Cval)
{
    extern __shared__ __align__(16) char wr_num_smem[];  // [warps][WR_UMAX] acc, then [warps][WR_HSLOTS] hash
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    double *acc = reinterpret_cast<double *>(wr_num_smem) + warp * WR_UMAX;
    uint32_t *tab = reinterpret_cast<uint32_t *>(wr_num_smem + WR_NUM_WARPS * WR_UMAX * 8) + warp * WR_HSLOTS;
    const int64_t nwarps = int64_t(gridDim.x) * WR_NUM_WARPS;
    // The next row's header, its list offset and the first 4 x 32 entries of
    // its column list are loaded while the current row accumulates (rows of
    // one warp are independent), hiding their latency chain.
    struct Hdr {
        int32_t cb, ce, a0, a1, lo, skip;
    };
    auto load_hdr = [&](int64_t rr) {
        Hdr h{0, 0, 0, 0, 0, 1};
        if (rr < m) {
            h.skip = wmode[rr] != WM_BITMAP;
            h.cb = Crp[rr];
            h.ce = Crp[rr + 1];
            h.a0 = Arp[rr];
            h.a1 = Arp[rr + 1];
            h.lo = spanlo[rr];
        }
        return h;
    };
    int64_t r = int64_t(blockIdx.x) * WR_NUM_WARPS + warp;
    Hdr cur = load_hdr(r);
    int64_t cur_off = (cur.skip || cur.ce == cur.cb) ? 0 : S[cur.a0];
    int32_t pre[4];  // entries lane + 32 u of the current row's column list
#pragma unroll
    for (int u = 0; u < 4; ++u) pre[u] = (lane + 32 * u < cur.ce - cur.cb) ? ucol[cur_off + lane + 32 * u] : 0;
    for (; r < m; r += nwarps) {
        const Hdr nxt = load_hdr(r + nwarps);
        const int32_t cb = cur.cb, U = cur.ce - cur.cb;
        const bool work = !cur.skip && U > 0;
        if (work) {
        const int32_t a0 = cur.a0, a1 = cur.a1;
        const int32_t lo = cur.lo;
        const int32_t *src = ucol + cur_off;
        // the first chunk of A nonzeros is loaded before the hash build, so
        // its dependent B-row offsets are in flight meanwhile (reused by
        // every column pass)
        int32_t f_b0 = 0, f_len = 0;
        double f_av = 0.0;
        {
            const int32_t j = a0 + lane;
            if (j < a1) {
                const int32_t k = Acol[j];
                f_av = double(Aval[j]);
                f_b0 = Brp[k];
                f_len = Brp[k + 1] - f_b0;
            }
        }
        for (int cs = 0; cs < U; cs += WR_UMAX) {
            const int nu = min(WR_UMAX, U - cs);
            for (int i = lane; i < WR_HSLOTS; i += 32) tab[i] = WR_EMPTY;
            for (int i = lane; i < nu; i += 32) acc[i] = -0.0;  // -0 + p == p for every p
            __syncwarp();
            auto insert = [&](int i, int32_t col) {
                const uint32_t x = uint32_t(col - lo);
                uint32_t h = wr_hash(x);
                while (atomicCAS(&tab[h], WR_EMPTY, x | (uint32_t(i) << 16)) != WR_EMPTY) h = (h + 1) & (WR_HSLOTS - 1);
            };
#pragma unroll
            for (int t = 0; t < 4; ++t) {
                const int i = lane + 32 * t;
                if (i < nu) insert(i, cs == 0 ? pre[t] : src[cs + i]);
            }
            for (int i = lane + 128; i < nu; i += 32) insert(i, src[cs + i]);
            __syncwarp();
            const int32_t cmin = src[cs], cmax = src[cs + nu - 1];
            for (int32_t jc = a0; jc < a1; jc += 32) {
                const int32_t j = jc + lane;
                int32_t b0 = f_b0, len = f_len;
                double av = f_av;
                if (jc != a0) {
                    b0 = 0;
                    len = 0;
                    av = 0.0;
                    if (j < a1) {
                        const int32_t k = Acol[j];
                        b0 = Brp[k];
                        len = Brp[k + 1] - b0;
                        av = double(Aval[j]);
                    }
                }
                wr_steps<true, V>(min(32, a1 - jc), lane, b0, len, Bcol, Bval, true, [&](int sidx, int32_t c, V v) {
                    const double a = __shfl_sync(0xffffffffu, av, sidx & 31);
                    if (c >= cmin && c <= cmax) {
                        const uint32_t x = uint32_t(c - lo);
                        uint32_t h = wr_hash(x), e;
                        while (((e = tab[h]) & 0xffffu) != x || e == WR_EMPTY) h = (h + 1) & (WR_HSLOTS - 1);
                        const int rk = int(e >> 16);
                        acc[rk] = __dadd_rn(acc[rk], __dmul_rn(a, double(v)));
                    }
                });
            }
            __syncwarp();
#pragma unroll
            for (int t = 0; t < 4; ++t) {
                const int i = lane + 32 * t;
                if (i < nu) {
                    Ccol[cb + cs + i] = cs == 0 ? pre[t] : src[cs + i];
                    Cval[cb + cs + i] = V(acc[i]);
                }
            }
            for (int i = lane + 128; i < nu; i += 32) {
                Ccol[cb + cs + i] = src[cs + i];
                Cval[cb + cs + i] = V(acc[i]);
            }
            __syncwarp();
        }
        }
        // the next row's list offset and first entries
        cur = nxt;
        cur_off = (cur.skip || cur.ce == cur.cb) ? 0 : S[cur.a0];
#pragma unroll
        for (int u = 0; u < 4; ++u) pre[u] = (lane + 32 * u < cur.ce - cur.cb) ? ucol[cur_off + lane + 32 * u] : 0;
    }
}

struct SetupWs {
    int32_t *arow;
    int64_t *S;          // [nnzA + 1]
    uint8_t *rowlong;    // [m]
    int32_t *longflag;   // [m]
    int64_t *longpos;    // [m + 1]
    int32_t *longrow;    // [m]
    int64_t *longP;      // [m]  (products of the i-th long row)
    int64_t *longO;      // [m + 1] prefix of longP
    int64_t *longC;      // [m]  chunks of the i-th long row
    int64_t *longCO;     // [m + 1] prefix of longC
    unsigned long long *stats;  // [16]: [0] max row products, [1..6] gathered setup sizes, [7] short rows
                                //       too wide for the row accumulator (small path off), [8] widest
                                //       BITMAP span, [9] SMALL rows, [10] BITMAP rows, [11] promoted rows
    int32_t *spanlo, *spanhi;   // [m] output column span of each long row (segmented path, f3)
    int32_t *spaflag;           // [m] windows of the row on the segmented path (0: not segmented)
    int64_t *spapos;            // [m + 1] exclusive scan of spaflag: first window item of each row
    int32_t *bstart;            // [nnzA] B row start of each A nonzero (Brp[Acol[j]])
    uint8_t *wmode;             // [m] warp-row path mode of each short row (WM_*)
    void *scan;
    size_t scan_bytes;
    size_t bytes;
};

SetupWs carve_setup(const msp_csr *A, void *ws, size_t cap, bool *ok)
{
    SetupWs w;
    const int64_t m = A->nrows, nnz = A->nnz;
    Carve cv(ws, cap);
    w.arow = cv.take<int32_t>(size_t(nnz > 0 ? nnz : 1));
    w.S = cv.take<int64_t>(size_t(nnz + 1));
    w.rowlong = cv.take<uint8_t>(size_t(m > 0 ? m : 1));
    w.longflag = cv.take<int32_t>(size_t(m > 0 ? m : 1));
    w.longpos = cv.take<int64_t>(size_t(m + 1));
    w.longrow = cv.take<int32_t>(size_t(m > 0 ? m : 1));
    w.longP = cv.take<int64_t>(size_t(m > 0 ? m : 1));
    w.longO = cv.take<int64_t>(size_t(m + 1));
    w.longC = cv.take<int64_t>(size_t(m > 0 ? m : 1));
    w.longCO = cv.take<int64_t>(size_t(m + 1));
    w.stats = cv.take<unsigned long long>(16);
    w.spanlo = cv.take<int32_t>(size_t(m > 0 ? m : 1));
    w.spanhi = cv.take<int32_t>(size_t(m > 0 ? m : 1));
    w.spaflag = cv.take<int32_t>(size_t(m > 0 ? m : 1));
    w.spapos = cv.take<int64_t>(size_t(m + 1));
    w.bstart = cv.take<int32_t>(size_t(nnz > 0 ? nnz : 1));
    w.wmode = cv.take<uint8_t>(size_t(m > 0 ? m : 1));
    w.scan_bytes = scan_ws_bytes(std::max<int64_t>(std::max<int64_t>(m, nnz), 1));
    w.scan = cv.take<char>(w.scan_bytes);
    w.bytes = cv.off;
    *ok = cv.ok();
    return w;
}

// ================================================================ main ====

struct GSplit {
    int64_t j, p;  // nonzero ends consumed, products consumed
};

__global__ void gemm_partition_kernel(int32_t m, int64_t nnzA, int64_t nprods, const int32_t *__restrict__ Arp,
                                      const int32_t *__restrict__ arow, const int64_t *__restrict__ S,
                                      const uint8_t *__restrict__ rowlong, int64_t ntiles, GSplit *__restrict__ splits)
{
    const int64_t total = nnzA + nprods;
    for (int64_t k = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; k <= ntiles; k += int64_t(gridDim.x) * blockDim.x) {
        const int64_t d = dmin(k * GM_TP, total);
        int64_t lo = dmax(0, d - nprods), hi = dmin(d, nnzA);
        while (lo < hi) {
            const int64_t mid = (lo + hi) >> 1;
            if (S[mid + 1] <= d - mid - 1) lo = mid + 1;
            else hi = mid;
        }
        GSplit s{lo, d - lo};
        if (lo < nnzA && d < total) {
            // snap to the nearest boundary of a short row (short rows never straddle)
            const int32_t r = arow[lo];
            if (!rowlong[r]) {
                const int64_t j_a = Arp[r], j_b = Arp[r + 1];
                const int64_t i_a = j_a + S[j_a], i_b = j_b + S[j_b];
                if (d > i_a && d < i_b) s = (d - i_a <= i_b - d) ? GSplit{j_a, S[j_a]} : GSplit{j_b, S[j_b]};
            }
        }
        splits[k] = s;
    }
}

// Key layouts: 64-bit (row offset << 32 | col) always works; 32-bit
// (row offset << cbits | col) is used when every tile's row span fits,
// halving the staging / sort shared memory (2 CTAs per SM) and compare cost.
template <typename KT>
struct KeyOps;
template <>
struct KeyOps<uint64_t> {
    static constexpr uint64_t MASKED = ~0ull;
    static constexpr uint64_t NONE = 1ull << 63;  // never equal to a real key
    __device__ static uint64_t make(uint32_t r, uint32_t c, int) { return (uint64_t(r) << 32) | c; }
    __device__ static uint32_t row(uint64_t k, int) { return uint32_t(k >> 32); }
    __device__ static uint32_t col(uint64_t k, int) { return uint32_t(k); }
};
template <>
struct KeyOps<uint32_t> {
    static constexpr uint32_t MASKED = ~0u;
    static constexpr uint32_t NONE = ~0u - 1u;  // real keys stay below (tile_span_ok)
    __device__ static uint32_t make(uint32_t r, uint32_t c, int cb) { return (r << cb) | c; }
    __device__ static uint32_t row(uint32_t k, int cb) { return k >> cb; }
    __device__ static uint32_t col(uint32_t k, int cb) { return k & ((1u << cb) - 1u); }
};

// Shared memory of one tile.  Symbolic: the staging buffer (keys by product
// slot) is reused by the sort.  Numeric: staging keys + product values only
// (the permutation comes from the symbolic pass).
template <typename KT, bool NUM>
struct TileKeys {
    union {
        KT stage[GM_T];
        BlockSortSmem<GM_NT, GM_IPT, KT> sort;
    };
};
template <>
struct TileKeys<uint32_t, false> {
    union {
        uint32_t stage[GM_T];
        BlockSortSmem<GM_NT, GM_IPT, uint32_t> sort;
        RunSortSmem<GM_T, uint32_t> rm;
    };
};
template <typename KT>
struct TileKeys<KT, true> {
    KT stage[GM_T];
};
// symbolic with 32-bit keys: run table of the run-aware sort (64-bit keys
// keep the generic sort: their larger state would spill at 2 CTAs/SM)
template <typename KT, bool NUM> struct TileRuns { char t; };
template <> struct TileRuns<uint32_t, false> { RunTable t; };
template <typename KT, bool NUM>
struct TileSmem {
    TileKeys<KT, NUM> keys;
    TileRuns<KT, NUM> runs;
    double vals[NUM ? GM_T : 1];
    KT edge_first[GM_NT];
    KT edge_last[GM_NT];
    SegPair<double> scan_w[GM_NT / 32];
    int32_t wsum[GM_NT / 32];
};

__device__ __forceinline__ unsigned long long warp_reduce_max_u64(unsigned long long v)
{
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        const unsigned long long t = __shfl_xor_sync(0xffffffffu, v, o);
        v = v > t ? v : t;
    }
    return v;
}

// Largest row span of any tile (decides the key width for the whole launch).
__global__ void tile_span_kernel(int64_t ntiles, const GSplit *__restrict__ splits, const int32_t *__restrict__ arow,
                                 unsigned long long *__restrict__ maxspan)
{
    unsigned long long mx = 0;
    for (int64_t k = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; k < ntiles; k += int64_t(gridDim.x) * blockDim.x) {
        const GSplit s0 = splits[k], s1 = splits[k + 1];
        if (s1.p == s0.p) continue;
        const int64_t nz = s1.j - s0.j;
        const int64_t span = nz > 0 ? int64_t(arow[s0.j + nz - 1]) - arow[s0.j] + 1 : 1;
        mx = mx > (unsigned long long)span ? mx : (unsigned long long)span;
    }
    mx = warp_reduce_max_u64(mx);
    if ((threadIdx.x & 31) == 0 && mx) atomicMax(maxspan, mx);
}

// Symbolic: sort the staged keys and store the tile's sorting permutation;
// numeric: apply the stored permutation instead of sorting again (the paper
// keeps the CTA sort's permutation in global memory and re-expands the
// products into it).  Then compress (see kernel).
template <typename KT, bool NUM, typename V>
__device__ __forceinline__ void sort_compress(TileSmem<KT, NUM> &Sm, int np, int32_t rbase, int cbits,
                                              uint16_t *__restrict__ tperm, int32_t *__restrict__ Crp,
                                              int32_t *__restrict__ Ccol, V *__restrict__ Cval)
{
    using O = KeyOps<KT>;
    const int tid = threadIdx.x;
    KT k[GM_IPT];
    int v[GM_IPT];
    static_assert(GM_IPT == 16 && GM_T <= 65536, "permutation packing");
    uint4 *pp = reinterpret_cast<uint4 *>(tperm + tid * GM_IPT);
    if constexpr (!NUM) {
        // products arrive as sorted B-row runs grouped by row: merge runs
        // within rows; the generic block sort is the fallback for tiles with
        // very many runs
        bool sorted = false;
        if constexpr (sizeof(KT) == 4)
            sorted = run_merge_sort<GM_NT, GM_IPT, KT>(Sm.keys.stage, np, Sm.keys.rm, Sm.runs.t, Sm.wsum,
                                                       [&](KT kk) { return O::row(kk, cbits); }, k, v);
        if (!sorted) {
#pragma unroll
            for (int u = 0; u < GM_IPT; ++u) {
                const int slot = tid + u * GM_NT;
                k[u] = slot < np ? Sm.keys.stage[slot] : O::MASKED;
                v[u] = slot;
            }
            __syncthreads();  // staging is reused by the sort
            block_merge_sort<GM_NT, GM_IPT, KT>(k, v, Sm.keys.sort);
        }
        uint32_t w[GM_IPT / 2];
#pragma unroll
        for (int i = 0; i < GM_IPT / 2; ++i) w[i] = uint32_t(v[2 * i]) | (uint32_t(v[2 * i + 1]) << 16);
        pp[0] = make_uint4(w[0], w[1], w[2], w[3]);
        pp[1] = make_uint4(w[4], w[5], w[6], w[7]);
    } else {
        const uint4 q0 = pp[0], q1 = pp[1];
        const uint32_t w[GM_IPT / 2] = {q0.x, q0.y, q0.z, q0.w, q1.x, q1.y, q1.z, q1.w};
#pragma unroll
        for (int i = 0; i < GM_IPT; ++i) {
            const int pos = tid * GM_IPT + i;
            const int slot = int((w[i >> 1] >> ((i & 1) * 16)) & 0xffffu);
            // masked (long-row) products and padding share the MASKED key, so a
            // position < np may hold a padding slot >= np
            k[i] = (pos < np && slot < np) ? Sm.keys.stage[slot] : O::MASKED;
            v[i] = slot;
        }
    }
    // neighbours across thread boundaries
    Sm.edge_first[tid] = k[0];
    Sm.edge_last[tid] = k[GM_IPT - 1];
    __syncthreads();
    const KT prevk = tid > 0 ? Sm.edge_last[tid - 1] : O::NONE;
    const KT nextk = tid + 1 < GM_NT ? Sm.edge_first[tid + 1] : O::NONE;
    auto newrow = [&](KT pk, KT kk) { return pk == O::MASKED || pk == O::NONE || O::row(pk, cbits) != O::row(kk, cbits); };

    if constexpr (!NUM) {
        // ---- unique count per row (rows are complete in the tile) ----
        KT pk = prevk;
        int cnt = 0;
        int64_t row = -1;
#pragma unroll
        for (int i = 0; i < GM_IPT; ++i) {
            if (k[i] != O::MASKED) {
                const int64_t r = int64_t(rbase) + int64_t(O::row(k[i], cbits));
                if (r != row) {
                    if (cnt) atomicAdd(&Crp[row + 1], cnt);
                    cnt = 0;
                    row = r;
                }
                if (k[i] != pk) ++cnt;
            }
            pk = k[i];
        }
        if (cnt) atomicAdd(&Crp[row + 1], cnt);
    } else {
        // ---- unique (col, sum): position = C.rp[row] + rank of the key in its row ----
        int heads = 0, last_rs = -1;  // heads in this thread; heads before its last row start
        double trail = 0.0;           // sum after the last head in this thread
        {
            KT pk = prevk;
#pragma unroll
            for (int i = 0; i < GM_IPT; ++i) {
                if (k[i] != O::MASKED) {
                    const double val = Sm.vals[v[i]];
                    if (k[i] != pk) {
                        if (newrow(pk, k[i])) last_rs = heads;
                        ++heads;
                        trail = val;
                    } else {
                        trail = trail + val;
                    }
                }
                pk = k[i];
            }
        }
        int tot;
        const int u0 = block_exclusive_sum<int, GM_NT / 32>(heads, Sm.wsum, 0, &tot);
        SegPair<double> all;
        const SegPair<double> carry =
            block_seg_exclusive<double, GM_NT / 32>(SegPair<double>{heads > 0, trail}, SegPair<double>{0, 0.0},
                                                    Sm.scan_w, 0, &all);
        // tile rank of the first key of the row open at this thread's start
        const int rs_carry = block_exclusive_max<GM_NT / 32>(last_rs >= 0 ? u0 + last_rs : -1, Sm.wsum, 0);
        KT pk = prevk;
        int u = u0 - 1, row_u = rs_carry;
        double run = carry.v;
#pragma unroll
        for (int i = 0; i < GM_IPT; ++i) {
            if (k[i] != O::MASKED) {
                const double val = Sm.vals[v[i]];
                if (k[i] != pk) {
                    ++u;
                    if (newrow(pk, k[i])) row_u = u;
                    run = val;
                } else {
                    run = run + val;
                }
                const KT nk = (i + 1 < GM_IPT) ? k[i + 1] : nextk;
                if (nk != k[i]) {  // run ends here
                    const int64_t row = int64_t(rbase) + int64_t(O::row(k[i], cbits));
                    const int64_t pos = int64_t(Crp[row]) + (u - row_u);
                    Ccol[pos] = int32_t(O::col(k[i], cbits));
                    Cval[pos] = V(run);
                }
            }
            pk = k[i];
        }
    }
}

// One CTA per tile: expand -> sort by (row, col) -> compress.  Products are
// expanded in merge-path order (each thread finds its split of the tile's
// (nonzero ends, products) once, then walks), staged by product index, sorted
// (symbolic; the permutation is kept for numeric), reduced with head flags.
// Symbolic: unique counts per row into C.row_offsets.  Numeric: (col, sum) at
// C.row_offsets[row] + rank in row.
template <typename KT, typename V, bool NUM>
__global__ void __launch_bounds__(GM_NT, 2)
gemm_tile_kernel(const int32_t *__restrict__ Acol, const V *__restrict__ Aval, const int32_t *__restrict__ Brp,
                 const int32_t *__restrict__ Bcol, const V *__restrict__ Bval, const int32_t *__restrict__ arow,
                 const int64_t *__restrict__ S, const uint8_t *__restrict__ rowlong, const GSplit *__restrict__ splits,
                 int cbits, uint16_t *__restrict__ perm, int32_t *__restrict__ Crp, int32_t *__restrict__ Ccol,
                 V *__restrict__ Cval)
{
    using O = KeyOps<KT>;
    extern __shared__ __align__(16) char smem_raw[];
    TileSmem<KT, NUM> &Sm = *reinterpret_cast<TileSmem<KT, NUM> *>(smem_raw);
    const int tid = threadIdx.x;
    const GSplit s0 = splits[blockIdx.x], s1 = splits[blockIdx.x + 1];
    const int64_t j0 = s0.j, p0 = s0.p;
    const int nz = int(s1.j - j0), np = int(s1.p - p0);
    if (np == 0) return;
    const int32_t rbase = arow[j0];
    {   // a tile inside one long / segmented row has nothing to do (its
        // products are handled by the long-row or segmented pass)
        const int64_t jl = (S[s1.j] < s1.p) ? s1.j : s1.j - 1;  // nonzero of the tile's last product
        if (rowlong[rbase] && arow[jl] == rbase) return;
    }
    // ---- expansion: merge path over (nonzero ends, products) of the tile ----
    {
        const int items = nz + np;
        const int dt = min(tid * GM_IPT, items);
        int lo = max(0, dt - np), hi = min(dt, nz);
        while (lo < hi) {
            const int mid = (lo + hi) >> 1;
            if (S[j0 + mid + 1] - p0 <= dt - mid - 1) lo = mid + 1;
            else hi = mid;
        }
        int64_t j = j0 + lo;
        int64_t p = p0 + (dt - lo);
        const int64_t jend = j0 + nz;
        const int todo = min(GM_IPT, items - dt);
        int64_t sj1 = (j < jend) ? S[j + 1] : INT64_MAX;
        int64_t bofs = 0;
        uint32_t rofs = 0;
        bool masked = true;
        double av = 0.0;
        bool loaded = false;
        for (int q = 0; q < todo; ++q) {
            if (j < jend && sj1 <= p) {  // nonzero j ends
                ++j;
                sj1 = (j < jend) ? S[j + 1] : INT64_MAX;
                loaded = false;
                continue;
            }
            if (!loaded) {
                const int32_t r = arow[j];
                masked = rowlong[r] != 0;
                rofs = uint32_t(r - rbase);
                const int32_t kk = Acol[j];
                bofs = int64_t(Brp[kk]) - S[j];
                if (NUM) av = double(Aval[j]);
                loaded = true;
            }
            const int slot = int(p - p0);
            const int64_t bi = bofs + p;
            Sm.keys.stage[slot] = masked ? O::MASKED : O::make(rofs, uint32_t(Bcol[bi]), cbits);
            if (NUM) Sm.vals[slot] = av * double(Bval[bi]);
            ++p;
        }
    }
    __syncthreads();
    sort_compress<KT, NUM, V>(Sm, np, rbase, cbits, perm + size_t(blockIdx.x) * GM_T, Crp, Ccol, Cval);
}

// ---------------------------------------------------------- long rows ----

template <typename V, bool NUM>
struct LongSmem {
    BlockSortSmem<GM_NT, GM_IPT> sort;
    double vals[NUM ? GM_TL : 1];
};

// Chunk c of long row l: expand products [c*TL, ...) of the row, sort by
// column (stable), write the sorted run at longO[l] + c*TL.
template <typename V, bool NUM>
__global__ void __launch_bounds__(GM_NT)
long_chunk_kernel(const int32_t *__restrict__ Arp, const int32_t *__restrict__ Acol, const V *__restrict__ Aval,
                  const int32_t *__restrict__ Brp, const int32_t *__restrict__ Bcol, const V *__restrict__ Bval,
                  const int64_t *__restrict__ S, int64_t nlong, const int32_t *__restrict__ longrow,
                  const int64_t *__restrict__ longP, const int64_t *__restrict__ longO,
                  const int64_t *__restrict__ longCO, int32_t *__restrict__ Xcol, double *__restrict__ Xval)
{
    extern __shared__ __align__(16) char smem_raw[];
    LongSmem<V, NUM> &Sm = *reinterpret_cast<LongSmem<V, NUM> *>(smem_raw);
    const int tid = threadIdx.x;
    const int64_t b = blockIdx.x;
    int64_t lo = 0, hi = nlong;  // l: last with longCO[l] <= b
    while (hi - lo > 1) {
        const int64_t mid = (lo + hi) >> 1;
        if (longCO[mid] <= b) lo = mid;
        else hi = mid;
    }
    const int64_t l = lo;
    const int64_t c = b - longCO[l];
    const int32_t r = longrow[l];
    const int64_t P = longP[l];
    const int64_t q0 = c * GM_TL;
    const int nq = int(dmin(GM_TL, P - q0));
    const int64_t ja = Arp[r], jb = Arp[r + 1];
    const int64_t pr0 = S[ja];  // global product index of the row's first product
    uint64_t k[GM_IPT];
    int v[GM_IPT];
    {
        const int64_t qs = q0 + int64_t(tid) * GM_IPT;
        // nonzero of product pr0 + qs: last j in [ja, jb) with S[j] <= pr0 + qs
        int64_t j = ja;
        if (qs < P) {
            int64_t lo2 = ja, hi2 = jb;
            const int64_t pg = pr0 + qs;
            while (hi2 - lo2 > 1) {
                const int64_t mid = (lo2 + hi2) >> 1;
                if (S[mid] <= pg) lo2 = mid;
                else hi2 = mid;
            }
            j = lo2;
        }
        int64_t sj1 = S[j + 1];
        int64_t bofs = int64_t(Brp[Acol[j]]) - S[j];
        double av = NUM ? double(Aval[j]) : 0.0;
#pragma unroll
        for (int i = 0; i < GM_IPT; ++i) {
            const int64_t q = qs + i;
            const int slot = tid * GM_IPT + i;
            v[i] = slot;
            if (q < q0 + nq) {
                const int64_t pg = pr0 + q;
                while (sj1 <= pg) {  // skip to the nonzero holding product pg
                    ++j;
                    sj1 = S[j + 1];
                    bofs = int64_t(Brp[Acol[j]]) - S[j];
                    if (NUM) av = double(Aval[j]);
                }
                const int64_t bi = bofs + pg;
                k[i] = uint32_t(Bcol[bi]);
                if (NUM) Sm.vals[slot] = av * double(Bval[bi]);
            } else {
                k[i] = KEY_MASKED;
            }
        }
    }
    __syncthreads();
    block_merge_sort<GM_NT, GM_IPT>(k, v, Sm.sort);
    const int64_t out = longO[l] + q0;
#pragma unroll
    for (int i = 0; i < GM_IPT; ++i) {
        const int pos = tid * GM_IPT + i;
        if (pos < nq) {
            Xcol[out + pos] = int32_t(k[i]);
            if (NUM) Xval[out + pos] = Sm.vals[v[i]];
        }
    }
}

// One merge pass: runs of `w` entries inside each long row are merged
// pairwise (stable, left run first).  Outputs [e, e_end) by one thread: a
// merge-path search in global memory, then a serial merge (the fallback for
// CTAs whose output range crosses a pair or a row boundary).
template <bool NUM>
__device__ __forceinline__ void long_merge_thread(int64_t e, int64_t e_end, int64_t nlong,
                                                  const int64_t *__restrict__ longO, const int64_t *__restrict__ longP,
                                                  int64_t w, const int32_t *__restrict__ Xc,
                                                  const double *__restrict__ Xv, int32_t *__restrict__ Yc,
                                                  double *__restrict__ Yv)
{
    while (e < e_end) {
        int64_t lo = 0, hi = nlong;
        while (hi - lo > 1) {
            const int64_t mid = (lo + hi) >> 1;
            if (longO[mid] <= e) lo = mid;
            else hi = mid;
        }
        const int64_t O = longO[lo], P = longP[lo];
        const int64_t q = e - O;
        const int64_t a0 = (q / (2 * w)) * (2 * w);
        const int64_t la = dmin(w, P - a0);
        const int64_t lb = dmax(0, dmin(w, P - a0 - la));
        const int64_t d = q - a0;
        const int64_t A0 = O + a0, B0 = O + a0 + la;
        int64_t l2 = dmax(0, d - lb), h2 = dmin(d, la);
        while (l2 < h2) {
            const int64_t mid = (l2 + h2) >> 1;
            if (Xc[A0 + mid] <= Xc[B0 + d - mid - 1]) l2 = mid + 1;
            else h2 = mid;
        }
        int64_t ia = l2, ib = d - l2;
        const int64_t n = dmin(e_end - e, la + lb - d);
        for (int64_t t = 0; t < n; ++t) {
            const bool ta = ib >= lb || (ia < la && Xc[A0 + ia] <= Xc[B0 + ib]);
            if (ta) {
                Yc[e + t] = Xc[A0 + ia];
                if (NUM) Yv[e + t] = Xv[A0 + ia];
                ++ia;
            } else {
                Yc[e + t] = Xc[B0 + ib];
                if (NUM) Yv[e + t] = Xv[B0 + ib];
                ++ib;
            }
        }
        e += n;
    }
}

// CTA-level merge pass (P:1154-1170 global merge of the sorted runs): each CTA
// owns LM_T consecutive outputs.  When they lie inside one pair of runs (the
// common case: pairs are >= 2 * GM_TL = 16K long), two merge-path searches
// bound the CTA's windows of both runs, the windows are staged in shared
// memory with coalesced loads, and every thread merges 16 outputs from shared
// memory; other CTAs fall back to the per-thread merge.
constexpr int LM_NT = 256, LM_IPT = 12, LM_T = LM_NT * LM_IPT;  // 36 KB of static shared memory

template <bool NUM>
__global__ void __launch_bounds__(LM_NT)
long_merge_kernel(int64_t LP, int64_t nlong, const int64_t *__restrict__ longO, const int64_t *__restrict__ longP,
                  int64_t w, const int32_t *__restrict__ Xc, const double *__restrict__ Xv, int32_t *__restrict__ Yc,
                  double *__restrict__ Yv)
{
    __shared__ int32_t sc[LM_T];
    __shared__ double sv[NUM ? LM_T : 1];
    __shared__ int64_t sA, sB, sna, snb;
    __shared__ int sfast;
    const int tid = threadIdx.x;
    const int64_t e0 = int64_t(blockIdx.x) * LM_T, e1 = dmin(e0 + LM_T, LP);
    if (tid == 0) {
        int64_t lo = 0, hi = nlong;
        while (hi - lo > 1) {
            const int64_t mid = (lo + hi) >> 1;
            if (longO[mid] <= e0) lo = mid;
            else hi = mid;
        }
        const int64_t O = longO[lo], P = longP[lo];
        const int64_t a0 = ((e0 - O) / (2 * w)) * (2 * w);
        const int64_t la = dmin(w, P - a0);
        const int64_t lb = dmax(0, dmin(w, P - a0 - la));
        const int64_t A0 = O + a0, B0 = A0 + la;
        sfast = (e1 <= A0 + la + lb) ? 1 : 0;
        if (sfast) {
            auto split = [&](int64_t d) {
                int64_t l2 = dmax(0, d - lb), h2 = dmin(d, la);
                while (l2 < h2) {
                    const int64_t mid = (l2 + h2) >> 1;
                    if (Xc[A0 + mid] <= Xc[B0 + d - mid - 1]) l2 = mid + 1;
                    else h2 = mid;
                }
                return l2;
            };
            const int64_t d0 = e0 - A0, d1 = e1 - A0;
            const int64_t i0 = split(d0), i1 = split(d1);
            sA = A0 + i0;
            sB = B0 + (d0 - i0);
            sna = i1 - i0;
            snb = (d1 - i1) - (d0 - i0);
        }
    }
    __syncthreads();
    if (!sfast) {
        const int64_t e = e0 + int64_t(tid) * LM_IPT;
        long_merge_thread<NUM>(e, dmin(e + LM_IPT, e1), nlong, longO, longP, w, Xc, Xv, Yc, Yv);
        return;
    }
    const int na = int(sna), nb = int(snb);
    const int64_t gA = sA, gB = sB;
    for (int x = tid; x < na + nb; x += LM_NT) {
        const int64_t g = x < na ? gA + x : gB + (x - na);
        sc[x] = Xc[g];
        if (NUM) sv[x] = Xv[g];
    }
    __syncthreads();
    const int d = min(tid * LM_IPT, na + nb);
    int lo = max(0, d - nb), hi = min(d, na);
    while (lo < hi) {
        const int mid = (lo + hi) >> 1;
        if (sc[mid] <= sc[na + d - mid - 1]) lo = mid + 1;
        else hi = mid;
    }
    int ia = lo, ib = d - lo;
    const int n = min(LM_IPT, na + nb - d);
    const int64_t out = e0 + d;
    for (int t = 0; t < n; ++t) {
        const bool ta = ib >= nb || (ia < na && sc[ia] <= sc[na + ib]);
        const int src = ta ? ia : na + ib;
        Yc[out + t] = sc[src];
        if (NUM) Yv[out + t] = sv[src];
        ia += ta ? 1 : 0;
        ib += ta ? 0 : 1;
    }
}

// Head flags of the sorted long rows; symbolic adds per-row unique counts.
__global__ void long_heads_kernel(int64_t LP, int64_t nlong, const int64_t *__restrict__ longO,
                                  const int32_t *__restrict__ longrow, const int32_t *__restrict__ Fc,
                                  int32_t *__restrict__ heads, int32_t *__restrict__ Crp_counts)
{
    const int64_t e0 = (int64_t(blockIdx.x) * blockDim.x + threadIdx.x) * 16;
    if (e0 >= LP) return;
    int64_t lo = 0, hi = nlong;
    while (hi - lo > 1) {
        const int64_t mid = (lo + hi) >> 1;
        if (longO[mid] <= e0) lo = mid;
        else hi = mid;
    }
    int64_t l = lo;
    int64_t rowend = (l + 1 < nlong) ? longO[l + 1] : LP;
    int cnt = 0;
    const int64_t e1 = dmin(e0 + 16, LP);
    for (int64_t e = e0; e < e1; ++e) {
        while (e >= rowend) {
            if (cnt && Crp_counts) atomicAdd(&Crp_counts[longrow[l]], cnt);
            cnt = 0;
            ++l;
            rowend = (l + 1 < nlong) ? longO[l + 1] : LP;
        }
        const int h = (e == longO[l] || Fc[e] != Fc[e - 1]) ? 1 : 0;
        if (heads) heads[e] = h;
        cnt += h;
    }
    if (cnt && Crp_counts) atomicAdd(&Crp_counts[longrow[l]], cnt);
}

// Numeric: every head writes (col, sum of its run) at C.rp[row] + rank.
template <typename V>
__global__ void long_emit_kernel(int64_t LP, int64_t nlong, const int64_t *__restrict__ longO,
                                 const int32_t *__restrict__ longrow, const int32_t *__restrict__ Fc,
                                 const double *__restrict__ Fv, const int32_t *__restrict__ heads,
                                 const int64_t *__restrict__ U, const int32_t *__restrict__ Crp,
                                 int32_t *__restrict__ Ccol, V *__restrict__ Cval)
{
    for (int64_t e = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; e < LP; e += int64_t(gridDim.x) * blockDim.x) {
        if (!heads[e]) continue;
        int64_t lo = 0, hi = nlong;
        while (hi - lo > 1) {
            const int64_t mid = (lo + hi) >> 1;
            if (longO[mid] <= e) lo = mid;
            else hi = mid;
        }
        const int64_t O = longO[lo];
        const int64_t rowend = (lo + 1 < nlong) ? longO[lo + 1] : LP;
        const int64_t pos = int64_t(Crp[longrow[lo]]) + (U[e] - U[O]);
        double s = Fv[e];
        for (int64_t e2 = e + 1; e2 < rowend && !heads[e2]; ++e2) s = s + Fv[e2];
        Ccol[pos] = Fc[e];
        Cval[pos] = V(s);
    }
}

struct MainWs {
    GSplit *splits;
    uint16_t *perm;  // per tile: the symbolic sort's permutation (GM_T entries)
    int32_t *ucol;   // row-accumulator path: each short row's output columns at its product offset
    int32_t *xcol;   // small-row path: B column of every product (symbolic expand; numeric reads it)
    double *xval;    // small-row path: every product a_ik * b_kj (numeric expand)
    uint8_t *xrank;  // small-row path: every product's rank in its row (symbolic compress)
    int32_t *spawcnt;  // segmented path: output count of every window (symbolic; numeric's offsets)
    int32_t *Xc[2];
    double *Xv[2];
    int32_t *heads;
    int64_t *U;
    int64_t *totals;
    void *scan;
    size_t scan_bytes;
    size_t bytes;
};

MainWs carve_main(int64_t m, int64_t ntiles, int64_t LP, int64_t nucol, int64_t nx, int64_t nspa, void *ws,
                  size_t cap, bool *ok)
{
    MainWs w;
    Carve cv(ws, cap);
    w.splits = cv.take<GSplit>(size_t(ntiles + 1));
    w.perm = cv.take<uint16_t>(size_t(ntiles) * GM_T);
    w.ucol = cv.take<int32_t>(size_t(nucol > 0 ? nucol : 1));
    w.xcol = cv.take<int32_t>(size_t(nx > 0 ? nx : 1));
    w.xval = cv.take<double>(size_t(nx > 0 ? nx : 1));
    w.xrank = cv.take<uint8_t>(size_t((WS_RANKS && nx > 0) ? nx : 1));
    w.spawcnt = cv.take<int32_t>(size_t(nspa > 0 ? nspa : 1));
    for (int i = 0; i < 2; ++i) {
        w.Xc[i] = cv.take<int32_t>(size_t(LP > 0 ? LP : 1));
        w.Xv[i] = cv.take<double>(size_t(LP > 0 ? LP : 1));
    }
    w.heads = cv.take<int32_t>(size_t(LP > 0 ? LP : 1));
    w.U = cv.take<int64_t>(size_t(LP + 1));
    w.totals = cv.take<int64_t>(4);
    w.scan_bytes = scan_ws_bytes(std::max<int64_t>(std::max<int64_t>(m, LP), 1));
    w.scan = cv.take<char>(w.scan_bytes);
    w.bytes = cv.off;
    *ok = cv.ok();
    return w;
}

struct HostInfo {  // read back by setup (one synchronisation), passed to symbolic / numeric in msp_spgemm_info
    int64_t nprods, nlong, LP, LC, maxP, nspa, rowacc, nsmall, nbitmap;
};

// The setup sizes gathered into one device array (so setup reads them back
// with ONE copy and one synchronisation): S[nnzA], longpos[m], longO[nlong],
// longCO[nlong], max row products.
__global__ void info_gather_kernel(const int64_t *__restrict__ S, int64_t nnzA, const int64_t *__restrict__ longpos,
                                   int64_t m, const int64_t *__restrict__ longO, const int64_t *__restrict__ longCO,
                                   const unsigned long long *__restrict__ stats, const int64_t *__restrict__ spapos,
                                   int64_t *__restrict__ out)
{
    if (threadIdx.x != 0) return;
    const int64_t nlong = longpos[m];
    out[0] = S[nnzA];
    out[1] = nlong;
    out[2] = nlong > 0 ? longO[nlong] : 0;
    out[3] = nlong > 0 ? longCO[nlong] : 0;
    out[4] = int64_t(stats[0]);
    out[5] = spapos[m];
    // out[6..9] are stats[7..10] themselves: short rows too wide for the row
    // accumulator, widest BITMAP span, SMALL rows, BITMAP rows
}

// A pinned host staging word array per host thread for the synchronising reads.
int64_t *pinned_words()
{
    static thread_local int64_t *p = nullptr;
    if (!p && cudaMallocHost(reinterpret_cast<void **>(&p), 16 * sizeof(int64_t)) != cudaSuccess) p = nullptr;
    return p;
}

msp_status read_back(const int64_t *dev, int n, int64_t *host, cudaStream_t s, const char *where)
{
    int64_t *pin = pinned_words();
    msp_status st = cuda_check(cudaMemcpyAsync(pin ? pin : host, dev, size_t(n) * 8, cudaMemcpyDeviceToHost, s), where);
    if (st == MSP_OK) st = cuda_check(cudaStreamSynchronize(s), where);
    if (st == MSP_OK && pin)
        for (int i = 0; i < n; ++i) host[i] = pin[i];
    return st;
}

bool rowacc_enabled();
bool small_enabled();

msp_status read_info(const SetupWs &sw, int64_t m, int64_t nnzA, HostInfo *h, cudaStream_t s)
{
    info_gather_kernel<<<1, 32, 0, s>>>(sw.S, nnzA, sw.longpos, m, sw.longO, sw.longCO, sw.stats, sw.spapos,
                                        reinterpret_cast<int64_t *>(sw.stats) + 1);
    msp_status st = last_launch("info_gather_kernel");
    if (st != MSP_OK) return st;
    int64_t v[10];
    st = read_back(reinterpret_cast<const int64_t *>(sw.stats) + 1, 10, v, s, "spgemm: setup sizes");
    if (st != MSP_OK) return st;
    h->nprods = v[0];
    h->nlong = v[1];
    h->LP = v[2];
    h->LC = v[3];
    h->maxP = v[4];
    h->nspa = v[5];
    // warp-row path: 0 = off (ESC tiles), else the widest BITMAP span, at least 1 (sizes the bitmaps)
    h->rowacc = (rowacc_enabled() && v[6] == 0) ? std::max<int64_t>(v[7], 1) : 0;
    h->nsmall = h->rowacc ? v[8] : 0;
    h->nbitmap = h->rowacc ? v[9] : 0;
    return MSP_OK;
}

template <typename KT, typename V, bool NUM>
msp_status launch_tiles(const msp_csr *A, const msp_csr *B, const SetupWs &sw, const MainWs &mw, int64_t ntiles,
                        int cbits, int32_t *Crp, int32_t *Ccol, void *Cval, cudaStream_t s)
{
    auto kern = gemm_tile_kernel<KT, V, NUM>;
    const int smem = int(sizeof(TileSmem<KT, NUM>));
    static const bool fit = getenv("MSP_SPGEMM_FIT") != nullptr;  // experiment: carveout fitted to the CTAs
    msp_status st = fit ? set_smem_attr(reinterpret_cast<const void *>(kern), smem, "spgemm: tile smem", GM_NT,
                                        nullptr, true)
                        : set_smem_attr(reinterpret_cast<const void *>(kern), smem, "spgemm: tile smem");
    if (st != MSP_OK) return st;
    kern<<<unsigned(ntiles), GM_NT, smem, s>>>(A->col_idx, static_cast<const V *>(A->vals), B->row_offsets,
                                                B->col_idx, static_cast<const V *>(B->vals), sw.arow, sw.S,
                                                sw.rowlong, mw.splits, cbits, mw.perm, Crp, Ccol,
                                                static_cast<V *>(Cval));
    return last_launch("gemm_tile_kernel");
}

// Key width for the launch: 32-bit keys when (row offset, col) of every tile
// fits below the two reserved values, else 64-bit.
template <typename V, bool NUM>
msp_status run_tiles(const msp_csr *A, const msp_csr *B, const SetupWs &sw, const MainWs &mw, int64_t ntiles,
                     int64_t maxspan, int32_t *Crp, int32_t *Ccol, void *Cval, cudaStream_t s)
{
    if (ntiles <= 0) return MSP_OK;
    int cbits = 1;
    while (cbits < 31 && (int64_t(1) << cbits) < int64_t(B->ncols)) ++cbits;
    const bool use32 = cbits < 31 && (maxspan + 2 <= (int64_t(1) << (32 - cbits)));
    return use32 ? launch_tiles<uint32_t, V, NUM>(A, B, sw, mw, ntiles, cbits, Crp, Ccol, Cval, s)
                 : launch_tiles<uint64_t, V, NUM>(A, B, sw, mw, ntiles, cbits, Crp, Ccol, Cval, s);
}

template <typename V, bool NUM>
msp_status run_long(const msp_csr *A, const msp_csr *B, const SetupWs &sw, const MainWs &mw, const HostInfo &h,
                    int32_t *Crp, int32_t *Ccol, void *Cval, cudaStream_t s)
{
    if (h.nlong == 0 || h.LP == 0) return MSP_OK;
    auto ck = long_chunk_kernel<V, NUM>;
    const int smem = int(sizeof(LongSmem<V, NUM>));
    msp_status st = set_smem_attr(reinterpret_cast<const void *>(ck), smem, "spgemm: chunk smem");
    if (st != MSP_OK) return st;
    ck<<<unsigned(h.LC), GM_NT, smem, s>>>(A->row_offsets, A->col_idx, static_cast<const V *>(A->vals),
                                           B->row_offsets, B->col_idx, static_cast<const V *>(B->vals), sw.S,
                                           h.nlong, sw.longrow, sw.longP, sw.longO, sw.longCO, mw.Xc[0], mw.Xv[0]);
    st = last_launch("long_chunk_kernel");
    if (st != MSP_OK) return st;
    int cur = 0;
    int64_t maxlong = h.maxP;
    for (int64_t w = GM_TL; w < maxlong; w *= 2) {
        long_merge_kernel<NUM><<<unsigned(ceil_div(h.LP, LM_T)), LM_NT, 0, s>>>(
            h.LP, h.nlong, sw.longO, sw.longP, w, mw.Xc[cur], mw.Xv[cur], mw.Xc[cur ^ 1], mw.Xv[cur ^ 1]);
        st = last_launch("long_merge_kernel");
        if (st != MSP_OK) return st;
        cur ^= 1;
    }
    const unsigned hb = unsigned(ceil_div(ceil_div(h.LP, 16), 256));
    if (!NUM) {
        long_heads_kernel<<<hb, 256, 0, s>>>(h.LP, h.nlong, sw.longO, sw.longrow, mw.Xc[cur], nullptr, Crp + 1);
        return last_launch("long_heads_kernel");
    }
    long_heads_kernel<<<hb, 256, 0, s>>>(h.LP, h.nlong, sw.longO, sw.longrow, mw.Xc[cur], mw.heads, nullptr);
    st = last_launch("long_heads_kernel");
    if (st != MSP_OK) return st;
    st = scan_i32_to_i64(mw.heads, mw.U, h.LP, mw.scan, mw.scan_bytes, s);
    if (st != MSP_OK) return st;
    const unsigned eb = unsigned(std::min<int64_t>(ceil_div(h.LP, 256), 148 * 16));
    long_emit_kernel<V><<<eb, 256, 0, s>>>(h.LP, h.nlong, sw.longO, sw.longrow, mw.Xc[cur], mw.Xv[cur], mw.heads,
                                           mw.U, Crp, Ccol, static_cast<V *>(Cval));
    return last_launch("long_emit_kernel");
}

bool rowacc_enabled()
{
    static int v = -1;
    if (v < 0) {
        const char *e = getenv("MSP_SPGEMM_ROWACC");  // 0 disables the short-row accumulator (ablation)
        v = (e && atoi(e) == 0) ? 0 : 1;
    }
    return v != 0;
}

bool small_enabled()
{
    static int v = -1;
    if (v < 0) {
        const char *e = getenv("MSP_SPGEMM_SMALL");  // 0: no compare-count path (round-2 behaviour, ablation)
        v = (e && atoi(e) == 0) ? 0 : 1;
    }
    return v != 0;
}

template <typename V, bool NUM>
msp_status run_small(const msp_csr *A, const msp_csr *B, const SetupWs &sw, const MainWs &mw, const HostInfo &h,
                     int32_t *Crp, int32_t *Ccol, void *Cval, cudaStream_t s)
{
    const int64_t nnz = A->nnz;
    const int all_small = (h.nbitmap == 0 && h.nlong == 0 && h.nspa == 0) ? 1 : 0;
    ws_expand_kernel<V, NUM><<<unsigned(std::min<int64_t>(ceil_div(nnz, 256), 148 * 32)), 256, 0, s>>>(
        nnz, sw.arow, sw.wmode, sw.S, sw.bstart, static_cast<const V *>(A->vals), B->col_idx,
        static_cast<const V *>(B->vals), mw.xcol, mw.xval, all_small);
    msp_status st = last_launch(NUM ? "ws_expand_kernel<numeric>" : "ws_expand_kernel<symbolic>");
    if (st != MSP_OK) return st;
    auto kern = ws_small_kernel<V, NUM>;
    int occ = 1;
    st = set_smem_attr(reinterpret_cast<const void *>(kern), 0, "spgemm: small rows", WS_WARPS * 32, &occ, true);
    if (st != MSP_OK) return st;
    const int32_t m = A->nrows;
    const int64_t g = std::min<int64_t>(int64_t(occ) * sm_count(), ceil_div(m, WS_WARPS * 32));
    kern<<<unsigned(g > 0 ? g : 1), WS_WARPS * 32, 0, s>>>(m, A->row_offsets, sw.wmode, sw.S, mw.xcol, mw.xval,
                                                          mw.xrank, Crp, Ccol, static_cast<V *>(Cval));
    return last_launch(NUM ? "ws_small_kernel<numeric>" : "ws_small_kernel<symbolic>");
}

template <bool NUM>
msp_status run_rowacc(const msp_csr *A, const msp_csr *B, const SetupWs &sw, const MainWs &mw, const HostInfo &h,
                      int32_t *Crp, int32_t *Ccol, void *Cval, cudaStream_t s)
{
    const int32_t m = A->nrows;
    if (h.nsmall > 0) {
        msp_status st = (A->dtype == MSP_F64) ? run_small<double, NUM>(A, B, sw, mw, h, Crp, Ccol, Cval, s)
                                              : run_small<float, NUM>(A, B, sw, mw, h, Crp, Ccol, Cval, s);
        if (st != MSP_OK) return st;
    }
    if (h.nbitmap <= 0) return MSP_OK;
    if (!NUM) {
        // bitmap words per warp: the widest short row's span, in rounds of 128 words
        const int nw_max = int(ceil_div(ceil_div(h.rowacc, 32), 128) * 128);
        const int smem = WR_SYM_WARPS * nw_max * 4;
        // the carveout / occupancy query is per bitmap size: no per-kernel cache here
        msp_status st = cuda_check(cudaFuncSetAttribute(reinterpret_cast<const void *>(wr_symbolic_kernel),
                                                        cudaFuncAttributeMaxDynamicSharedMemorySize, smem),
                                   "spgemm: row accumulator smem");
        if (st != MSP_OK) return st;
        int occ = 1;
        st = cuda_check(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, wr_symbolic_kernel, WR_SYM_WARPS * 32,
                                                                      size_t(smem)),
                        "spgemm: row accumulator occupancy");
        if (st != MSP_OK) return st;
        if (occ < 1) occ = 1;
        const int64_t g = std::min<int64_t>(int64_t(occ) * sm_count(), ceil_div(m, WR_SYM_WARPS));
        wr_symbolic_kernel<<<unsigned(g > 0 ? g : 1), WR_SYM_WARPS * 32, smem, s>>>(
            m, nw_max, A->row_offsets, A->col_idx, B->row_offsets, B->col_idx, sw.wmode, sw.S, sw.spanlo,
            sw.spanhi, Crp + 1, mw.ucol);
        return last_launch("wr_symbolic_kernel");
    }
    if (A->dtype == MSP_F64) {
        auto kern = wr_numeric_kernel<double>;
        int occ = 1;
        msp_status st = set_smem_attr(reinterpret_cast<const void *>(kern), WR_NUM_SMEM, "spgemm: row accumulator",
                                      WR_NUM_WARPS * 32, &occ, true);
        if (st != MSP_OK) return st;
        const int64_t g = std::min<int64_t>(int64_t(occ) * sm_count(), ceil_div(m, WR_NUM_WARPS));
        kern<<<unsigned(g > 0 ? g : 1), WR_NUM_WARPS * 32, WR_NUM_SMEM, s>>>(
            m, A->row_offsets, A->col_idx, static_cast<const double *>(A->vals), B->row_offsets, B->col_idx,
            static_cast<const double *>(B->vals), sw.wmode, sw.S, sw.spanlo, mw.ucol, Crp, Ccol,
            static_cast<double *>(Cval));
    } else {
        auto kern = wr_numeric_kernel<float>;
        int occ = 1;
        msp_status st = set_smem_attr(reinterpret_cast<const void *>(kern), WR_NUM_SMEM, "spgemm: row accumulator",
                                      WR_NUM_WARPS * 32, &occ, true);
        if (st != MSP_OK) return st;
        const int64_t g = std::min<int64_t>(int64_t(occ) * sm_count(), ceil_div(m, WR_NUM_WARPS));
        kern<<<unsigned(g > 0 ? g : 1), WR_NUM_WARPS * 32, WR_NUM_SMEM, s>>>(
            m, A->row_offsets, A->col_idx, static_cast<const float *>(A->vals), B->row_offsets, B->col_idx,
            static_cast<const float *>(B->vals), sw.wmode, sw.S, sw.spanlo, mw.ucol, Crp, Ccol,
            static_cast<float *>(Cval));
    }
    return last_launch("wr_numeric_kernel");
}

bool spa_enabled()
{
    static int v = -1;
    if (v < 0) {
        const char *e = getenv("MSP_SPGEMM_SEGMENTED");  // 0 disables the f3 path (ablation)
        v = (e && atoi(e) == 0) ? 0 : 1;
    }
    return v != 0;
}

template <typename V, bool NUM>
msp_status run_spa(const msp_csr *A, const msp_csr *B, const SetupWs &sw, const MainWs &mw, const HostInfo &h,
                   int32_t *Crp,
                   int32_t *Ccol, void *Cval, cudaStream_t s)
{
    if (h.nspa <= 0) return MSP_OK;
    auto kern = spa_row_kernel<V, NUM>;
    const int smem = (NUM ? SPA_W * 8 : 0) + SPA_W / 8 + 64;
    msp_status st = set_smem_attr(reinterpret_cast<const void *>(kern), smem, "spgemm: segmented smem");
    if (st != MSP_OK) return st;
    kern<<<unsigned(h.nspa), SPA_NT, smem, s>>>(A->nrows, sw.spapos, A->row_offsets, A->col_idx,
                                                static_cast<const V *>(A->vals), B->row_offsets, B->col_idx,
                                                static_cast<const V *>(B->vals), sw.spanlo, sw.spanhi,
                                                NUM ? nullptr : Crp + 1, Crp, mw.spawcnt, Ccol,
                                                static_cast<V *>(Cval));
    return last_launch(NUM ? "spa_row_kernel<numeric>" : "spa_row_kernel<symbolic>");
}

// Product tiles of the main pass (none when the row accumulator takes every short row).
int64_t ntiles_of(int64_t nnzA, int64_t nprods, int64_t rowacc = 0)
{
    if (rowacc) return 0;
    return ceil_div(nnzA + nprods > 0 ? nnzA + nprods : 1, GM_TP);
}

msp_status prepare_main(const msp_csr *A, const void *ws1, size_t b1, void *ws2, size_t b2, SetupWs *sw, MainWs *mw,
                        const HostInfo &h)
{
    bool ok1, ok2;
    *sw = carve_setup(A, const_cast<void *>(ws1), b1, &ok1);
    if (!ok1) return MSP_ERR_WORKSPACE;
    *mw = carve_main(A->nrows, ntiles_of(A->nnz, h.nprods, h.rowacc), h.LP, h.nbitmap > 0 ? h.nprods : 0,
                     h.nsmall > 0 ? h.nprods : 0, h.nspa, ws2, b2, &ok2);
    if (!ok2) return MSP_ERR_WORKSPACE;
    return MSP_OK;
}

HostInfo host_info(const msp_spgemm_info *info)
{
    HostInfo h;
    h.nprods = info->nprods;
    h.nlong = info->long_rows;
    h.LP = info->long_products;
    h.LC = info->long_chunks;
    h.maxP = info->max_row_products;
    h.nspa = info->segmented_rows;
    h.rowacc = info->row_accumulator;
    h.nsmall = info->small_rows;
    h.nbitmap = info->bitmap_rows;
    return h;
}

}  // namespace

msp_status spgemm_setup_arrays(const msp_csr *A, const void *ws1, size_t b1, const int32_t **arow, const int64_t **S)
{
    bool ok;
    const SetupWs w = carve_setup(A, const_cast<void *>(ws1), b1, &ok);
    if (!ok) return MSP_ERR_WORKSPACE;
    *arow = w.arow;
    *S = w.S;
    return MSP_OK;
}

size_t spgemm_setup_ws_bytes(const msp_csr *A, const msp_csr *)
{
    bool ok;
    SetupWs w = carve_setup(A, nullptr, SIZE_MAX, &ok);
    return w.bytes + 256;
}

msp_status spgemm_setup_run(const msp_csr *A, const msp_csr *B, void *ws1, size_t b1, msp_spgemm_info *info,
                            cudaStream_t s)
{
    bool ok;
    SetupWs w = carve_setup(A, ws1, b1, &ok);
    if (!ok) return MSP_ERR_WORKSPACE;
    const int64_t m = A->nrows, nnz = A->nnz;
    msp_status st = cuda_check(cudaMemsetAsync(w.stats, 0, 16 * sizeof(unsigned long long), s), "spgemm: clear");
    if (st != MSP_OK) return st;
    if (nnz > 0) {
        const int64_t thr = ceil_div(m + nnz, AROW_ITEMS);
        arow_kernel<<<unsigned(ceil_div(thr, 256)), 256, 0, s>>>(A->nrows, nnz, A->row_offsets, w.arow);
        st = last_launch("arow_kernel");
        if (st != MSP_OK) return st;
    }
    st = scan_widths_to_S_bstart(A->col_idx, B->row_offsets, nnz, w.S, w.bstart, w.scan, w.scan_bytes, s);
    if (st != MSP_OK) return st;
    if (m > 0) {
        const unsigned blocks = unsigned(std::min<int64_t>(ceil_div(m, 256), 148 * 16));
        rowclass_kernel<<<blocks, 256, 0, s>>>(A->nrows, A->row_offsets, w.S, w.rowlong, w.longflag, w.longP,
                                               w.stats);
        st = last_launch("rowclass_kernel");
        if (st != MSP_OK) return st;
        if (nnz > 0 && rowacc_enabled()) {  // warp-row path: SMALL / BITMAP rows, wide rows promoted to long
            wr_class_kernel<<<unsigned(std::min<int64_t>(ceil_div(m, 8 * 32), 148 * 16)), 256, 0, s>>>(
                A->nrows, A->row_offsets, A->col_idx, B->row_offsets, B->col_idx, w.S, w.rowlong, w.longflag,
                w.spanlo, w.spanhi, w.wmode, w.stats, small_enabled() ? 1 : 0);
            st = last_launch("wr_class_kernel");
            if (st != MSP_OK) return st;
        }
        // Matrices with >= 1024 rows: one extra synchronisation reads the long-row count
        // (from the classification and the promotions); without long rows the
        // global-phase bookkeeping (spans, segmented classification, four
        // row scans, scatters) is skipped -- C5: ~4.7 ms of setup.
        bool any_long = true;
        if (m >= 1024) {
            int64_t v[13];
            st = read_back(reinterpret_cast<const int64_t *>(w.stats), 13, v, s, "spgemm: long rows");
            if (st != MSP_OK) return st;
            any_long = (v[11] + v[12]) > 0;
        }
        if (!any_long) {
            st = cuda_check(cudaMemsetAsync(w.longpos + m, 0, sizeof(int64_t), s), "spgemm: clear");
            if (st == MSP_OK) st = cuda_check(cudaMemsetAsync(w.spapos + m, 0, sizeof(int64_t), s), "spgemm: clear");
            if (st != MSP_OK) return st;
        } else {
        // segmented path for long rows with a narrow output span (f3)
        span_init_kernel<<<blocks, 256, 0, s>>>(A->nrows, w.rowlong, w.spanlo, w.spanhi);
        st = last_launch("span_init_kernel");
        if (st != MSP_OK) return st;
        if (nnz > 0 && spa_enabled()) {
            span_kernel<<<unsigned(std::min<int64_t>(ceil_div(nnz, 256), 148 * 16)), 256, 0, s>>>(
                nnz, A->col_idx, w.arow, w.rowlong, B->row_offsets, B->col_idx, w.spanlo, w.spanhi);
            st = last_launch("span_kernel");
            if (st != MSP_OK) return st;
        }
        spa_classify_kernel<<<blocks, 256, 0, s>>>(A->nrows, A->row_offsets, w.S, w.spanlo, w.spanhi, w.rowlong,
                                                   w.longflag, w.spaflag);
        st = last_launch("spa_classify_kernel");
        if (st != MSP_OK) return st;
        st = scan_i32_to_i64(w.spaflag, w.spapos, m, w.scan, w.scan_bytes, s);
        if (st != MSP_OK) return st;
        st = scan_i32_to_i64(w.longflag, w.longpos, m, w.scan, w.scan_bytes, s);
        if (st != MSP_OK) return st;
        st = cuda_check(cudaMemsetAsync(w.longC, 0, size_t(m) * sizeof(int64_t), s), "spgemm: clear");
        if (st != MSP_OK) return st;
        long_scatter_kernel<<<blocks, 256, 0, s>>>(A->nrows, A->row_offsets, w.S, w.longflag, w.longpos,
                                                   w.longrow, w.longP, w.longC);
        st = last_launch("long_scatter_kernel");
        if (st != MSP_OK) return st;
        st = scan_i64_to_i64(w.longP, w.longO, m, w.scan, w.scan_bytes, s);
        if (st != MSP_OK) return st;
        st = scan_i64_to_i64(w.longC, w.longCO, m, w.scan, w.scan_bytes, s);
        if (st != MSP_OK) return st;
        }
    } else {
        st = cuda_check(cudaMemsetAsync(w.longpos, 0, sizeof(int64_t), s), "spgemm: clear");
        if (st == MSP_OK) st = cuda_check(cudaMemsetAsync(w.spapos, 0, sizeof(int64_t), s), "spgemm: clear");
        if (st != MSP_OK) return st;
    }
    HostInfo h;
    st = read_info(w, m, nnz, &h, s);
    if (st != MSP_OK) return st;
    const int64_t ntiles = ntiles_of(nnz, h.nprods, h.rowacc);
    bool ok2;
    MainWs mw = carve_main(m, ntiles, h.LP, h.nbitmap > 0 ? h.nprods : 0, h.nsmall > 0 ? h.nprods : 0, h.nspa,
                           nullptr, SIZE_MAX, &ok2);
    info->nprods = h.nprods;
    info->ntiles = ntiles;
    info->long_rows = h.nlong;
    info->long_products = h.LP;
    info->max_row_products = h.maxP;
    info->main_ws_bytes = int64_t(mw.bytes + 256);
    info->long_chunks = h.LC;
    info->max_tile_span = -1;  // set by symbolic
    info->segmented_rows = h.nspa;
    info->row_accumulator = h.rowacc;
    info->small_rows = h.nsmall;
    info->bitmap_rows = h.nbitmap;
    return MSP_OK;
}

// Symbolic: partition, tile spans (ONE synchronisation: the key width of the
// tile launch depends on the largest tile row span), tile + long-row passes,
// scan of the row counts (second synchronisation: nnz(C)).  Numeric: the same
// launches with values, every size taken from the host info -- no
// synchronisation.
template <bool NUM>
msp_status spgemm_pass(const msp_csr *A, const msp_csr *B, const void *ws1, size_t b1, void *ws2, size_t b2,
                       msp_spgemm_info *info, int32_t *Crp, int32_t *Ccol, void *Cval, int64_t *nnzC, cudaStream_t s)
{
    SetupWs sw;
    MainWs mw;
    const HostInfo h = host_info(info);
    msp_status st = prepare_main(A, ws1, b1, ws2, b2, &sw, &mw, h);
    if (st != MSP_OK) return st;
    const int64_t m = A->nrows;
    const int64_t ntiles = ntiles_of(A->nnz, h.nprods, h.rowacc);
    int64_t maxspan = info->max_tile_span;
    if (!NUM && h.rowacc && m > 0) {
        st = cuda_check(cudaMemsetAsync(Crp, 0, size_t(m + 1) * sizeof(int32_t), s), "spgemm: clear rp");
        if (st != MSP_OK) return st;
        maxspan = 0;  // no product tiles
        info->max_tile_span = 0;
    } else if (!NUM) {
        st = cuda_check(cudaMemsetAsync(Crp, 0, size_t(m + 1) * sizeof(int32_t), s), "spgemm: clear rp");
        if (st != MSP_OK) return st;
        if (m == 0) {
            *nnzC = 0;
            info->max_tile_span = 0;
            return cuda_check(cudaStreamSynchronize(s), "spgemm: sync");
        }
        gemm_partition_kernel<<<unsigned(std::min<int64_t>(ceil_div(ntiles + 1, 256), 148 * 16)), 256, 0, s>>>(
            A->nrows, A->nnz, h.nprods, A->row_offsets, sw.arow, sw.S, sw.rowlong, ntiles, mw.splits);
        st = last_launch("gemm_partition_kernel");
        if (st != MSP_OK) return st;
        st = cuda_check(cudaMemsetAsync(&mw.totals[1], 0, 8, s), "spgemm: clear span");
        if (st != MSP_OK) return st;
        tile_span_kernel<<<unsigned(std::min<int64_t>(ceil_div(ntiles, 256), 148 * 4)), 256, 0, s>>>(
            ntiles, mw.splits, sw.arow, reinterpret_cast<unsigned long long *>(&mw.totals[1]));
        st = last_launch("tile_span_kernel");
        if (st != MSP_OK) return st;
        st = read_back(&mw.totals[1], 1, &maxspan, s, "spgemm: tile span");
        if (st != MSP_OK) return st;
        info->max_tile_span = maxspan;
    } else if (m == 0 || h.nprods == 0) {
        return MSP_OK;
    } else if (maxspan < 0) {
        set_error("spgemm: numeric needs the info returned by symbolic (max_tile_span unset)");
        return MSP_ERR_ARG;
    }
    if (h.nprods > 0 && m > 0) {
        if (h.rowacc) st = run_rowacc<NUM>(A, B, sw, mw, h, Crp, Ccol, Cval, s);
        else
            st = (A->dtype == MSP_F64) ? run_tiles<double, NUM>(A, B, sw, mw, ntiles, maxspan, Crp, Ccol, Cval, s)
                                       : run_tiles<float, NUM>(A, B, sw, mw, ntiles, maxspan, Crp, Ccol, Cval, s);
        if (st != MSP_OK) return st;
        st = (A->dtype == MSP_F64) ? run_long<double, NUM>(A, B, sw, mw, h, Crp, Ccol, Cval, s)
                                   : run_long<float, NUM>(A, B, sw, mw, h, Crp, Ccol, Cval, s);
        if (st != MSP_OK) return st;
        st = (A->dtype == MSP_F64) ? run_spa<double, NUM>(A, B, sw, mw, h, Crp, Ccol, Cval, s)
                                   : run_spa<float, NUM>(A, B, sw, mw, h, Crp, Ccol, Cval, s);
        if (st != MSP_OK) return st;
    }
    if (!NUM) {
        st = scan_counts_to_offsets_i32(Crp + 1, m, &mw.totals[0], mw.scan, mw.scan_bytes, s);
        if (st != MSP_OK) return st;
        int64_t tot = 0;
        st = read_back(&mw.totals[0], 1, &tot, s, "spgemm: nnz");
        if (st != MSP_OK) return st;
        *nnzC = tot;
        if (tot > INT32_MAX) {
            set_error("spgemm: nnz(C) = %lld exceeds int32", (long long)tot);
            return MSP_ERR_OVERFLOW;
        }
    }
    return MSP_OK;
}

msp_status spgemm_symbolic_run(const msp_csr *A, const msp_csr *B, const void *ws1, size_t b1, void *ws2,
                               size_t b2, msp_spgemm_info *info, int32_t *Crp, int64_t *nnzC, cudaStream_t s)
{
    return spgemm_pass<false>(A, B, ws1, b1, ws2, b2, info, Crp, nullptr, nullptr, nnzC, s);
}

msp_status spgemm_numeric_run(const msp_csr *A, const msp_csr *B, const void *ws1, size_t b1, void *ws2,
                              size_t b2, const msp_spgemm_info *info, const int32_t *Crp, int32_t *Ccol, void *Cval,
                              cudaStream_t s)
{
    msp_spgemm_info copy = *info;
    return spgemm_pass<true>(A, B, ws1, b1, ws2, b2, &copy, const_cast<int32_t *>(Crp), Ccol, Cval, nullptr, s);
}

}  // namespace msp
