// spmv_wt.cu -- merge-path SpMV with warp-owned tiles (row-aligned lanes), sm_100a.
//
// Paper: Section III-A: partition, reduction
// (P:432-460), update.  Same merge grid, tile semantics and
// carry rules as spmv.cu (readings Z4, Z6, Z21, R2, R3); what differs is who
// owns a tile ("warp tiles"):
//
//   * A tile is 32*K merge items and belongs to ONE worker warp (tile t of a
//     CTA goes to warp t mod NW); every lane owns K consecutive products of
//     the tile, K the odd width nearest the mean row length, so on a stencil
//     lane l starts on row l's first nonzero and gather u of the warp touches
//     the same stencil position of 32 consecutive rows.
//   * The producer warp computes 32 tile splits at a time (one binary search
//     per lane) and streams every tile's row_offsets / col / val windows with
//     TMA bulk copies into a ring of S slots (S > NW): the workers are not
//     tied to a common tile, so their load bursts (shared memory, x gathers)
//     and their ALU-heavy walks interleave instead of happening in lockstep
//     (the CTA-tile kernel of spmv.cu keeps all 8 workers on one tile; its
//     trace shows the whole SM alternating between gather and walk phases).
//   * A worker copies its tile's columns (-> K gathers in flight per lane),
//     values and row ends (own row map from the staged row_offsets window)
//     into registers / a warp-private map, zero-fills the tile's empty rows
//     and releases the slot BEFORE the walk, so slots are held briefly and the
//     TMA ring keeps far more bytes in flight.
//   * Carries between tiles use a decoupled look-back over a ring of per-tile
//     records (aggregate, then inclusive carry), deferred to the warp's next
//     tile so that it rarely waits; one (row, partial) carry per CTA goes to
//     the update phase as in spmv.cu (the last CTA adds them in CTA order).
#include <climits>
#include <cstdio>
#include <cstdlib>
#include <type_traits>

#include "common.cuh"
#include "internal.h"

#ifdef MSP_SPMV_TRACE
// timeline stamps (experiment builds): [CTA < 4][tile < 256][slot < 8]
__device__ long long g_spmv_wt_trace[4][256][8];
extern "C" int msp_debug_spmv_wt_trace(void *host)
{
    return int(cudaMemcpyFromSymbol(host, g_spmv_wt_trace, sizeof(g_spmv_wt_trace)));
}
#define WTR(t, slot)                                                                                    \
    do {                                                                                                \
        if (blockIdx.x < 4 && (t) < 256) g_spmv_wt_trace[blockIdx.x][(t)][(slot)] = clock64() - tr_t0;  \
    } while (0)
#else
#define WTR(t, slot) \
    do {             \
    } while (0)
#endif

namespace msp {
namespace {

struct WtRecord {  // one per CTA (same meaning as spmv.cu's CtaRecord)
    int32_t carry_key;
    int32_t head_row;
    double carry_val;
    double head_val;
};

struct WtMeta {
    int32_t i_s, i_e, wr_end, j_s, j_e;
    uint32_t rp_first, col_first, val_first;
};

template <typename V, int K_, int NW_, int NSUB_, int STAGES_>
struct WtCfg {
    static constexpr int K = K_;
    static constexpr int NW = NW_;                       // worker warps
    static constexpr int TI = 32 * K;                    // merge items per warp tile
    static constexpr int NSUB = NSUB_;                   // warp tiles per TMA stage
    static constexpr int T = NSUB * TI;                  // merge items per stage
    static constexpr int STAGES = STAGES_;
    static constexpr int THREADS = (NW + 1) * 32;        // + producer warp
    static constexpr int SLOT_BYTES = int(((4 + sizeof(V)) * T + 64 + 15) / 16 * 16);
    static constexpr int WMAP_BYTES = (32 * 4 + TI * 2 + 15) / 16 * 16;  // lane masks + row per position
    static constexpr int RL = 256;                       // look-back ring (warp tiles; > STAGES*NSUB + NW)
    static constexpr int SMEM = STAGES * SLOT_BYTES + NW * WMAP_BYTES + RL * 32 + STAGES * 48 + 256;
    static_assert(K % 2 == 1 && K < 32, "K odd and < 32");
    static_assert(SMEM <= 227 * 1024, "shared memory");
    static_assert(RL > STAGES * NSUB + 2 * NW, "look-back ring must cover the tiles in flight");
};

__device__ __forceinline__ double ldg_xv(const double *p)
{
    double v;
    asm volatile("ld.global.f64 %0, [%1];" : "=d"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ double ldg_xv(const float *p)
{
    float v;
    asm volatile("ld.global.f32 %0, [%1];" : "=f"(v) : "l"(p) : "memory");
    return double(v);
}

// 32-ary warp search on the CSR merge grid in global memory: smallest i in
// [lo, hi] with NOT(rp[i+1] <= d - i - 1).  All lanes return the same value.
__device__ __forceinline__ int warp_grid_search_wt(const int32_t *__restrict__ rp, int64_t d, int lo, int hi, int lane)
{
    while (hi - lo > 32) {
        const int64_t step = (int64_t(hi) - lo + 31) / 32;
        const int64_t p = int64_t(lo) + (lane + 1) * step - 1;
        bool pred = false;
        if (p < hi) pred = int64_t(__ldg(rp + p + 1)) <= d - p - 1;
        const int c = __popc(__ballot_sync(0xffffffffu, pred));
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

// Same with a guess: the 32 rows around g first (one ballot when the stage
// holds about as many rows as the previous one).
__device__ __forceinline__ int warp_grid_search_wt_guess(const int32_t *__restrict__ rp, int64_t d, int lo, int hi,
                                                         int g, int lane)
{
    if (hi - lo <= 32) return warp_grid_search_wt(rp, d, lo, hi, lane);
    int base = g - 16;
    base = max(lo, min(base, hi - 32));
    const int64_t p = int64_t(base) + lane;
    const bool pred = int64_t(__ldg(rp + p + 1)) <= d - p - 1;
    const int c = __popc(__ballot_sync(0xffffffffu, pred));
    if (c > 0 && c < 32) return base + c;
    if (c == 0) return (base == lo) ? lo : warp_grid_search_wt(rp, d, lo, base, lane);
    return warp_grid_search_wt(rp, d, base + 32, hi, lane);
}

// Split of stage-relative diagonal d (0 <= d <= srows + snz) in the staged
// row_offsets window: smallest i in [max(0, d - snz), min(d, srows)] with
// NOT(rpb[i+1] - j_s <= d - i - 1).  32-ary warp search in shared memory.
__device__ __forceinline__ int stage_split(const int32_t *rpb, int j_s, int d, int srows, int snz, int lane)
{
    int lo = max(0, d - snz), hi = min(d, srows);
    while (hi - lo > 32) {
        const int step = (hi - lo + 31) >> 5;
        const int p = lo + (lane + 1) * step - 1;
        const bool pred = p < hi && rpb[p + 1] - j_s <= d - p - 1;
        const int c = __popc(__ballot_sync(0xffffffffu, pred));
        const int nhi = (c < 32) ? min(hi, lo + (c + 1) * step - 1) : hi;
        lo += c * step;
        hi = nhi;
    }
    const int p = lo + lane;
    const bool pred = p < hi && rpb[p + 1] - j_s <= d - p - 1;
    return lo + __popc(__ballot_sync(0xffffffffu, pred));
}

// Look-back record of a tile.  The aggregate (trailing sum) and the
// inclusive carry-out live in SEPARATE fields, each written once before its
// bit in the tag word ((tile+1) << 2 | 1 aggregate | 2 inclusive): a reader
// that sees bit 1 only must never read an inclusive value written after it
// checked the tag (an earlier single-value record was upgraded in place and
// could be read half-way: nondeterministic double counting on long rows).
struct alignas(16) LbRec {
    double agg;   // trailing sum of the tile
    double inc;   // inclusive carry-out (the carry into the next tile)
    int f_agg;    // the tile has a row end
    int f_inc;    // some tile of the CTA up to this one has a row end
    int tag;
    int pad;
};

__device__ __forceinline__ void lb_publish_agg(LbRec *r, double v, int tile)
{
    *reinterpret_cast<volatile double *>(&r->agg) = v;
    *reinterpret_cast<volatile int *>(&r->f_agg) = 0;
    __threadfence_block();
    *reinterpret_cast<volatile int *>(&r->tag) = ((tile + 1) << 2) | 1;
}

__device__ __forceinline__ void lb_publish_inc(LbRec *r, double agg, double inc, int f_agg, int f_inc, int tile)
{
    *reinterpret_cast<volatile double *>(&r->agg) = agg;
    *reinterpret_cast<volatile double *>(&r->inc) = inc;
    *reinterpret_cast<volatile int *>(&r->f_agg) = f_agg;
    *reinterpret_cast<volatile int *>(&r->f_inc) = f_inc;
    __threadfence_block();
    *reinterpret_cast<volatile int *>(&r->tag) = ((tile + 1) << 2) | 3;
}

// (the aggregate fields of a record are rewritten with the same values when
// its inclusive carry is published, so a concurrent aggregate read is exact)

template <typename V, class C>
__global__ void __launch_bounds__(C::THREADS, 1)
spmv_wt_kernel(int32_t m, int64_t nnz, const int32_t *__restrict__ rp, const int32_t *__restrict__ col,
               const V *__restrict__ val, const V *__restrict__ x, V *__restrict__ y, int32_t n_cols,
               WtRecord *__restrict__ recs, unsigned *__restrict__ counter)
{
    constexpr int K = C::K, NW = C::NW, S = C::STAGES, TI = C::TI, RL = C::RL, NSUB = C::NSUB, T = C::T;
    extern __shared__ __align__(128) char smem[];
    char *slots = smem;
    char *wmaps = slots + size_t(S) * C::SLOT_BYTES;
    LbRec *lb = reinterpret_cast<LbRec *>(wmaps + size_t(NW) * C::WMAP_BYTES);  // [RL]
    WtMeta *meta = reinterpret_cast<WtMeta *>(lb + RL);                          // [S]
    uint64_t *full = reinterpret_cast<uint64_t *>(meta + S);
    uint64_t *empty = full + S;
    __shared__ int s_carry_key, s_head_row, s_last;
    __shared__ double s_head_val, s_carry_val;

    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int G = gridDim.x;
    const int64_t total = int64_t(m) + nnz;
    const int64_t d_begin = int64_t(blockIdx.x) * total / G;
    const int64_t d_end = int64_t(blockIdx.x + 1) * total / G;
    const int ntiles = int((d_end - d_begin + TI - 1) / TI);  // warp tiles
    const int nstages = (ntiles + NSUB - 1) / NSUB;           // TMA tiles
#ifdef MSP_SPMV_TRACE
    const long long tr_t0 = clock64();
#endif

    if (tid == 0) {
        for (int s = 0; s < S; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], NSUB);  // every warp tile of the stage releases it
        }
        fence_mbar_init();
        s_carry_key = -1;
        s_head_row = -1;
        s_head_val = 0.0;
        s_carry_val = 0.0;
    }
    for (int i = tid; i < RL; i += blockDim.x) lb[i].tag = 0;
    __syncthreads();

    if (warp == NW) {
        // ============================ producer ================================
        // One 32-ary warp search per stage of T = NSUB * TI items (guessing the
        // previous stage's row count), then the stage's row_offsets / col /
        // val windows in three TMA bulk copies.  The warp tiles inside a stage
        // are split by the workers themselves (search in the staged window).
        const uint64_t pol = policy_evict_first();
        int i_s = warp_grid_search_wt(rp, d_begin, int(max(int64_t(0), d_begin - nnz)), int(min(d_begin, int64_t(m))),
                                      lane);
        int j_s = int(d_begin - i_s);
        int prev_rows = 0;
        for (int b = 0; b < nstages; ++b) {
            const int slot = b % S;
            int64_t de = d_begin + int64_t(b + 1) * T;
            if (de > d_end) de = d_end;
            const int lo = int(max(int64_t(i_s), de - nnz));
            const int hi = int(min(int64_t(m), de - j_s));
            const int ie = warp_grid_search_wt_guess(rp, de, lo, hi, i_s + prev_rows, lane);
            const int je = int(de - ie);
            prev_rows = ie - i_s;
            if (lane == 0) WTR(b, 0);  // split known
            if (b >= S) mbar_wait(&empty[slot], ((b / S) - 1) & 1);
            if (lane == 0) WTR(b, 1);  // slot free
            char *sb = slots + size_t(slot) * C::SLOT_BYTES;
            const int wr_end = min(ie + 1, m);
            const WindowCopy wr = plan_window<4>(rp, i_s, int64_t(wr_end) + 1, int64_t(m) + 1);
            const WindowCopy wc = plan_window<4>(col, j_s, je, nnz);
            const WindowCopy wv = plan_window<int(sizeof(V))>(val, j_s, je, nnz);
            const uint32_t off_r = 0, off_c = wr.span, off_v = wr.span + wc.span;
            const int nr = int(wr.head_elems + wr.tail_elems);
            const int nc = int(wc.head_elems + wc.tail_elems);
            const int nv = int(wv.head_elems + wv.tail_elems);
            if (nr + nc + nv) {
                if (lane < nr) window_manual<int32_t>(wr, rp, i_s, int64_t(wr_end) + 1, sb + off_r, lane);
                else if (lane < nr + nc) window_manual<int32_t>(wc, col, j_s, je, sb + off_c, lane - nr);
                else if (lane < nr + nc + nv) window_manual<V>(wv, val, j_s, je, sb + off_v, lane - nr - nc);
                __syncwarp();
            }
            if (lane == 0) {
                WtMeta &mt = meta[slot];
                mt.i_s = i_s; mt.i_e = ie; mt.wr_end = wr_end; mt.j_s = j_s; mt.j_e = je;
                mt.rp_first = off_r + wr.first;
                mt.col_first = off_c + wc.first;
                mt.val_first = off_v + wv.first;
                mbar_arrive_expect_tx(&full[slot], wr.bulk_bytes + wc.bulk_bytes + wv.bulk_bytes);
                if (wr.bulk_bytes) bulk_g2s(sb + off_r + wr.bulk_dst, wr.bulk_src, wr.bulk_bytes, &full[slot], 0);
                if (wc.bulk_bytes) bulk_g2s(sb + off_c + wc.bulk_dst, wc.bulk_src, wc.bulk_bytes, &full[slot], pol);
                if (wv.bulk_bytes) bulk_g2s(sb + off_v + wv.bulk_dst, wv.bulk_src, wv.bulk_bytes, &full[slot], pol);
            }
            i_s = ie;
            j_s = je;
        }
    } else {
        // ============================ workers ==================================
        uint32_t *wmask = reinterpret_cast<uint32_t *>(wmaps + size_t(warp) * C::WMAP_BYTES);  // [32]
        uint16_t *wrow = reinterpret_cast<uint16_t *>(wmask + 32);                             // [TI]
        const int q0 = lane * K;
        // deferred completion of a tile's first row (lane flane) and, for a
        // tile without row ends, its inclusive carry-out (finish, below)
        int pend_t = -1, pend_r = -1, pend_fl = 0;
        double pend_v = 0.0, pend_agg = 0.0;
        auto finish = [&](int tt, int r, int has_rows, double v0, double agg) {
            // carry into tile tt from earlier tiles (nearest first)
            double c = 0.0;
            bool head = true;  // no earlier row end in this CTA
            for (int j = tt - 1; j >= 0; --j) {
                LbRec *rec = &lb[j & (RL - 1)];
                int tg;
                while (((tg = *reinterpret_cast<volatile int *>(&rec->tag)) >> 2) != j + 1) {}
                __threadfence_block();
                if (tg & 2) {  // inclusive carry-out of tile j, head status in f_inc
                    c = *reinterpret_cast<volatile double *>(&rec->inc) + c;
                    head = *reinterpret_cast<volatile int *>(&rec->f_inc) == 0;
                    break;
                }
                c = *reinterpret_cast<volatile double *>(&rec->agg) + c;  // aggregate of a tile without row ends
            }
            if (has_rows) {
                const double v = v0 + c;
                y[r] = V(v);
                if (head) {
                    s_head_row = r;
                    s_head_val = v;
                }
            } else {
                // no row end in tile tt: publish its inclusive carry-out (f_inc
                // = 1 if some earlier tile of the CTA had a row end)
                lb_publish_inc(&lb[tt & (RL - 1)], agg, c + agg, 0, head ? 0 : 1, tt);
            }
        };
        for (int t = warp; t < ntiles; t += NW) {
            const int b = t / NSUB, slot = b % S;
            if (lane == 0) WTR(t, 2);  // worker ready
            mbar_wait(&full[slot], (b / S) & 1);
            if (lane == 0) WTR(t, 3);  // landed
            const WtMeta st = meta[slot];
            const char *sb = slots + size_t(slot) * C::SLOT_BYTES;
            const int32_t *rpb = reinterpret_cast<const int32_t *>(sb + st.rp_first);  // rpb[k] = rp[st.i_s + k]
            // this warp tile: stage diagonals [d0, d1) -> splits (i0, j0), (i1, j1)
            // of the stage's merge grid (rows st.i_s + i, nonzeros st.j_s + j)
            const int srows = st.i_e - st.i_s, snz = st.j_e - st.j_s;
            const int sub = t - b * NSUB;
            const int d0 = sub * TI, d1 = min(d0 + TI, srows + snz);
            const int i0 = stage_split(rpb, st.j_s, d0, srows, snz, lane);
            const int i1 = stage_split(rpb, st.j_s, d1, srows, snz, lane);
            const int j0 = d0 - i0, j1 = d1 - i1;
            WtMeta mt;  // the warp tile in global terms
            mt.i_s = st.i_s + i0;
            mt.i_e = st.i_s + i1;
            mt.wr_end = min(mt.i_e + 1, st.wr_end);
            mt.j_s = st.j_s + j0;
            mt.j_e = st.j_s + j1;
            const int z = j1 - j0;
            const int32_t *cs = reinterpret_cast<const int32_t *>(sb + st.col_first) + j0;
            const V *vs = reinterpret_cast<const V *>(sb + st.val_first) + j0;
            const int32_t *rps = rpb + i0;  // rps[k] = rp[mt.i_s + k]
            // ---- gathers (K in flight per lane), values into registers ----
            // positions >= z (the tile's last lanes) read stale slot bytes:
            // their columns are clamped into x (a valid address) and their
            // products are masked in the walk (no per-position select here)
            const unsigned cmax = unsigned(n_cols - 1);
            int cidx[K];
#pragma unroll
            for (int u = 0; u < K; ++u) cidx[u] = int(min(unsigned(cs[q0 + u]), cmax));
            double xv[K];
#pragma unroll
            for (int u = 0; u < K; ++u) xv[u] = ldg_xv(x + cidx[u]);
            double vv[K];
#pragma unroll
            for (int u = 0; u < K; ++u) vv[u] = double(vs[q0 + u]);
            // ---- row ends of the tile -> lane masks + row ids; empty rows ----
            wmask[lane] = 0u;
            __syncwarp();
            const int nwin = mt.wr_end - mt.i_s, nend = mt.i_e - mt.i_s, j_s = mt.j_s;
            int ckey = -1;
            for (int k = lane; k < nwin; k += 32) {
                const int a = rps[k] - j_s, e = rps[k + 1] - j_s;
                if (a == e) {
                    if (k < nend) y[mt.i_s + k] = V(0);  // empty row ending in the tile (Z6)
                } else {
                    if (e > 0 && e <= z) {
                        const int pos = e - 1;
                        const int ol = pos / K;
                        atomicOr(&wmask[ol], 1u << (pos - ol * K));
                        wrow[pos] = uint16_t(k);
                    }
                    if (z > 0 && a < z && e > z) ckey = mt.i_s + k;  // row continues past the tile
                }
            }
            if (t == ntiles - 1) {  // the CTA's carry key: row of its last product if it continues
                const unsigned bk = __ballot_sync(0xffffffffu, ckey >= 0);
                const int key = bk ? __shfl_sync(0xffffffffu, ckey, __ffs(bk) - 1) : -1;
                if (lane == 0) s_carry_key = key;
            }
            __syncwarp();
            const unsigned mask = wmask[lane];
#ifndef MSP_WT_NO_VV_FENCE
            {   // the values must be IN registers before the slot is handed back
                // to the TMA engine: consume every vv register (scoreboard wait)
                unsigned long long acc = 0;
#pragma unroll
                for (int u = 0; u < K; ++u) acc |= __double_as_longlong(vv[u]);
                asm volatile("" ::"l"(acc));
            }
#endif
            __syncwarp();
            if (lane == 0) mbar_arrive(&empty[slot]);  // this warp tile of the stage is in regs / the map
            if (lane == 0) WTR(t, 4);  // released
            // ---- walk: K fp64 multiply-adds, y at each row end ----
            V *ybase = y + mt.i_s;
            const uint16_t *lrow = wrow + q0;
            double run = 0.0, first_v = 0.0;
            int first_k = -1;
            const int lim = z - q0;  // products of this lane: u < lim
#pragma unroll
            for (int u = 0; u < K; ++u) {
                if (u < lim) run = fma(vv[u], xv[u], run);
                if ((mask >> u) & 1u) {
                    if (first_k < 0) {
                        first_k = u;
                        first_v = run;
                    } else {
                        ybase[lrow[u]] = V(run);
                    }
                    run = 0.0;
                }
            }
            const int first_r = first_k >= 0 ? mt.i_s + int(lrow[first_k]) : -1;
            if (lane == 0) WTR(t, 5);  // walked
            const bool flagged = first_r >= 0;
            // ---- carries between lanes ----
            const unsigned fmask = __ballot_sync(0xffffffffu, flagged);
            const unsigned active = __ballot_sync(0xffffffffu, lim > 0);  // lanes 0.. with products
            const int flane = fmask ? __ffs(fmask) - 1 : -1;
            double exv, agg;
            if (fmask == active && active) {
                // every lane with products ends a row (a stencil tile): the
                // carry into a lane is its left neighbour's trailing sum
                exv = __shfl_up_sync(0xffffffffu, run, 1);
                agg = __shfl_sync(0xffffffffu, run, 31 - __clz(active));
            } else {  // general case: warp segmented scan
                const SegPair<double> inc = warp_seg_inclusive(SegPair<double>{flagged, run}, lane);
                exv = __shfl_up_sync(0xffffffffu, inc.v, 1);
                agg = __shfl_sync(0xffffffffu, inc.v, 31);  // trailing sum of the tile
            }
            double nv = 0.0;
            if (flagged) {
                const double v = lane ? first_v + exv : first_v;
                if (lane == flane) nv = v;
                else y[first_r] = V(v);
            }
            if (lane == 0 && fmask) lb_publish_inc(&lb[t & (RL - 1)], agg, agg, 1, 1, t);  // carry-out known
            else if (lane == 0) lb_publish_agg(&lb[t & (RL - 1)], agg, t);                  // aggregate only
            // ---- finish the previous tile of this warp (deferred look-back) ----
            if (pend_t >= 0) {
                const int hr = __shfl_sync(0xffffffffu, pend_r, pend_fl >= 0 ? pend_fl : 0);
                const double hv = __shfl_sync(0xffffffffu, pend_v, pend_fl >= 0 ? pend_fl : 0);
                if (lane == 0) finish(pend_t, hr, pend_fl >= 0, hv, pend_agg);
            }
            if (lane == 0) WTR(t, 6);  // published + previous finished
            pend_t = t;
            pend_fl = flane;
            pend_r = first_r;
            pend_v = nv;
            pend_agg = agg;
            __syncwarp();
        }
        if (pend_t >= 0) {
            const int hr = __shfl_sync(0xffffffffu, pend_r, pend_fl >= 0 ? pend_fl : 0);
            const double hv = __shfl_sync(0xffffffffu, pend_v, pend_fl >= 0 ? pend_fl : 0);
            if (lane == 0) finish(pend_t, hr, pend_fl >= 0, hv, pend_agg);
        }
    }
    __syncthreads();
    if (tid == 0 && ntiles > 0) {
        // the CTA's carry-out: inclusive carry of its last tile
        const int j = ntiles - 1;
        LbRec *rec = &lb[j & (RL - 1)];
        int tg;
        while (((tg = *reinterpret_cast<volatile int *>(&rec->tag)) >> 2) != j + 1 || !(tg & 2)) {}
        __threadfence_block();
        s_carry_val = *reinterpret_cast<volatile double *>(&rec->inc);
    }
    __syncthreads();
    if (tid == 0) {
        WtRecord rec;
        rec.carry_key = s_carry_key;
        rec.carry_val = s_carry_val;
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
    for (int k = tid; k < G; k += blockDim.x) {
        const int key = __ldcg(&recs[k].carry_key);
        if (key < 0 || key >= m) continue;
        if (k > 0 && __ldcg(&recs[k - 1].carry_key) == key) continue;  // not the head of a run
        double s = 0.0;
        int k2 = k;
        while (k2 < G && __ldcg(&recs[k2].carry_key) == key) {
            s += __ldcg(&recs[k2].carry_val);
            ++k2;
        }
        if (k2 < G && __ldcg(&recs[k2].head_row) == key) y[key] = V(s + __ldcg(&recs[k2].head_val));
    }
    if (tid == 0) *counter = 0u;
}

template <typename V, int K>
msp_status launch_wt(const msp_csr *A, const void *x, void *y, void *ws, size_t ws_bytes, cudaStream_t s)
{
    // 11 workers + the producer: 12 warps = 3 per SM sub-partition, so up to
    // 168 registers per thread (each sub-partition holds 16K registers);
    // 4 stages of warp tiles (about 47 KB each; 4 x 4 tiles for K = 27 fp64)
#ifndef MSP_WT_STAGES  // tuning builds: ring depth and tiles per stage
#define MSP_WT_STAGES 4  // C2: 4 x 4 warp tiles 68.4 us vs 3 x 6 70.7 us (profiles/r2/spmv_wt_ring_sweep.txt)
#endif
#ifndef MSP_WT_NSUB
#define MSP_WT_NSUB 0  // 0: as many warp tiles as fit ~188 KB over the stages
#endif
    constexpr int NSUB0 = MSP_WT_NSUB > 0 ? MSP_WT_NSUB
                                          : (188 * 1024 / MSP_WT_STAGES) / int((4 + sizeof(V)) * 32 * K);
#ifndef MSP_WT_NW
#define MSP_WT_NW 11  // worker warps (tuning builds)
#endif
    using C = WtCfg<V, K, MSP_WT_NW, (NSUB0 < 24 ? NSUB0 : 24), MSP_WT_STAGES>;
    auto kern = spmv_wt_kernel<V, C>;
    int occ = 1;
    static const bool fit = getenv("MSP_SPMV_WT_L1") != nullptr;  // experiment: carveout fitted to the CTA
    msp_status st = set_smem_attr(reinterpret_cast<const void *>(kern), C::SMEM, "spmv_wt: smem", C::THREADS, &occ, fit);
    if (st != MSP_OK) return st;
    static bool said = false;
    if (!said && getenv("MSP_VERBOSE")) {
        cudaFuncAttributes fa;
        cudaFuncGetAttributes(&fa, reinterpret_cast<const void *>(kern));
        fprintf(stderr,
                "msp spmv: warp tiles K=%d NW=%d stages=%d x %d tiles TI=%d smem=%d occupancy=%d CTAs/SM (regs %d, "
                "max threads %d, static smem %zu)\n",
                C::K, C::NW, C::STAGES, C::NSUB, C::TI, C::SMEM, occ, fa.numRegs, fa.maxThreadsPerBlock,
                fa.sharedSizeBytes);
        said = true;
    }
    if (A->nrows == 0) return MSP_OK;
    if (A->nnz == 0) return cuda_check(cudaMemsetAsync(y, 0, size_t(A->nrows) * sizeof(V), s), "spmv: zero y");
    const int64_t tiles = ceil_div(int64_t(A->nrows) + A->nnz, C::TI);
    int64_t g = int64_t(occ) * sm_count();
    if (g > tiles) g = tiles;
    const int grid = int(g);
    Carve cv(ws, ws_bytes);
    unsigned *counter = cv.take<unsigned>(1);
    WtRecord *recs = cv.take<WtRecord>(size_t(grid));
    if (!cv.ok()) return MSP_ERR_WORKSPACE;
    kern<<<grid, C::THREADS, C::SMEM, s>>>(A->nrows, A->nnz, A->row_offsets, A->col_idx,
                                          static_cast<const V *>(A->vals), static_cast<const V *>(x),
                                          static_cast<V *>(y), A->ncols, recs, counter);
    return last_launch("spmv_wt_kernel");
}

}  // namespace

msp_status spmv_wt_run(int K, const msp_csr *A, const void *x, void *y, void *ws, size_t ws_bytes, cudaStream_t s)
{
    const bool f64 = A->dtype == MSP_F64;
    switch (K) {
    case 7: return f64 ? launch_wt<double, 7>(A, x, y, ws, ws_bytes, s) : launch_wt<float, 7>(A, x, y, ws, ws_bytes, s);
    case 11: return f64 ? launch_wt<double, 11>(A, x, y, ws, ws_bytes, s) : launch_wt<float, 11>(A, x, y, ws, ws_bytes, s);
    case 15: return f64 ? launch_wt<double, 15>(A, x, y, ws, ws_bytes, s) : launch_wt<float, 15>(A, x, y, ws, ws_bytes, s);
    case 19: return f64 ? launch_wt<double, 19>(A, x, y, ws, ws_bytes, s) : launch_wt<float, 19>(A, x, y, ws, ws_bytes, s);
    case 23: return f64 ? launch_wt<double, 23>(A, x, y, ws, ws_bytes, s) : launch_wt<float, 23>(A, x, y, ws, ws_bytes, s);
    case 27: return f64 ? launch_wt<double, 27>(A, x, y, ws, ws_bytes, s) : launch_wt<float, 27>(A, x, y, ws, ws_bytes, s);
    default: return f64 ? launch_wt<double, 31>(A, x, y, ws, ws_bytes, s) : launch_wt<float, 31>(A, x, y, ws, ws_bytes, s);
    }
}

}  // namespace msp
