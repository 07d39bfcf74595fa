// spadd.cu -- C = A + B as a balanced-path set union (sm_100a).
//
// Paper: Section III-B.  With both inputs sorted by row and by
// column within a row, SpAdd is the union of two sorted (row, col) tuple
// lists in Algorithm 1 order.  Merge path splits the
// merge into equal non-overlapping ranges; balanced path shifts a
// split by one B entry when a matched (equal key, equal rank) pair would
// straddle it (reading Z23), so every matched pair is reduced by
// one thread.  Two phases: count the unique tuples of each row,
// allocate C, then fill it.
//
// B200 design:
//   * The merge grid has the row ends as items too: item space = rows of C
//     + nnz(A) + nnz(B), so a tile of T items gets an equal share of rows
//     and elements whatever the row lengths (empty rows included).  A split
//     is found by a search over R_end[r] = A.rp[r+1] + B.rp[r+1] followed by
//     a merge-path search of A's and B's columns inside the split row, then
//     the balanced-path shift.
//   * partition kernel: one thread per tile boundary (the paper's partition
//     phase), results kept in the workspace and reused by the
//     numeric phase;
//   * tile kernel: one CTA per tile stages the tile's columns (and values)
//     in shared memory with coalesced loads, every thread finds its own
//     split in shared memory and walks IPT items serially; symbolic adds the
//     per-row unique counts into C.row_offsets (integer atomics are exact and
//     order-independent) and records the tile's unique count; a device scan
//     turns counts into offsets; numeric recounts, scans the per-thread
//     counts, stages its output run in shared memory and stores it
//     coalesced at the tile's offset.
//   * A matched pair gives (T)(a + b) with A's value first (Alg. 1): one
//     IEEE addition, so values are bit-exact with the oracle.
#include <algorithm>
#include <climits>
#include <cstdint>

#include "common.cuh"
#include "internal.h"

namespace msp {
namespace {

#ifndef MSP_ADD_NT
#define MSP_ADD_NT 128  // threads per tile: C3 one pass 0.880 -> 0.865 ms, C2 0.410 -> 0.389 ms vs 256 (64-512 swept)
#endif
constexpr int ADD_NT = MSP_ADD_NT;
#ifndef MSP_LB_BACKOFF
#define MSP_LB_BACKOFF 0  // 1: look-back spin with __nanosleep backoff (C3 0.882 -> 0.872 ms, C2 0.390 -> 0.410 ms: off)
#endif
#ifndef MSP_ADD_IPT
#define MSP_ADD_IPT 14  // measured on B200 (one-walk fill, 53-66 KB smem): C3 A+A^T 1.85 ms at 8, 1.42 at 12,
                        // 1.30 at 14, 1.31 at 16, 1.23 at 20; C2 0.47-0.49 ms at 12-20
#endif
constexpr int ADD_IPT = MSP_ADD_IPT;  // merge items per thread
constexpr int ADD_T = ADD_NT * ADD_IPT;  // merge items per tile
constexpr int ADD_STEPS = ADD_IPT + 1;   // register output slots per thread (fill)

struct Split {
    int32_t r, a, b;  // row (row-end items consumed), A index, B index (global)
};

// Merge path inside one row: first `d` merged entries of A[a_lo..a_hi) and
// B[b_lo..b_hi) (A first on equal columns, Alg. 1) end at (ia, ib).
template <class LA, class LB>
__device__ __forceinline__ void row_merge_path(LA Acol, int a_lo, int a_hi, LB Bcol, int b_lo, int b_hi, int d,
                                               int &ia, int &ib)
{
    const int la = a_hi - a_lo, lb = b_hi - b_lo;
    int lo = max(0, d - lb), hi = min(d, la);
    while (lo < hi) {
        const int mid = (lo + hi) >> 1;
        if (Acol(a_lo + mid) <= Bcol(b_lo + d - mid - 1)) lo = mid + 1;
        else hi = mid;
    }
    ia = a_lo + lo;
    ib = b_lo + d - lo;
}

// --------------------------------------------------------------- partition

__global__ void spadd_partition_kernel(int32_t m, int64_t nnzA, int64_t nnzB, const int32_t *__restrict__ Arp,
                                       const int32_t *__restrict__ Acol, const int32_t *__restrict__ Brp,
                                       const int32_t *__restrict__ Bcol, int64_t ntiles, Split *__restrict__ splits,
                                       uint64_t *__restrict__ states, unsigned *__restrict__ ticket)
{
    const int64_t E = nnzA + nnzB;
    const int64_t total = int64_t(m) + E;
    // fused form: clear the look-back state and the tile ticket (the fused
    // tile kernel runs after this launch on the same stream)
    if (states && blockIdx.x == 0 && threadIdx.x == 0) *ticket = 0u;
    for (int64_t k = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; k <= ntiles; k += int64_t(gridDim.x) * blockDim.x) {
        if (states && k < ntiles) states[k] = 0ull;
        const int64_t d = min(k * ADD_T, total);
        // rows: smallest i with NOT(R_end[i] <= d - i - 1)
        int64_t lo = max(int64_t(0), d - E), hi = min(d, int64_t(m));
        while (lo < hi) {
            const int64_t mid = (lo + hi) >> 1;
            const int64_t rend = int64_t(Arp[mid + 1]) + Brp[mid + 1];
            if (rend <= d - mid - 1) lo = mid + 1;
            else hi = mid;
        }
        Split s;
        const int r = int(lo);
        s.r = r;
        if (r >= m) {
            s.a = int(nnzA);
            s.b = int(nnzB);
        } else {
            const int o = int(d - r - (int64_t(Arp[r]) + Brp[r]));
            int ia, ib;
            row_merge_path([&](int i) { return Acol[i]; }, Arp[r], Arp[r + 1], [&](int i) { return Bcol[i]; },
                           Brp[r], Brp[r + 1], o, ia, ib);
            if (ia > Arp[r] && ib < Brp[r + 1] && Acol[ia - 1] == Bcol[ib]) ++ib;  // balanced path (Z23)
            s.a = ia;
            s.b = ib;
        }
        splits[k] = s;
    }
}

// --------------------------------------------------------------- tile kernel

// Shared-memory layout of one tile (one CTA per tile).  The int windows
// (A.rp, B.rp, A.col, B.col slices) and the value windows (A.val, B.val) are
// staged by TMA bulk copies; rows + nnzA + nnzB <= T items per tile bounds
// their total size.  Fill also stages its output run (col, val) so that C is
// written with coalesced stores.
template <typename V, bool FILL>
struct AddLayout {
    static constexpr int IBYTES = 4 * (2 * ADD_T + 8) + 4 * 32;        // 4 int windows (+alignment slack)
    static constexpr int VBYTES = FILL ? int(sizeof(V)) * ADD_T + 2 * 32 : 0;
    static constexpr int OBYTES = FILL ? (4 + int(sizeof(V))) * ADD_T : 0;
    static constexpr int V_OFF = IBYTES;
    // the output run overlays the input windows: it is written only after
    // the scan barrier, when every thread has finished reading them
    static constexpr int O_OFF = 0;
    static_assert(O_OFF + OBYTES <= V_OFF + VBYTES, "output run must fit over the input windows");
    static constexpr int ST_OFF = (V_OFF + VBYTES + 15) / 16 * 16;
    static constexpr int WS_OFF = ST_OFF + int(sizeof(Split)) * (ADD_NT + 1);
    static constexpr int BAR_OFF = (WS_OFF + 4 * (ADD_NT / 32) + 15) / 16 * 16;
    static constexpr int BYTES = BAR_OFF + 16;
};

// One staged window: elements [lo, hi) of an array of `len` elements, placed
// at a 16-byte aligned shared-memory offset; `first` = byte offset of lo.
struct Staged {
    WindowCopy w;
    int off;
};

template <typename T>
__device__ __forceinline__ Staged plan_stage(const T *base, int64_t lo, int64_t hi, int64_t len, int *off,
                                             uint32_t *tx)
{
    Staged st;
    st.w = plan_window<int(sizeof(T))>(base, lo, hi, len);
    st.off = *off;
    *off += int(st.w.span);
    *tx += st.w.bulk_bytes;
    return st;
}

// Thread 0 issues the bulk copy (after the barrier's expect_tx), lanes of
// warp 0 copy the ragged ends; returns a pointer to element lo.
template <typename T>
__device__ __forceinline__ T *issue_stage(const Staged &st, const T *base, int64_t lo, int64_t hi, char *smem,
                                          uint64_t *bar, uint64_t pol)
{
    char *dst = smem + st.off;
    if (threadIdx.x == 0 && st.w.bulk_bytes) bulk_g2s(dst + st.w.bulk_dst, st.w.bulk_src, st.w.bulk_bytes, bar, pol);
    if (threadIdx.x < 32) window_manual<T>(st.w, base, lo, hi, dst, threadIdx.x);
    return reinterpret_cast<T *>(dst + st.w.first);
}

// Tile kernel modes: COUNT (symbolic: per-row unique counts), FILL (numeric:
// writes C at the offsets the symbolic phase produced) and FUSED (one pass:
// the tile's output offset comes from a decoupled look-back over the tiles'
// output counts, and C.row_offsets from the row-end items -- DESIGN §4.2).
enum AddMode { ADD_COUNT = 0, ADD_FILL = 1, ADD_FUSED = 2 };
constexpr uint64_t AS_AGG = 1ull << 62, AS_PRE = 2ull << 62, AS_VAL = (1ull << 62) - 1;

template <typename V, int MODE>
__global__ void __launch_bounds__(ADD_NT)
spadd_tile_kernel(int32_t m, const int32_t *__restrict__ Arp, const int32_t *__restrict__ Acol,
                  const V *__restrict__ Aval, const int32_t *__restrict__ Brp, const int32_t *__restrict__ Bcol,
                  const V *__restrict__ Bval, int64_t nnzA, int64_t nnzB, const Split *__restrict__ splits,
                  int32_t *__restrict__ tile_count, const int64_t *__restrict__ tile_off,
                  int32_t *__restrict__ Crp_counts, int32_t *__restrict__ Ccol, V *__restrict__ Cval,
                  uint64_t *__restrict__ states, unsigned *__restrict__ ticket, int64_t *__restrict__ totals,
                  int64_t ntiles, int64_t cap)
{
    constexpr bool FILL = MODE != ADD_COUNT;
    constexpr bool FUSED = MODE == ADD_FUSED;
    using L = AddLayout<V, FILL>;
    extern __shared__ __align__(128) char smem_raw[];
    Split *S_st = reinterpret_cast<Split *>(smem_raw + L::ST_OFF);
    int32_t *S_wsum = reinterpret_cast<int32_t *>(smem_raw + L::WS_OFF);
    uint64_t *bar = reinterpret_cast<uint64_t *>(smem_raw + L::BAR_OFF);
    __shared__ int s_tile;
    __shared__ int64_t s_base;
    const int tid = threadIdx.x;
    int k = blockIdx.x;
    if constexpr (FUSED) {
        // tiles in claim order: the look-back never waits on an unstarted tile
        if (tid == 0) s_tile = int(atomicAdd(ticket, 1u));
        __syncthreads();
        k = s_tile;
    }
    const Split s0 = splits[k], s1 = splits[k + 1];
    const int r0 = s0.r, r1 = s1.r;
    const int ga0 = s0.a, gb0 = s0.b;
    const int nA = s1.a - ga0, nB = s1.b - gb0;
    const int nrw = min(r1, m - 1) - r0 + 2;  // row offsets r0 .. min(r1, m-1)+1
    // ---- stage the tile: one TMA bulk copy per window ----
    // Warp 0 plans the windows (the other warps only need their shared-memory
    // offsets, published with the barrier below) and copies their ragged ends.
    __shared__ int s_first[6];
    if (tid < 32) {
        if (tid == 0) {
            mbar_init(bar, 1);
            fence_mbar_init();
        }
        __syncwarp();
        const uint64_t pol = policy_evict_first();
        int ioff = 0, voff = L::V_OFF;
        uint32_t tx = 0;
        const Staged p_arp = plan_stage<int32_t>(Arp, r0, r0 + nrw, int64_t(m) + 1, &ioff, &tx);
        const Staged p_brp = plan_stage<int32_t>(Brp, r0, r0 + nrw, int64_t(m) + 1, &ioff, &tx);
        const Staged p_ac = plan_stage<int32_t>(Acol, ga0, ga0 + nA, nnzA, &ioff, &tx);
        const Staged p_bc = plan_stage<int32_t>(Bcol, gb0, gb0 + nB, nnzB, &ioff, &tx);
        Staged p_av{}, p_bv{};
        if constexpr (FILL) {
            p_av = plan_stage<V>(Aval, ga0, ga0 + nA, nnzA, &voff, &tx);
            p_bv = plan_stage<V>(Bval, gb0, gb0 + nB, nnzB, &voff, &tx);
        }
        if (tid == 0) mbar_arrive_expect_tx(bar, tx);
        int32_t *w_arp = issue_stage<int32_t>(p_arp, Arp, r0, r0 + nrw, smem_raw, bar, 0);
        int32_t *w_brp = issue_stage<int32_t>(p_brp, Brp, r0, r0 + nrw, smem_raw, bar, 0);
        const int32_t *w_ac = issue_stage<int32_t>(p_ac, Acol, ga0, ga0 + nA, smem_raw, bar, pol);
        const int32_t *w_bc = issue_stage<int32_t>(p_bc, Bcol, gb0, gb0 + nB, smem_raw, bar, pol);
        if (tid == 0) {
            s_first[0] = int(reinterpret_cast<char *>(w_arp) - smem_raw);
            s_first[1] = int(reinterpret_cast<char *>(w_brp) - smem_raw);
            s_first[2] = int(reinterpret_cast<const char *>(w_ac) - smem_raw);
            s_first[3] = int(reinterpret_cast<const char *>(w_bc) - smem_raw);
        }
        if constexpr (FILL) {
            const V *w_av = issue_stage<V>(p_av, Aval, ga0, ga0 + nA, smem_raw, bar, pol);
            const V *w_bv = issue_stage<V>(p_bv, Bval, gb0, gb0 + nB, smem_raw, bar, pol);
            if (tid == 0) {
                s_first[4] = int(reinterpret_cast<const char *>(w_av) - smem_raw);
                s_first[5] = int(reinterpret_cast<const char *>(w_bv) - smem_raw);
            }
        }
    }
    __syncthreads();  // mbarrier initialised, window offsets published
    int32_t *arp = reinterpret_cast<int32_t *>(smem_raw + s_first[0]);
    int32_t *brp = reinterpret_cast<int32_t *>(smem_raw + s_first[1]);
    const int32_t *acs = reinterpret_cast<const int32_t *>(smem_raw + s_first[2]);
    const int32_t *bcs = reinterpret_cast<const int32_t *>(smem_raw + s_first[3]);
    const V *avs = nullptr, *bvs = nullptr;
    if constexpr (FILL) {
        avs = reinterpret_cast<const V *>(smem_raw + s_first[4]);
        bvs = reinterpret_cast<const V *>(smem_raw + s_first[5]);
    }
    mbar_wait(bar, 0);
    __syncthreads();  // ragged ends written by warp 0
    for (int i = tid; i < nrw; i += ADD_NT) {  // tile-relative row offsets
        arp[i] -= ga0;
        brp[i] -= gb0;
    }
    __syncthreads();
    const int nrows = r1 - r0;  // row-end items in the tile
    const int items = nrows + nA + nB;
    auto a_lo = [&](int r) { return max(arp[r - r0], 0); };
    auto a_hi = [&](int r) { return min(arp[r - r0 + 1], nA); };
    auto b_lo = [&](int r) { return max(brp[r - r0], 0); };
    auto b_hi = [&](int r) { return min(brp[r - r0 + 1], nB); };
    auto acol = [&](int i) { return acs[i]; };
    auto bcol = [&](int i) { return bcs[i]; };
    // ---- this thread's split ----
    {
        const int dt = min(tid * ADD_IPT, items);
        int lo = max(0, dt - (nA + nB)), hi = min(dt, nrows);
        while (lo < hi) {
            const int mid = (lo + hi) >> 1;
            const int rend = min(arp[mid + 1], nA) + min(brp[mid + 1], nB);
            if (rend <= dt - mid - 1) lo = mid + 1;
            else hi = mid;
        }
        Split st;
        st.r = r0 + lo;
        const int e = dt - lo;  // tile-relative merged elements before the split
        if (st.r >= m || (st.r == r1 && e >= nA + nB)) {
            st.a = nA;
            st.b = nB;
        } else {
            const int r = st.r;
            const int al = a_lo(r), ah = a_hi(r), bl = b_lo(r), bh = b_hi(r);
            int ia, ib;
            row_merge_path(acol, al, ah, bcol, bl, bh, e - (al + bl), ia, ib);
            if (ia > al && ib < bh && acs[ia - 1] == bcs[ib]) ++ib;  // balanced path
            st.a = ia;
            st.b = ib;
        }
        S_st[tid] = st;
        if (tid == 0) S_st[ADD_NT] = Split{r1, nA, nB};
    }
    __syncthreads();
    const Split beg = S_st[tid], end = S_st[tid + 1];

    // ---- walk: Alg. 1 order; row-end items close rows ----
    auto walk = [&](auto &&on_out, auto &&on_row_end) {
        int r = beg.r, ia = beg.a, ib = beg.b;
        int ah = (r < m) ? a_hi(r) : nA, bh = (r < m) ? b_hi(r) : nB;
        while (r != end.r || ia != end.a || ib != end.b) {
            const bool ra = ia < ah, rb = ib < bh;
            if (!ra && !rb) {  // row r exhausted in this tile: its row-end item
                on_row_end(r);
                ++r;
                if (r < m) {
                    ah = a_hi(r);
                    bh = b_hi(r);
                }
                continue;
            }
            const int ca = ra ? acs[ia] : INT_MAX, cb = rb ? bcs[ib] : INT_MAX;
            if (ca <= cb) {
                if (ca == cb) {
                    on_out(ca, ia, ib);
                    ++ia;
                    ++ib;
                } else {
                    on_out(ca, ia, -1);
                    ++ia;
                }
            } else {
                on_out(cb, -1, ib);
                ++ib;
            }
        }
        return r;
    };

    if constexpr (!FILL) {
        int cnt = 0, total = 0;
        const int r_last = walk([&](int, int, int) { ++cnt; ++total; },
                                [&](int r) {
                                    if (cnt) atomicAdd(&Crp_counts[r], cnt);
                                    cnt = 0;
                                });
        if (cnt) atomicAdd(&Crp_counts[r_last], cnt);  // row continuing past this thread
        // tile's unique count
        int wsum = total;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) wsum += __shfl_xor_sync(0xffffffffu, wsum, o);
        if ((tid & 31) == 0) S_wsum[tid >> 5] = wsum;
        __syncthreads();
        if (tid == 0) {
            int t = 0;
            for (int w = 0; w < ADD_NT / 32; ++w) t += S_wsum[w];
            tile_count[k] = t;
        }
    } else {
        int32_t *ocol = reinterpret_cast<int32_t *>(smem_raw + L::O_OFF);
        V *oval = reinterpret_cast<V *>(smem_raw + L::O_OFF + 4 * ADD_T);
        // A thread's path holds (end - beg) items over the three coordinates
        // and every step consumes >= 1 of them: when all fit ADD_STEPS static
        // register slots, ONE walk forms the outputs (CTA-uniform choice;
        // otherwise count, scan, walk again).
        const int nit = (end.r - beg.r) + (end.a - beg.a) + (end.b - beg.b);
#ifdef MSP_ADD_FORCE_WALK2  // test build: exercise the fallback path
        const bool regs = __syncthreads_and(nit < 0);
#else
        const bool regs = __syncthreads_and(nit <= ADD_STEPS);
#endif
        int cnt = 0;
        int rc[ADD_STEPS];
        V rv[ADD_STEPS];
        unsigned em = 0, rem = 0;  // output steps, row-end steps
        if (regs) {
            int r = beg.r, ia = beg.a, ib = beg.b;
            int ah = (r < m) ? a_hi(r) : nA, bh = (r < m) ? b_hi(r) : nB;
#pragma unroll
            for (int st = 0; st < ADD_STEPS; ++st) {
                if (r != end.r || ia != end.a || ib != end.b) {
                    const bool ra = ia < ah, rb = ib < bh;
                    if (!ra && !rb) {  // row-end item
                        rem |= 1u << st;
                        ++r;
                        if (r < m) {
                            ah = a_hi(r);
                            bh = b_hi(r);
                        }
                    } else {
                        const int ca = ra ? acs[ia] : INT_MAX, cb = rb ? bcs[ib] : INT_MAX;
                        if (ca <= cb) {
                            rc[st] = ca;
                            rv[st] = (ca == cb) ? avs[ia] + bvs[ib] : avs[ia];  // one rounding, A first (Alg. 1)
                            ib += (ca == cb);
                            ++ia;
                        } else {
                            rc[st] = cb;
                            rv[st] = bvs[ib];
                            ++ib;
                        }
                        em |= 1u << st;
                        ++cnt;
                    }
                }
            }
        } else {
            walk([&](int, int, int) { ++cnt; }, [&](int) {});
        }
        int tot;
        int o = block_exclusive_sum<int, ADD_NT / 32>(cnt, S_wsum, 0, &tot);
        const int o_thread = o;
        if constexpr (FUSED) {
            if (tid < 32) {  // decoupled look-back over the tiles' output counts (warp 0)
                const int lane = tid;
                int64_t excl = 0;
                if (k == 0) {
                    if (lane == 0)  // flag and value share one word: no fence needed
                        atomicExch(reinterpret_cast<unsigned long long *>(&states[0]),
                                   (unsigned long long)(AS_PRE | uint64_t(tot)));
                } else {
                    if (lane == 0)
                        atomicExch(reinterpret_cast<unsigned long long *>(&states[k]),
                                   (unsigned long long)(AS_AGG | uint64_t(tot)));
                    for (int pos = k - 1;; pos -= 32) {
                        const int q = pos - lane;
                        uint64_t sw = AS_PRE;  // virtual prefix 0 before tile 0
                        if (q >= 0) {
                            sw = *reinterpret_cast<volatile uint64_t *>(&states[q]);
#if MSP_LB_BACKOFF
                            // predecessor not published yet: back off (the spin
                            // took 18 % of the kernel's issued instructions)
                            for (unsigned ns = 32; (sw & ~AS_VAL) == 0; ns = ns < 256 ? 2 * ns : ns) {
                                __nanosleep(ns);
                                sw = *reinterpret_cast<volatile uint64_t *>(&states[q]);
                            }
#else
                            while ((sw & ~AS_VAL) == 0)  // predecessor not published yet
                                sw = *reinterpret_cast<volatile uint64_t *>(&states[q]);
#endif
                        }
                        const unsigned pre = __ballot_sync(0xffffffffu, (sw & AS_PRE) != 0);
                        const int stop = pre ? __ffs(pre) - 1 : 32;  // nearest predecessor with a prefix
                        int64_t v = lane <= stop ? int64_t(sw & AS_VAL) : 0;
#pragma unroll
                        for (int d = 16; d > 0; d >>= 1) v += __shfl_xor_sync(0xffffffffu, v, d);
                        excl += v;
                        if (pre) break;
                    }
                    if (lane == 0)
                        atomicExch(reinterpret_cast<unsigned long long *>(&states[k]),
                                   (unsigned long long)(AS_PRE | uint64_t(excl + tot)));
                }
                if (lane == 0) {
                    s_base = excl;
                    if (k == ntiles - 1) totals[1] = excl + tot;  // nnz(C) by the tiles
                }
            }
        }
        if (regs) {
#pragma unroll
            for (int st = 0; st < ADD_STEPS; ++st) {
                if ((em & (1u << st)) && o < ADD_T) {  // bound binds only on malformed input
                    ocol[o] = rc[st];
                    oval[o] = rv[st];
                    ++o;
                }
            }
        }
        if constexpr (FUSED) __syncthreads();  // s_base published
        int64_t tbase;
        if constexpr (FUSED) tbase = s_base;
        else tbase = tile_off[k];
        if constexpr (FUSED) {
            if (k == 0 && tid == 0) Crp_counts[0] = 0;
            if (regs && rem) {  // C.row_offsets[r+1] at each row end of this thread's path
                int r = beg.r, p = o_thread;
#pragma unroll
                for (int st = 0; st < ADD_STEPS; ++st) {
                    if (rem & (1u << st)) {
                        Crp_counts[r + 1] = int32_t(tbase + p);
                        ++r;
                    }
                    p += (em >> st) & 1u;
                }
            }
        }
        if (!regs) {  // fallback: the windows are still being read, store straight to C
            int64_t p = tbase + o_thread;
            walk(
                [&](int c, int ia, int ib) {
                    V v;
                    if (ia >= 0 && ib >= 0) v = avs[ia] + bvs[ib];  // one rounding, A first (Alg. 1)
                    else v = (ia >= 0) ? avs[ia] : bvs[ib];
                    if (p < cap) {  // binds only on malformed (unsorted) input in the fused form
                        Ccol[p] = c;
                        Cval[p] = v;
                    }
                    ++p;
                },
                [&](int r) {
                    if constexpr (FUSED) Crp_counts[r + 1] = int32_t(p);
                });
        }
        if (regs) {
            __syncthreads();
            // the tile's run of C is contiguous: coalesced stores
            const int64_t base = tbase;
            // min(tot, ADD_T) and the capacity bind only on malformed input
            const int64_t room = cap - base > 0 ? cap - base : 0;
            const int nst = int(room < int64_t(min(tot, ADD_T)) ? room : int64_t(min(tot, ADD_T)));
            for (int i = tid; i < nst; i += ADD_NT) {
                Ccol[base + i] = ocol[i];
                Cval[base + i] = oval[i];
            }
        }
    }
}

struct AddWs {
    Split *splits;
    int32_t *tile_count;
    int64_t *tile_off;  // [ntiles + 1]
    int64_t *totals;    // [4]
    uint64_t *states;   // [ntiles] fused form: look-back status words
    unsigned *ticket;   // [4]      fused form: tile claim counter
    void *scan;
    size_t scan_bytes;
    int64_t ntiles;
    size_t bytes;  // total workspace bytes used
};

AddWs carve_ws(const msp_csr *A, const msp_csr *B, void *ws, size_t bytes, bool *ok)
{
    AddWs w;
    const int64_t items = int64_t(A->nrows) + A->nnz + B->nnz;
    w.ntiles = ceil_div(items > 0 ? items : 1, ADD_T);
    Carve cv(ws, bytes);
    w.splits = cv.take<Split>(size_t(w.ntiles + 1));
    w.tile_count = cv.take<int32_t>(size_t(w.ntiles));
    w.tile_off = cv.take<int64_t>(size_t(w.ntiles + 1));
    w.totals = cv.take<int64_t>(4);
    w.states = cv.take<uint64_t>(size_t(w.ntiles));
    w.ticket = cv.take<unsigned>(4);
    w.scan_bytes = scan_ws_bytes(std::max<int64_t>(A->nrows, w.ntiles));
    w.scan = cv.take<char>(w.scan_bytes);
    w.bytes = cv.off;
    *ok = cv.ok();
    return w;
}

template <typename V, int MODE>
msp_status launch_tiles(const msp_csr *A, const msp_csr *B, const AddWs &w, int32_t *Crp, int32_t *Ccol, void *Cval,
                        int64_t cap, cudaStream_t s)
{
    auto kern = spadd_tile_kernel<V, MODE>;
    const int smem = AddLayout<V, MODE != ADD_COUNT>::BYTES;
    msp_status st = set_smem_attr(reinterpret_cast<const void *>(kern), smem, "spadd: smem");
    if (st != MSP_OK) return st;
    // COUNT adds row counts into Crp + 1; FUSED writes Crp[0 .. m] itself
    int32_t *rp = Crp ? (MODE == ADD_FUSED ? Crp : Crp + 1) : nullptr;
    kern<<<unsigned(w.ntiles), ADD_NT, smem, s>>>(
        A->nrows, A->row_offsets, A->col_idx, static_cast<const V *>(A->vals), B->row_offsets, B->col_idx,
        static_cast<const V *>(B->vals), A->nnz, B->nnz, w.splits, w.tile_count, w.tile_off, rp, Ccol,
        static_cast<V *>(Cval), w.states, w.ticket, w.totals, w.ntiles, cap);
    return last_launch(MODE == ADD_FUSED ? "spadd_tile_kernel<fused>"
                                         : MODE == ADD_FILL ? "spadd_tile_kernel<fill>" : "spadd_tile_kernel<count>");
}

msp_status launch_partition(const msp_csr *A, const msp_csr *B, const AddWs &w, bool fused, cudaStream_t s)
{
    const int64_t n = w.ntiles + 1;
    const unsigned blocks = unsigned(std::min<int64_t>(ceil_div(n, 256), 148 * 8));
    spadd_partition_kernel<<<blocks, 256, 0, s>>>(A->nrows, A->nnz, B->nnz, A->row_offsets, A->col_idx,
                                                  B->row_offsets, B->col_idx, w.ntiles, w.splits,
                                                  fused ? w.states : nullptr, w.ticket);
    return last_launch("spadd_partition_kernel");
}

}  // namespace

size_t spadd_ws_bytes(const msp_csr *A, const msp_csr *B)
{
    bool ok;
    AddWs w = carve_ws(A, B, nullptr, SIZE_MAX, &ok);
    return w.bytes + 256;
}

msp_status spadd_symbolic_run(const msp_csr *A, const msp_csr *B, int32_t *Crp, int64_t *nnzC, void *ws,
                              size_t ws_bytes, cudaStream_t s)
{
    bool ok;
    AddWs w = carve_ws(A, B, ws, ws_bytes, &ok);
    if (!ok) return MSP_ERR_WORKSPACE;
    const int32_t m = A->nrows;
    msp_status st = cuda_check(cudaMemsetAsync(Crp, 0, (size_t(m) + 1) * sizeof(int32_t), s), "spadd: clear rp");
    if (st != MSP_OK) return st;
    if (m == 0) {
        *nnzC = 0;
        return cuda_check(cudaStreamSynchronize(s), "spadd: sync");
    }
    st = launch_partition(A, B, w, false, s);
    if (st != MSP_OK) return st;
    st = (A->dtype == MSP_F64) ? launch_tiles<double, ADD_COUNT>(A, B, w, Crp, nullptr, nullptr, INT64_MAX, s)
                               : launch_tiles<float, ADD_COUNT>(A, B, w, Crp, nullptr, nullptr, INT64_MAX, s);
    if (st != MSP_OK) return st;
    // row counts -> C.row_offsets (in place, Crp[0] stays 0); tile counts -> offsets
    st = scan_counts_to_offsets_i32(Crp + 1, m, &w.totals[0], w.scan, w.scan_bytes, s);
    if (st != MSP_OK) return st;
    st = scan_i32_to_i64(w.tile_count, w.tile_off, w.ntiles, w.scan, w.scan_bytes, s);
    if (st != MSP_OK) return st;
    int64_t hbuf[2] = {0, 0};
    int64_t *pin = pinned_scratch();
    int64_t *h = pin ? pin : hbuf;
    st = cuda_check(cudaMemcpyAsync(&h[0], &w.totals[0], sizeof(int64_t), cudaMemcpyDeviceToHost, s), "spadd: nnz");
    if (st != MSP_OK) return st;
    st = cuda_check(cudaMemcpyAsync(&h[1], &w.tile_off[w.ntiles], sizeof(int64_t), cudaMemcpyDeviceToHost, s),
                    "spadd: nnz");
    if (st != MSP_OK) return st;
    st = cuda_check(cudaStreamSynchronize(s), "spadd: sync");
    if (st != MSP_OK) return st;
    if (h[0] != h[1]) {
        set_error("spadd: row total %lld != tile total %lld (unsorted or duplicate columns?)", (long long)h[0],
                  (long long)h[1]);
        return MSP_ERR_INPUT;
    }
    *nnzC = h[0];
    if (h[0] > INT32_MAX) {
        set_error("spadd: nnz(C) = %lld exceeds int32", (long long)h[0]);
        return MSP_ERR_OVERFLOW;
    }
    return MSP_OK;
}

msp_status spadd_numeric_run(const msp_csr *A, const msp_csr *B, const int32_t *Crp, int32_t *Ccol, void *Cval,
                             void *ws, size_t ws_bytes, cudaStream_t s)
{
    bool ok;
    AddWs w = carve_ws(A, B, ws, ws_bytes, &ok);
    if (!ok) return MSP_ERR_WORKSPACE;
    (void)Crp;
    if (A->nrows == 0) return MSP_OK;
    return (A->dtype == MSP_F64) ? launch_tiles<double, ADD_FILL>(A, B, w, nullptr, Ccol, Cval, INT64_MAX, s)
                                 : launch_tiles<float, ADD_FILL>(A, B, w, nullptr, Ccol, Cval, INT64_MAX, s);
}

msp_status spadd_fused_run(const msp_csr *A, const msp_csr *B, int32_t *Crp, int32_t *Ccol, void *Cval, int64_t cap,
                           int64_t *nnzC, void *ws, size_t ws_bytes, cudaStream_t s)
{
    bool ok;
    AddWs w = carve_ws(A, B, ws, ws_bytes, &ok);
    if (!ok) return MSP_ERR_WORKSPACE;
    const int32_t m = A->nrows;
    msp_status st;
    if (m == 0) {
        *nnzC = 0;
        st = cuda_check(cudaMemsetAsync(Crp, 0, sizeof(int32_t), s), "spadd: rp");
        if (st != MSP_OK) return st;
        return cuda_check(cudaStreamSynchronize(s), "spadd: sync");
    }
    st = launch_partition(A, B, w, true, s);
    if (st != MSP_OK) return st;
    st = (A->dtype == MSP_F64) ? launch_tiles<double, ADD_FUSED>(A, B, w, Crp, Ccol, Cval, cap, s)
                               : launch_tiles<float, ADD_FUSED>(A, B, w, Crp, Ccol, Cval, cap, s);
    if (st != MSP_OK) return st;
    // nnz(C) twice: C.row_offsets[m] (from the row ends) and the tiles' total
    int64_t hbuf[2] = {0, 0};
    int64_t *pin = pinned_scratch();
    int64_t *h = pin ? pin : hbuf;
    h[0] = 0;
    st = cuda_check(cudaMemcpyAsync(&h[0], Crp + m, sizeof(int32_t), cudaMemcpyDeviceToHost, s), "spadd: nnz");
    if (st != MSP_OK) return st;
    st = cuda_check(cudaMemcpyAsync(&h[1], &w.totals[1], sizeof(int64_t), cudaMemcpyDeviceToHost, s), "spadd: nnz");
    if (st != MSP_OK) return st;
    st = cuda_check(cudaStreamSynchronize(s), "spadd: sync");
    if (st != MSP_OK) return st;
    const int64_t rows_total = int64_t(int32_t(uint32_t(uint64_t(h[0]))));
    if (h[1] > INT32_MAX) {
        set_error("spadd: nnz(C) = %lld exceeds int32", (long long)h[1]);
        return MSP_ERR_OVERFLOW;
    }
    if (rows_total != h[1] || h[1] > cap) {
        set_error("spadd: row total %lld != tile total %lld (unsorted or duplicate columns?)", (long long)rows_total,
                  (long long)h[1]);
        return MSP_ERR_INPUT;
    }
    *nnzC = h[1];
    return MSP_OK;
}

}  // namespace msp
