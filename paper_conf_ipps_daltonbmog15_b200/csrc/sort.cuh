// sort.cuh -- stable CTA merge sort of 64-bit keys with an int payload.
//
// Used by SpGEMM to sort a tile's expanded products by (row, col) so that
// duplicates become adjacent (Fig 3(c); the north star's "block
// merge-sort networks").  Each thread sorts IPT register items with an
// odd-even transposition network (stable: swaps only on strict >), then
// log2(NT) rounds merge pairs of sorted runs through shared memory; the
// merge-path split of each thread's output range keeps every
// thread's work equal.  Ties take the left run first, so the sort is stable.
#pragma once

#include <cstdint>

#include "common.cuh"

namespace msp {

// Padded shared index: 1 pad element every 16 keys (breaks the 128-byte
// stride of the blocked layout).
__device__ __forceinline__ int sort_pad(int i) { return i + (i >> 4); }

template <int NT, int IPT, typename KT = uint64_t>
struct BlockSortSmem {
    KT keys[NT * IPT + (NT * IPT) / 16 + 2];
    int vals[NT * IPT + (NT * IPT) / 16 + 2];
};

template <int IPT, typename KT>
__device__ __forceinline__ void thread_sort(KT (&k)[IPT], int (&v)[IPT])
{
#pragma unroll
    for (int r = 0; r < IPT; ++r) {
#pragma unroll
        for (int i = (r & 1); i + 1 < IPT; i += 2) {
            if (k[i] > k[i + 1]) {
                const KT tk = k[i];
                k[i] = k[i + 1];
                k[i + 1] = tk;
                const int tv = v[i];
                v[i] = v[i + 1];
                v[i + 1] = tv;
            }
        }
    }
}

// Sorts NT*IPT (key, val) items held IPT per thread (any assignment of items
// to threads); on return thread t holds sorted items [t*IPT, (t+1)*IPT).
// All NT threads of the CTA must call (uses __syncthreads).
template <int NT, int IPT, typename KT>
__device__ __forceinline__ void block_merge_sort(KT (&k)[IPT], int (&v)[IPT], BlockSortSmem<NT, IPT, KT> &S)
{
    const int tid = threadIdx.x;
    constexpr KT KMAX = ~KT(0);
    thread_sort<IPT, KT>(k, v);
#pragma unroll 1
    for (int w = 1; w < NT; w <<= 1) {
#pragma unroll
        for (int i = 0; i < IPT; ++i) {
            S.keys[sort_pad(tid * IPT + i)] = k[i];
            S.vals[sort_pad(tid * IPT + i)] = v[i];
        }
        __syncthreads();
        const int r = tid & (2 * w - 1);           // rank inside the merging group
        const int g0 = (tid - r) * IPT;            // group start
        const int la = w * IPT, lb = w * IPT;      // both runs are full
        const int d = r * IPT;                     // output diagonal of this thread
        int lo = max(0, d - lb), hi = min(d, la);
        while (lo < hi) {
            const int mid = (lo + hi) >> 1;
            if (S.keys[sort_pad(g0 + mid)] <= S.keys[sort_pad(g0 + la + d - mid - 1)]) lo = mid + 1;
            else hi = mid;
        }
        int ia = lo, ib = d - lo;
        KT ka = ia < la ? S.keys[sort_pad(g0 + ia)] : KMAX;
        KT kb = ib < lb ? S.keys[sort_pad(g0 + la + ib)] : KMAX;
        // branch-free serial merge (lanes of a warp take different sides)
#pragma unroll
        for (int i = 0; i < IPT; ++i) {
            const bool takea = (ib >= lb) || (ia < la && ka <= kb);
            const int src = takea ? (g0 + ia) : (g0 + la + ib);
            k[i] = takea ? ka : kb;
            v[i] = S.vals[sort_pad(src)];
            ia += takea ? 1 : 0;
            ib += takea ? 0 : 1;
            const bool more = takea ? (ia < la) : (ib < lb);
            const KT kn = more ? S.keys[sort_pad(src + 1)] : KMAX;
            ka = takea ? kn : ka;
            kb = takea ? kb : kn;
        }
        __syncthreads();
    }
}

}  // namespace msp

namespace msp {

// ------------------------------------------------------------------------
// Run-aware merge sort of one SpGEMM tile (symbolic pass).
//
// A tile's products arrive in expansion order: rows in order,
// and inside a row the products of one A nonzero are one B row, already
// sorted by column.  So the staged keys are a sequence of sorted runs, and
// only runs of the SAME row ever need merging (keys of different rows are
// already ordered).  Runs are the maximal non-decreasing stretches that do
// not cross a row; each round merges runs 2c and 2c+1 of every row (merge
// path per thread, stable: ties take the earlier run), so a tile needs
// ceil(log2(max runs per row)) rounds -- 5 for the 27-point stencil -- in
// place of the IPT-step register sort plus log2(NT) rounds of the generic
// block merge sort.  Tiles with more than RM_MAXRUNS runs, or runs shorter
// than 8 keys on average, use the generic sort.
constexpr int RM_MAXRUNS = 2048;

template <int T, typename KT>
struct RunSortSmem {  // aliases the staging buffer once the run table is built
    KT keys[T + T / 16 + 2];
    uint16_t pay[T + T / 16 + 2];
};

struct RunTable {
    uint16_t start[RM_MAXRUNS + 1];     // first position of run q; start[R] = np
    uint16_t rowidx[RM_MAXRUNS];        // row (ordinal among the tile's rows) of run q
    uint16_t rowfirst[RM_MAXRUNS + 1];  // first run of each row; rowfirst[rows] = R
};

// On success thread t holds sorted positions [t*IPT, (t+1)*IPT) in k (keys,
// ~0 past np) and v (original slots).  Returns false (uniformly) if the tile
// has too many runs; k / v are then the unsorted slot-order contents.
template <int NT, int IPT, typename KT, class RowOf>
__device__ __forceinline__ bool run_merge_sort(const KT *stage, int np, RunSortSmem<NT * IPT, KT> &S, RunTable &R,
                                               int *wsum, RowOf rowof, KT (&k)[IPT], int (&v)[IPT])
{
    constexpr int NW = NT / 32;
    constexpr KT KMAX = ~KT(0);
    constexpr int RPT = RM_MAXRUNS / NT;  // runs per thread in the table passes
    __shared__ int s_maxruns;
    const int tid = threadIdx.x;
    const int d0 = tid * IPT;
    // ---- 1. my positions; run starts = descents or row changes ----
    unsigned smask = 0;
    int cnt = 0;
    {
        KT prev = (d0 > 0 && d0 <= np) ? stage[d0 - 1] : KT(0);
#pragma unroll
        for (int i = 0; i < IPT; ++i) {
            const int pos = d0 + i;
            const KT key = pos < np ? stage[pos] : KMAX;
            k[i] = key;
            v[i] = pos;
            if (pos < np && (pos == 0 || key < prev || rowof(key) != rowof(prev))) {
                smask |= 1u << i;
                ++cnt;
            }
            prev = key;
        }
    }
    if (tid == 0) s_maxruns = 0;
    int nruns;
    const int q0 = block_exclusive_sum<int, NW>(cnt, wsum, 0, &nruns);
    // short runs (mean < 8 keys: random sparse rows) merge no faster than
    // the generic sort, whose rounds never cross run boundaries
    if (nruns > RM_MAXRUNS || nruns * 8 > np) return false;
    for (unsigned b = smask, c = 0; b; b &= b - 1, ++c) R.start[q0 + c] = uint16_t(d0 + __ffs(b) - 1);
    if (tid == 0) R.start[nruns] = uint16_t(np);
    __syncthreads();
    // ---- 2. rows among runs ----
    unsigned hmask = 0;
    int hc = 0;
#pragma unroll
    for (int u = 0; u < RPT; ++u) {
        const int q = tid * RPT + u;
        if (q < nruns && (q == 0 || rowof(stage[R.start[q]]) != rowof(stage[R.start[q - 1]]))) {
            hmask |= 1u << u;
            ++hc;
        }
    }
    int nrows;
    const int r0 = block_exclusive_sum<int, NW>(hc, wsum, 0, &nrows);
    {
        int ri = r0 - 1;
#pragma unroll
        for (int u = 0; u < RPT; ++u) {
            const int q = tid * RPT + u;
            if (q < nruns) {
                if ((hmask >> u) & 1u) {
                    ++ri;
                    R.rowfirst[ri] = uint16_t(q);
                }
                R.rowidx[q] = uint16_t(ri);
            }
        }
    }
    if (tid == 0) R.rowfirst[nrows] = uint16_t(nruns);
    __syncthreads();
    // ---- 3. rounds = ceil(log2(max runs in a row)) ----
    {
        int mx = 0;
#pragma unroll
        for (int u = 0; u < RPT; ++u) {
            const int q = tid * RPT + u;
            if ((hmask >> u) & 1u) mx = max(mx, int(R.rowfirst[R.rowidx[q] + 1]) - q);
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
        if ((tid & 31) == 0 && mx > 0) atomicMax(&s_maxruns, mx);
    }
    __syncthreads();
    const int mr = s_maxruns;
    const int W = mr > 1 ? 32 - __clz(mr - 1) : 0;
    // ---- 4. merge rounds (in place through the padded buffer) ----
    for (int w = 0; w < W; ++w) {
        __syncthreads();  // previous readers of the buffer (or of the stage) are done
#pragma unroll
        for (int i = 0; i < IPT; ++i) {
            S.keys[sort_pad(d0 + i)] = k[i];
            S.pay[sort_pad(d0 + i)] = uint16_t(v[i]);
        }
        __syncthreads();
        if (d0 >= np) continue;
        auto key = [&](int p) { return S.keys[sort_pad(p)]; };
        int lo = 0, hi = nruns - 1;  // run holding d0: last q with start[q] <= d0
        while (lo < hi) {
            const int mid = (lo + hi + 1) >> 1;
            if (int(R.start[mid]) <= d0) lo = mid;
            else hi = mid - 1;
        }
        const int q = lo;
        int re = R.rowfirst[R.rowidx[q] + 1];
        const int rb = R.rowfirst[R.rowidx[q]];
        int qa = rb + (((q - rb) >> (w + 1)) << (w + 1));
        int qe, a0, b0, la, lb;
        auto setpair = [&]() {
            const int qm = min(qa + (1 << w), re);
            qe = min(qa + (2 << w), re);
            a0 = R.start[qa];
            b0 = R.start[qm];
            la = b0 - a0;
            lb = int(R.start[qe]) - b0;
        };
        setpair();
        const int diag = d0 - a0;
        int mlo = max(0, diag - lb), mhi = min(diag, la);
        while (mlo < mhi) {
            const int mid = (mlo + mhi) >> 1;
            if (key(a0 + mid) <= key(b0 + diag - mid - 1)) mlo = mid + 1;
            else mhi = mid;
        }
        int ia = mlo, ib = diag - mlo;
        KT ka = ia < la ? key(a0 + ia) : KMAX;
        KT kb = ib < lb ? key(b0 + ib) : KMAX;
#pragma unroll
        for (int i = 0; i < IPT; ++i) {
            const int pos = d0 + i;
            if (pos >= np) {
                k[i] = KMAX;
                v[i] = pos;
                continue;
            }
            if (ia >= la && ib >= lb) {  // pair done: next pair of this row, or the next row's first
                qa = qe;
                if (qa >= re) re = R.rowfirst[R.rowidx[qa] + 1];
                setpair();
                ia = 0;
                ib = 0;
                ka = key(a0);
                kb = lb > 0 ? key(b0) : KMAX;
            }
            const bool takea = (ib >= lb) || (ia < la && ka <= kb);
            const int src = takea ? (a0 + ia) : (b0 + ib);
            k[i] = takea ? ka : kb;
            v[i] = S.pay[sort_pad(src)];
            if (takea) {
                ++ia;
                ka = ia < la ? key(a0 + ia) : KMAX;
            } else {
                ++ib;
                kb = ib < lb ? key(b0 + ib) : KMAX;
            }
        }
    }
    return true;
}

}  // namespace msp
