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
