// spgemm_radix.cu -- the paper's own SpGEMM sort pipeline as an ablation
// (SURVEY §8(f) f2), sm_100a.
//
// Paper: Section III-C, Figs 3 and 4.  Three phases:
//   1. per CTA tile of RT products (the products split evenly over CTAs by
//      the prefix S): expand the (row, col) indices only, "a
//      single radix sort on the column indices" -- rows stay ordered because
//      products are expanded in row order, so duplicates become adjacent
//       -- sorting only ceil(log2 n) column bits with the
//      permutation packed in the spare low bits (keys-only sort,
//      P:1122-1140), store the permutation as 16-bit integers,
//      reduce duplicates and store the reduced (row, col) entries
//      (P:1146-1152);
//   2. a global radix sort of the reduced entries by (row, col) that
//      "computes only the permutation";
//   3. re-expansion with values: each CTA loads its permutation and reduces
//      its permuted products by the precomputed duplicate flags, storing the
//      reduced values at their globally sorted positions; a global
//      reduce-by-key forms C.
// B200 choices: 4-bit LSD counting passes in shared memory for the CTA sort
// (stable, keys-only); 8-bit global LSD passes (histogram, scan, scatter with
// a stable in-CTA ranking); the tile outputs are compacted in tile order
// through a decoupled look-back, so the whole pipeline is deterministic.
// Compared with the shipped pipeline (spgemm.cu: merge sort by (row, col),
// rows kept inside tiles) this sorts far more entries globally; it is kept as
// the measured ablation the survey asks for.
#include <algorithm>
#include <climits>
#include <cstdint>
#include <cstdlib>

#include "common.cuh"
#include "internal.h"

namespace msp {
namespace {

constexpr int RX_NT = 256;
constexpr int RX_VT = 8;
constexpr int RX_T = RX_NT * RX_VT;  // products per tile (the paper: 128 threads x 11)
constexpr int RX_PB = 11;            // bits of a tile-local index
constexpr int GX_VT = 16;
constexpr int GX_T = RX_NT * GX_VT;  // reduced entries per global-sort tile

// ---- stable 4-bit LSD counting pass over n <= NT*VT keys (+ values) held in
// shared memory, thread t owning the blocked range [t*VT, t*VT+VT).  cnt:
// [16][NT] uint32.  Output to (ko, vo).  All threads of the CTA call it.
template <int VT, typename K, typename V, class Digit>
__device__ __forceinline__ void cta_pass4d(const K *ki, const V *vi, K *ko, V *vo, int n, Digit digit, uint32_t *cnt,
                                           uint32_t *wsum)
{
    const int tid = threadIdx.x;
    uint32_t c[16];
#pragma unroll
    for (int d = 0; d < 16; ++d) c[d] = 0;
    int dg[VT];
#pragma unroll
    for (int u = 0; u < VT; ++u) {
        const int i = tid * VT + u;
        dg[u] = (i < n) ? digit(ki[i]) : -1;
#pragma unroll
        for (int d = 0; d < 16; ++d) c[d] += (dg[u] == d);
    }
#pragma unroll
    for (int d = 0; d < 16; ++d) cnt[d * RX_NT + tid] = c[d];
    __syncthreads();
    // exclusive scan of cnt in (digit, thread) order: thread t owns the 16
    // consecutive entries [16t, 16t+16)
    uint32_t loc[16], run = 0;
#pragma unroll
    for (int e = 0; e < 16; ++e) {
        loc[e] = run;
        run += cnt[tid * 16 + e];
    }
    uint32_t tot;
    const uint32_t base = block_exclusive_sum<uint32_t, RX_NT / 32>(run, wsum, 1, &tot);
#pragma unroll
    for (int e = 0; e < 16; ++e) cnt[tid * 16 + e] = base + loc[e];
    __syncthreads();
#pragma unroll
    for (int d = 0; d < 16; ++d) c[d] = cnt[d * RX_NT + tid];
#pragma unroll
    for (int u = 0; u < VT; ++u) {
        const int i = tid * VT + u;
        if (dg[u] >= 0) {
            uint32_t p = 0;
#pragma unroll
            for (int d = 0; d < 16; ++d)
                if (dg[u] == d) p = c[d]++;
            ko[p] = ki[i];
            vo[p] = vi[i];
        }
    }
    __syncthreads();
}

template <int VT, typename K, typename V>
__device__ __forceinline__ void cta_pass4(const K *ki, const V *vi, K *ko, V *vo, int n, int shift, uint32_t *cnt,
                                          uint32_t *wsum)
{
    cta_pass4d<VT>(ki, vi, ko, vo, n, [&](K k) { return int((k >> shift) & 15); }, cnt, wsum);
}

// ---- decoupled look-back for tile output offsets (deterministic tile order)
constexpr uint64_t LB_AGG = 1ull << 62, LB_PRE = 2ull << 62, LB_VAL = (1ull << 62) - 1;

__device__ int64_t tile_prefix(uint64_t *states, int64_t tile, int64_t count)
{
    // warp 0 only; returns the exclusive prefix of `tile`
    const int lane = threadIdx.x & 31;
    int64_t excl = 0;
    if (tile == 0) {
        if (lane == 0) atomicExch(reinterpret_cast<unsigned long long *>(&states[0]), LB_PRE | uint64_t(count));
        return 0;
    }
    if (lane == 0) atomicExch(reinterpret_cast<unsigned long long *>(&states[tile]), LB_AGG | uint64_t(count));
    for (int64_t pos = tile - 1;; pos -= 32) {
        const int64_t k = pos - lane;
        uint64_t st = LB_PRE;
        if (k >= 0) {
            do {
                st = *reinterpret_cast<volatile uint64_t *>(&states[k]);
            } while ((st & ~LB_VAL) == 0);
        }
        const unsigned pre = __ballot_sync(0xffffffffu, (st & LB_PRE) != 0);
        const int stop = pre ? __ffs(pre) - 1 : 32;
        int64_t v = lane <= stop ? int64_t(st & LB_VAL) : 0;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
        excl += v;
        if (pre) break;
    }
    if (lane == 0) atomicExch(reinterpret_cast<unsigned long long *>(&states[tile]), LB_PRE | uint64_t(excl + count));
    return excl;
}

// ================================ phase 1 ==================================
// Symbolic: expand (row, col), keys-only radix by column bits (index in the
// low RX_PB bits), duplicates, reduced entries (packed (row << cb) | col) in
// tile order, 16-bit permutation and head flags per tile.
template <typename K>
__global__ void __launch_bounds__(RX_NT)
rx_tile_kernel(int64_t nprods, int64_t nnzA, const int32_t *__restrict__ Acol, const int32_t *__restrict__ Brp,
               const int32_t *__restrict__ Bcol, const int32_t *__restrict__ arow, const int64_t *__restrict__ S,
               int cb, uint16_t *__restrict__ perm, uint32_t *__restrict__ heads, int32_t *__restrict__ tcount,
               int64_t *__restrict__ toff, uint64_t *__restrict__ states, uint64_t *__restrict__ red,
               unsigned long long *__restrict__ ticket, int sort_bits, int row_bits)
{
    extern __shared__ __align__(16) char rx_smem[];
    K *ka = reinterpret_cast<K *>(rx_smem);
    K *kb = ka + RX_T;
    uint16_t *va = reinterpret_cast<uint16_t *>(kb + RX_T);
    uint16_t *vb = va + RX_T;
    int32_t *rows = reinterpret_cast<int32_t *>(vb + RX_T);
    uint32_t *cnt = reinterpret_cast<uint32_t *>(rows + RX_T);  // [16][RX_NT]
    __shared__ uint32_t wsum[RX_NT / 32];
    __shared__ int64_t s_j0, s_j1, s_base;
    __shared__ uint32_t s_heads[RX_T / 32];
    const int tid = threadIdx.x;
    __shared__ int64_t s_tile;
    // tiles in claim order: the look-back below never waits on an unstarted tile
    if (tid == 0) s_tile = int64_t(atomicAdd(ticket, 1ull));
    __syncthreads();
    const int64_t tile = s_tile;
    const int64_t p0 = tile * RX_T;
    const int n = int(min(int64_t(RX_T), nprods - p0));
    if (tid < 2) {  // first / last A nonzero of the tile: upper_bound(S, p) - 1 (reading Z7)
        const int64_t pq = tid == 0 ? p0 : p0 + n - 1;
        int64_t lo = 0, hi = nnzA;
        while (lo < hi) {
            const int64_t mid = (lo + hi + 1) >> 1;
            if (S[mid] <= pq) lo = mid;
            else hi = mid - 1;
        }
        if (tid == 0) s_j0 = lo;
        else s_j1 = lo;
    }
    __syncthreads();
    // ---- expansion: thread t expands products [t*VT, t*VT+VT) (blocked)
    {
        const int i0 = tid * RX_VT;
        if (i0 < n) {
            const int64_t p = p0 + i0;
            int64_t lo = s_j0, hi = s_j1;  // upper_bound(S, p) - 1 inside the tile's nonzeros
            while (lo < hi) {
                const int64_t mid = (lo + hi + 1) >> 1;
                if (S[mid] <= p) lo = mid;
                else hi = mid - 1;
            }
            int64_t j = lo, s_next = S[j + 1];
            int r = arow[j];
            int64_t bpos = int64_t(Brp[Acol[j]]) + (p - S[j]);
#pragma unroll
            for (int u = 0; u < RX_VT; ++u) {
                const int i = i0 + u;
                if (i < n) {
                    while (p0 + i >= s_next) {  // next A nonzero with products (Z7 skips empty B rows)
                        ++j;
                        s_next = S[j + 1];
                        r = arow[j];
                        bpos = Brp[Acol[j]] + (p0 + i - S[j]);
                    }
                    rows[i] = r;
                    ka[i] = (K(Bcol[bpos]) << RX_PB) | K(i);
                    va[i] = uint16_t(i);
                    ++bpos;
                }
            }
        }
    }
    __syncthreads();
    // ---- keys-only radix sort on the column bits only (one "pass" in the
    //      paper's sense: ceil(log2 n) bits, 4 at a time)
    K *kin = ka, *kout = kb;
    uint16_t *vin = va, *vout = vb;
    // (sort_bits > cb and row_bits > 0 only for the Fig 4 ablation: more key
    // bits sorted, and a second sort by row after the column sort)
    for (int sh = RX_PB; sh < RX_PB + sort_bits; sh += 4) {
        if (sh >= int(sizeof(K)) * 8) break;
        cta_pass4<RX_VT>(kin, vin, kout, vout, n, sh, cnt, wsum);
        K *t1 = kin; kin = kout; kout = t1;
        uint16_t *t2 = vin; vin = vout; vout = t2;
    }
    for (int sh = 0; sh < row_bits; sh += 4) {
        const int32_t *rw = rows;
        cta_pass4d<RX_VT>(kin, vin, kout, vout, n,
                          [&](K k) { return int((uint32_t(rw[int(k & ((K(1) << RX_PB) - 1))]) >> sh) & 15); }, cnt,
                          wsum);
        K *t1 = kin; kin = kout; kout = t1;
        uint16_t *t2 = vin; vin = vout; vout = t2;
    }
    // ---- duplicates are adjacent (same column, rows in expansion order)
    int hc = 0;
    uint32_t hbits = 0;
#pragma unroll
    for (int u = 0; u < RX_VT; ++u) {
        const int s = tid * RX_VT + u;
        bool h = false;
        if (s < n) {
            const int ix = int(kin[s] & ((K(1) << RX_PB) - 1));
            h = s == 0;
            if (!h) {
                const int ip = int(kin[s - 1] & ((K(1) << RX_PB) - 1));
                h = (kin[s] >> RX_PB) != (kin[s - 1] >> RX_PB) || rows[ix] != rows[ip];
            }
            perm[tile * RX_T + s] = uint16_t(ix);  // 16-bit permutation
        }
        hbits |= uint32_t(h) << u;
        hc += h;
    }
    // pack the head bits: 8 per thread -> 32-bit words of 4 threads
    {
        const unsigned w = __shfl_sync(0xffffffffu, hbits, (tid & 31) & ~3) |
                           (__shfl_sync(0xffffffffu, hbits, ((tid & 31) & ~3) + 1) << 8) |
                           (__shfl_sync(0xffffffffu, hbits, ((tid & 31) & ~3) + 2) << 16) |
                           (__shfl_sync(0xffffffffu, hbits, ((tid & 31) & ~3) + 3) << 24);
        if ((tid & 3) == 0) s_heads[tid >> 2] = w;
    }
    uint32_t tot;
    const uint32_t rank0 = block_exclusive_sum<uint32_t, RX_NT / 32>(uint32_t(hc), wsum, 1, &tot);
    if (tid < 32) {
        const int64_t base = tile_prefix(states, tile, int64_t(tot));
        if (tid == 0) {
            s_base = base;
            tcount[tile] = int32_t(tot);
            toff[tile] = base;
        }
    }
    for (int w = tid; w < RX_T / 32; w += RX_NT) heads[tile * (RX_T / 32) + w] = s_heads[w];
    __syncthreads();
    // reduced entries in the tile's (column) order
    int64_t o = s_base + rank0;
#pragma unroll
    for (int u = 0; u < RX_VT; ++u) {
        if ((hbits >> u) & 1u) {
            const int s = tid * RX_VT + u;
            const int ix = int(kin[s] & ((K(1) << RX_PB) - 1));
            red[o++] = (uint64_t(uint32_t(rows[ix])) << cb) | uint64_t(kin[s] >> RX_PB);
        }
    }
}

// ================================ phase 2 ==================================
// Global LSD radix sort of the reduced entries (packed keys) carrying their
// index: 8-bit digit passes.
__global__ void __launch_bounds__(RX_NT)
gx_hist_kernel(const uint64_t *__restrict__ keys, int64_t n, int shift, int64_t ntiles, int32_t *__restrict__ counts)
{
    __shared__ uint32_t h[256];
    const int tid = threadIdx.x;
    h[tid] = 0;
    __syncthreads();
    const int64_t base = int64_t(blockIdx.x) * GX_T;
    for (int u = 0; u < GX_VT; ++u) {
        const int64_t i = base + u * RX_NT + tid;
        if (i < n) atomicAdd(&h[(keys[i] >> shift) & 255], 1u);
    }
    __syncthreads();
    counts[int64_t(tid) * ntiles + blockIdx.x] = int32_t(h[tid]);  // digit-major: the scan gives global offsets
}

__global__ void __launch_bounds__(RX_NT)
gx_scatter_kernel(const uint64_t *__restrict__ keys, const uint32_t *__restrict__ vals, int64_t n, int shift,
                  int64_t ntiles, const int64_t *__restrict__ offs, uint64_t *__restrict__ okeys,
                  uint32_t *__restrict__ ovals)
{
    extern __shared__ __align__(16) char gx_smem[];
    uint64_t *k1 = reinterpret_cast<uint64_t *>(gx_smem);
    uint64_t *k2 = k1 + GX_T;
    uint32_t *v1 = reinterpret_cast<uint32_t *>(k2 + GX_T);
    uint32_t *v2 = v1 + GX_T;
    uint32_t *cnt = v2 + GX_T;  // [16][RX_NT]
    __shared__ uint32_t wsum[RX_NT / 32];
    __shared__ int32_t first[256];
    const int tid = threadIdx.x;
    const int64_t base = int64_t(blockIdx.x) * GX_T;
    const int nt = int(min(int64_t(GX_T), n - base));
    for (int i = tid; i < nt; i += RX_NT) {
        k1[i] = keys[base + i];
        v1[i] = vals[base + i];
    }
    __syncthreads();
    // stable in-tile ordering by the 8-bit digit: low nibble, then high nibble
    cta_pass4<GX_VT>(k1, v1, k2, v2, nt, shift, cnt, wsum);
    cta_pass4<GX_VT>(k2, v2, k1, v1, nt, shift + 4, cnt, wsum);
    // first position of every digit in the tile
    first[tid] = INT_MAX;
    __syncthreads();
    for (int i = tid; i < nt; i += RX_NT) {
        const int d = int((k1[i] >> shift) & 255);
        if (i == 0 || int((k1[i - 1] >> shift) & 255) != d) first[d] = i;
    }
    __syncthreads();
    for (int i = tid; i < nt; i += RX_NT) {
        const int d = int((k1[i] >> shift) & 255);
        const int64_t o = offs[int64_t(d) * ntiles + blockIdx.x] + (i - first[d]);
        okeys[o] = k1[i];
        ovals[o] = v1[i];
    }
}

__global__ void gx_iota_kernel(uint32_t *__restrict__ v, int64_t n)
{
    for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n; i += int64_t(gridDim.x) * blockDim.x)
        v[i] = uint32_t(i);
}

// sorted keys -> C structure: group heads, row counts, C.col, and the sorted
// position of every reduced entry (inverse permutation)
__global__ void gx_structure_kernel(const uint64_t *__restrict__ sk, const uint32_t *__restrict__ sv, int64_t n, int cb,
                                    int32_t *__restrict__ hflag, int32_t *__restrict__ Crow_counts,
                                    uint32_t *__restrict__ pos_of)
{
    for (int64_t s = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; s < n; s += int64_t(gridDim.x) * blockDim.x) {
        const bool h = s == 0 || sk[s] != sk[s - 1];
        hflag[s] = h;
        if (h && Crow_counts) atomicAdd(&Crow_counts[int32_t(sk[s] >> cb)], 1);
        pos_of[sv[s]] = uint32_t(s);
    }
}

__global__ void gx_cols_kernel(const uint64_t *__restrict__ sk, const int32_t *__restrict__ hflag,
                               const int64_t *__restrict__ grp, const int64_t *__restrict__ n_dev, int cb,
                               int32_t *__restrict__ Ccol)
{
    const int64_t n = *n_dev;
    const uint64_t cm = (uint64_t(1) << cb) - 1;
    for (int64_t s = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; s < n; s += int64_t(gridDim.x) * blockDim.x)
        if (hflag[s]) Ccol[grp[s]] = int32_t(sk[s] & cm);
}

// ================================ phase 3 ==================================
// Re-expansion with values, the tile's permutation, segmented reduction by
// the stored head flags, reduced values stored at their sorted positions.
template <typename V>
__global__ void __launch_bounds__(RX_NT)
rx_value_kernel(int64_t nprods, int64_t nnzA, const int32_t *__restrict__ Acol, const V *__restrict__ Aval,
                const int32_t *__restrict__ Brp, const V *__restrict__ Bval, const int64_t *__restrict__ S,
                const uint16_t *__restrict__ perm, const uint32_t *__restrict__ heads,
                const int64_t *__restrict__ toff, const uint32_t *__restrict__ pos_of, double *__restrict__ vbuf)
{
    __shared__ double prod[RX_T];
    __shared__ SegPair<double> wseg[RX_NT / 32];
    __shared__ uint32_t wsum[RX_NT / 32];
    __shared__ int64_t s_j0, s_j1;
    const int tid = threadIdx.x;
    const int64_t tile = blockIdx.x;
    const int64_t p0 = tile * RX_T;
    const int n = int(min(int64_t(RX_T), nprods - p0));
    if (tid < 2) {
        const int64_t pq = tid == 0 ? p0 : p0 + n - 1;
        int64_t lo = 0, hi = nnzA;
        while (lo < hi) {
            const int64_t mid = (lo + hi + 1) >> 1;
            if (S[mid] <= pq) lo = mid;
            else hi = mid - 1;
        }
        if (tid == 0) s_j0 = lo;
        else s_j1 = lo;
    }
    __syncthreads();
    {
        const int i0 = tid * RX_VT;
        if (i0 < n) {
            const int64_t p = p0 + i0;
            int64_t lo = s_j0, hi = s_j1;
            while (lo < hi) {
                const int64_t mid = (lo + hi + 1) >> 1;
                if (S[mid] <= p) lo = mid;
                else hi = mid - 1;
            }
            int64_t j = lo, s_next = S[j + 1];
            double a = double(Aval[j]);
            int64_t bpos = int64_t(Brp[Acol[j]]) + (p - S[j]);
#pragma unroll
            for (int u = 0; u < RX_VT; ++u) {
                const int i = i0 + u;
                if (i < n) {
                    while (p0 + i >= s_next) {
                        ++j;
                        s_next = S[j + 1];
                        a = double(Aval[j]);
                        bpos = Brp[Acol[j]] + (p0 + i - S[j]);
                    }
                    prod[i] = a * double(Bval[bpos]);
                    ++bpos;
                }
            }
        }
    }
    __syncthreads();
    // permuted products, segmented by the head flags (sorted order)
    const uint32_t hw = heads[tile * (RX_T / 32) + ((tid * RX_VT) >> 5)];
    const unsigned hb = (hw >> ((tid * RX_VT) & 31)) & 0xffu;
    double run = 0.0;
    int hc = 0;
    double seg_v[RX_VT];
#pragma unroll
    for (int u = 0; u < RX_VT; ++u) {
        const int s = tid * RX_VT + u;
        if ((hb >> u) & 1u) run = 0.0;
        if (s < n) run += prod[perm[tile * RX_T + s]];
        seg_v[u] = run;
        hc += (hb >> u) & 1u;
    }
    // the carry into this thread's first segment piece from earlier threads
    SegPair<double> stot;
    const SegPair<double> ex = block_seg_exclusive<double, RX_NT / 32>(SegPair<double>{int(hb != 0), run},
                                                                       SegPair<double>{0, 0.0}, wseg, 1, &stot);
    uint32_t tot;
    const uint32_t rank0 = block_exclusive_sum<uint32_t, RX_NT / 32>(uint32_t(hc), wsum, 2, &tot);
    // a segment ends at s if s is the tile's last product or s+1 is a head
    const uint32_t nw = (tid * RX_VT + RX_VT < RX_T) ? heads[tile * (RX_T / 32) + ((tid * RX_VT + RX_VT) >> 5)] : 0u;
    const unsigned nb = (tid * RX_VT + RX_VT < RX_T) ? ((nw >> ((tid * RX_VT + RX_VT) & 31)) & 1u) : 1u;
    int rank = int(rank0) - 1;  // index of the current segment within the tile
    bool seen = false;
#pragma unroll
    for (int u = 0; u < RX_VT; ++u) {
        const int s = tid * RX_VT + u;
        if ((hb >> u) & 1u) {
            ++rank;
            seen = true;
        }
        if (s < n) {
            const bool end = (s == n - 1) || (u < RX_VT - 1 ? ((hb >> (u + 1)) & 1u) : nb);
            if (end) {
                const double v = seen ? seg_v[u] : seg_v[u] + ex.v;  // piece started in an earlier thread
                const int64_t ridx = toff[tile] + rank;
                vbuf[pos_of[ridx]] = v;
            }
        }
    }
}

// reduce-by-key over the sorted positions: C value of each group
template <typename V>
__global__ void gx_reduce_kernel(const int32_t *__restrict__ hflag, const int64_t *__restrict__ grp,
                                 const double *__restrict__ vbuf, const int64_t *__restrict__ n_dev,
                                 V *__restrict__ Cval)
{
    const int64_t n = *n_dev;
    for (int64_t s = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; s < n; s += int64_t(gridDim.x) * blockDim.x) {
        if (!hflag[s]) continue;
        double v = vbuf[s];
        for (int64_t t = s + 1; t < n && !hflag[t]; ++t) v += vbuf[t];
        Cval[grp[s]] = V(v);
    }
}

struct RxWs {
    uint16_t *perm;
    uint32_t *heads;
    int32_t *tcount;
    int64_t *toff;
    uint64_t *states;
    uint64_t *red, *red2;     // reduced keys (packed), sort buffers
    uint32_t *rv, *rv2;       // reduced indices carried by the sort
    int32_t *counts;          // [256][gtiles]
    int64_t *offs;            // [256 * gtiles + 1]
    int32_t *hflag;           // [U]
    int64_t *grp;             // [U + 1] group index of every sorted position (scan of hflag)
    uint32_t *pos_of;         // [U]
    double *vbuf;             // [U]
    int64_t *total;           // [4]
    unsigned long long *ticket;
    void *scan;
    size_t scan_bytes;
    int64_t ntiles, ubound;
    size_t bytes;
};

RxWs carve_rx(int64_t nprods, int64_t m, void *ws, size_t cap, bool *ok)
{
    RxWs w;
    w.ntiles = ceil_div(nprods > 0 ? nprods : 1, RX_T);
    w.ubound = nprods > 0 ? nprods : 1;  // reduced entries <= products
    const int64_t gt = ceil_div(w.ubound, GX_T);
    Carve cv(ws, cap);
    w.states = cv.take<uint64_t>(size_t(w.ntiles));
    w.total = cv.take<int64_t>(4);
    w.ticket = cv.take<unsigned long long>(1);
    w.perm = cv.take<uint16_t>(size_t(w.ntiles) * RX_T);
    w.heads = cv.take<uint32_t>(size_t(w.ntiles) * (RX_T / 32));
    w.tcount = cv.take<int32_t>(size_t(w.ntiles));
    w.toff = cv.take<int64_t>(size_t(w.ntiles));
    w.red = cv.take<uint64_t>(size_t(w.ubound));
    w.red2 = cv.take<uint64_t>(size_t(w.ubound));
    w.rv = cv.take<uint32_t>(size_t(w.ubound));
    w.rv2 = cv.take<uint32_t>(size_t(w.ubound));
    w.counts = cv.take<int32_t>(size_t(256 * gt));
    w.offs = cv.take<int64_t>(size_t(256 * gt + 1));
    w.hflag = cv.take<int32_t>(size_t(w.ubound));
    w.grp = cv.take<int64_t>(size_t(w.ubound + 1));
    w.pos_of = cv.take<uint32_t>(size_t(w.ubound));
    w.vbuf = cv.take<double>(size_t(w.ubound));
    w.scan_bytes = scan_ws_bytes(std::max<int64_t>(std::max<int64_t>(256 * gt, w.ubound), std::max<int64_t>(m, 1)));
    w.scan = cv.take<char>(w.scan_bytes);
    w.bytes = cv.off;
    *ok = cv.ok();
    return w;
}

int bits_for(int64_t n)
{
    int b = 0;
    while ((int64_t(1) << b) < n) ++b;
    return b < 1 ? 1 : b;
}

// Phases 1 and 2 (symbolic).  The sorted keys end in red or red2 depending
// on the parity of the number of 8-bit passes (numeric recomputes which).
int rx_passes(const msp_csr *A, int cb) { return (bits_for(A->nrows) + cb + 7) / 8; }

template <typename Kern>
msp_status set_dyn_smem(Kern kern, int bytes, const char *what)
{
    return set_smem_attr(reinterpret_cast<const void *>(kern), bytes, what);
}

msp_status rx_sort(const msp_csr *A, const msp_csr *B, const int32_t *arow, const int64_t *S, const RxWs &w,
                   int64_t nprods, int cb, int64_t *U_host, uint64_t **sk, uint32_t **sv, cudaStream_t s)
{
    msp_status st = cuda_check(cudaMemsetAsync(w.states, 0, size_t(w.ntiles) * 8, s), "spgemm_radix: clear");
    if (st == MSP_OK) st = cuda_check(cudaMemsetAsync(w.ticket, 0, 8, s), "spgemm_radix: clear");
    if (st != MSP_OK) return st;
    const bool k32 = cb + RX_PB <= 32;
    // Fig 4 ablation knobs (tuning only): MSP_RX_SORT_BITS sorts that many key
    // bits instead of ceil(log2 n); MSP_RX_TWO_PASS=1 adds a sort by row
    static const int env_bits = getenv("MSP_RX_SORT_BITS") ? atoi(getenv("MSP_RX_SORT_BITS")) : 0;
    static const int env_two = getenv("MSP_RX_TWO_PASS") ? atoi(getenv("MSP_RX_TWO_PASS")) : 0;
    const int sort_bits = env_bits > cb ? env_bits : cb;
    const int row_bits = env_two ? bits_for(A->nrows) : 0;
    if (k32) {
        const int smem = RX_T * (2 * 4 + 2 * 2 + 4) + 16 * RX_NT * 4;
        st = set_dyn_smem(rx_tile_kernel<uint32_t>, smem, "spgemm_radix: tile smem");
        if (st != MSP_OK) return st;
        rx_tile_kernel<uint32_t><<<unsigned(w.ntiles), RX_NT, smem, s>>>(nprods, A->nnz, A->col_idx, B->row_offsets,
                                                                         B->col_idx, arow, S, cb, w.perm, w.heads,
                                                                         w.tcount, w.toff, w.states, w.red,
                                                                         w.ticket, sort_bits, row_bits);
    } else {
        const int smem = RX_T * (2 * 8 + 2 * 2 + 4) + 16 * RX_NT * 4;
        st = set_dyn_smem(rx_tile_kernel<uint64_t>, smem, "spgemm_radix: tile smem");
        if (st != MSP_OK) return st;
        rx_tile_kernel<uint64_t><<<unsigned(w.ntiles), RX_NT, smem, s>>>(nprods, A->nnz, A->col_idx, B->row_offsets,
                                                                         B->col_idx, arow, S, cb, w.perm, w.heads,
                                                                         w.tcount, w.toff, w.states, w.red,
                                                                         w.ticket, sort_bits, row_bits);
    }
    st = last_launch("rx_tile_kernel");
    if (st != MSP_OK) return st;
    // U = reduced entries (prefix of the last tile + its count); one read-back
    int64_t hv[2] = {0, 0};
    int64_t *pin = pinned_scratch();
    int64_t *h = pin ? pin : hv;
    st = cuda_check(cudaMemcpyAsync(&h[0], &w.toff[w.ntiles - 1], 8, cudaMemcpyDeviceToHost, s), "spgemm_radix: U");
    if (st == MSP_OK)
        st = cuda_check(cudaMemcpyAsync(&h[1], &w.tcount[w.ntiles - 1], 4, cudaMemcpyDeviceToHost, s),
                        "spgemm_radix: U");
    if (st == MSP_OK) st = cuda_check(cudaStreamSynchronize(s), "spgemm_radix: sync");
    if (st != MSP_OK) return st;
    const int64_t U = h[0] + int64_t(*reinterpret_cast<int32_t *>(&h[1]));
    *U_host = U;
    st = cuda_check(cudaMemcpyAsync(&w.total[1], &U, 8, cudaMemcpyHostToDevice, s), "spgemm_radix: U");
    if (st != MSP_OK) return st;
    // ---- global LSD radix sort of the reduced keys, carrying their index
    const int64_t gt = ceil_div(U, GX_T);
    gx_iota_kernel<<<unsigned(std::min<int64_t>(ceil_div(U, 256), 148 * 16)), 256, 0, s>>>(w.rv, U);
    st = last_launch("gx_iota_kernel");
    if (st != MSP_OK) return st;
    const int gsmem = GX_T * (2 * 8 + 2 * 4) + 16 * RX_NT * 4;
    st = set_dyn_smem(gx_scatter_kernel, gsmem, "spgemm_radix: scatter smem");
    if (st != MSP_OK) return st;
    uint64_t *ki = w.red, *ko = w.red2;
    uint32_t *vi = w.rv, *vo = w.rv2;
    const int passes = rx_passes(A, cb);
    for (int ps = 0; ps < passes; ++ps) {
        const int sh = 8 * ps;
        gx_hist_kernel<<<unsigned(gt), RX_NT, 0, s>>>(ki, U, sh, gt, w.counts);
        st = last_launch("gx_hist_kernel");
        if (st != MSP_OK) return st;
        st = scan_i32_to_i64(w.counts, w.offs, 256 * gt, w.scan, w.scan_bytes, s);
        if (st != MSP_OK) return st;
        gx_scatter_kernel<<<unsigned(gt), RX_NT, gsmem, s>>>(ki, vi, U, sh, gt, w.offs, ko, vo);
        st = last_launch("gx_scatter_kernel");
        if (st != MSP_OK) return st;
        std::swap(ki, ko);
        std::swap(vi, vo);
    }
    *sk = ki;
    *sv = vi;
    return MSP_OK;
}

}  // namespace

size_t spgemm_radix_ws_bytes(const msp_csr *A, const msp_csr *, int64_t nprods)
{
    bool ok;
    return carve_rx(nprods, A->nrows, nullptr, SIZE_MAX, &ok).bytes + 256;
}

msp_status spgemm_radix_symbolic_run(const msp_csr *A, const msp_csr *B, const void *ws1, size_t b1, void *ws,
                                     size_t bytes, int64_t nprods, int32_t *Crp, int64_t *nnzC, cudaStream_t s)
{
    bool ok;
    const RxWs w = carve_rx(nprods, A->nrows, ws, bytes, &ok);
    if (!ok) return MSP_ERR_WORKSPACE;
    const int32_t m = A->nrows;
    msp_status st = cuda_check(cudaMemsetAsync(Crp, 0, (size_t(m) + 1) * 4, s), "spgemm_radix: clear rp");
    if (st != MSP_OK) return st;
    if (m == 0 || nprods == 0) {
        *nnzC = 0;
        return cuda_check(cudaStreamSynchronize(s), "spgemm_radix: sync");
    }
    const int32_t *arow;
    const int64_t *S;
    st = spgemm_setup_arrays(A, ws1, b1, &arow, &S);
    if (st != MSP_OK) return st;
    const int cb = bits_for(B->ncols);
    int64_t U = 0;
    uint64_t *sk;
    uint32_t *sv;
    st = rx_sort(A, B, arow, S, w, nprods, cb, &U, &sk, &sv, s);
    if (st != MSP_OK) return st;
    const unsigned gb = unsigned(std::min<int64_t>(ceil_div(U, 256), 148 * 16));
    gx_structure_kernel<<<gb, 256, 0, s>>>(sk, sv, U, cb, w.hflag, Crp + 1, w.pos_of);
    st = last_launch("gx_structure_kernel");
    if (st != MSP_OK) return st;
    st = scan_i32_to_i64(w.hflag, w.grp, U, w.scan, w.scan_bytes, s);  // grp[s] = groups before sorted position s
    if (st != MSP_OK) return st;
    st = scan_counts_to_offsets_i32(Crp + 1, m, &w.total[0], w.scan, w.scan_bytes, s);
    if (st != MSP_OK) return st;
    int64_t hv = 0;
    int64_t *pin = pinned_scratch();
    int64_t *h = pin ? pin : &hv;
    st = cuda_check(cudaMemcpyAsync(h, &w.total[0], 8, cudaMemcpyDeviceToHost, s), "spgemm_radix: nnz");
    if (st == MSP_OK) st = cuda_check(cudaStreamSynchronize(s), "spgemm_radix: sync");
    if (st != MSP_OK) return st;
    *nnzC = *h;
    if (*nnzC > INT32_MAX) return MSP_ERR_OVERFLOW;
    return MSP_OK;
}

// Numeric: phase 3 on what symbolic left in ws (sorted keys, positions,
// groups, per-tile permutations and head flags).  Async.
msp_status spgemm_radix_numeric_run(const msp_csr *A, const msp_csr *B, const void *ws1, size_t b1, void *ws,
                                    size_t bytes, int64_t nprods, const int32_t *Crp, int32_t *Ccol, void *Cval,
                                    cudaStream_t s)
{
    (void)Crp;
    bool ok;
    const RxWs w = carve_rx(nprods, A->nrows, ws, bytes, &ok);
    if (!ok) return MSP_ERR_WORKSPACE;
    if (A->nrows == 0 || nprods == 0) return MSP_OK;
    const int32_t *arow;
    const int64_t *S;
    msp_status st = spgemm_setup_arrays(A, ws1, b1, &arow, &S);
    if (st != MSP_OK) return st;
    const int cb = bits_for(B->ncols);
    const uint64_t *sk = (rx_passes(A, cb) & 1) ? w.red2 : w.red;
    const unsigned gb = unsigned(std::min<int64_t>(ceil_div(w.ubound, 256), 148 * 16));
    gx_cols_kernel<<<gb, 256, 0, s>>>(sk, w.hflag, w.grp, &w.total[1], cb, Ccol);
    st = last_launch("gx_cols_kernel");
    if (st != MSP_OK) return st;
    if (A->dtype == MSP_F64)
        rx_value_kernel<double><<<unsigned(w.ntiles), RX_NT, 0, s>>>(
            nprods, A->nnz, A->col_idx, static_cast<const double *>(A->vals), B->row_offsets,
            static_cast<const double *>(B->vals), S, w.perm, w.heads, w.toff, w.pos_of, w.vbuf);
    else
        rx_value_kernel<float><<<unsigned(w.ntiles), RX_NT, 0, s>>>(
            nprods, A->nnz, A->col_idx, static_cast<const float *>(A->vals), B->row_offsets,
            static_cast<const float *>(B->vals), S, w.perm, w.heads, w.toff, w.pos_of, w.vbuf);
    st = last_launch("rx_value_kernel");
    if (st != MSP_OK) return st;
    if (A->dtype == MSP_F64)
        gx_reduce_kernel<double><<<gb, 256, 0, s>>>(w.hflag, w.grp, w.vbuf, &w.total[1], static_cast<double *>(Cval));
    else
        gx_reduce_kernel<float><<<gb, 256, 0, s>>>(w.hflag, w.grp, w.vbuf, &w.total[1], static_cast<float *>(Cval));
    return last_launch("gx_reduce_kernel");
}

}  // namespace msp
