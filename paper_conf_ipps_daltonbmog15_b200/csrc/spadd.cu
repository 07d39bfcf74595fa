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

constexpr int ADD_NT = 256;
constexpr int ADD_IPT = 8;
constexpr int ADD_T = ADD_NT * ADD_IPT;  // merge items per tile

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
                                       const int32_t *__restrict__ Bcol, int64_t ntiles, Split *__restrict__ splits)
{
    const int64_t E = nnzA + nnzB;
    const int64_t total = int64_t(m) + E;
    for (int64_t k = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; k <= ntiles; k += int64_t(gridDim.x) * blockDim.x) {
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

template <typename V, bool FILL>
struct AddSmem {
    int32_t acol[ADD_T + 2];
    int32_t bcol[ADD_T + 2];
    int32_t arp[ADD_T + 4];
    int32_t brp[ADD_T + 4];
    Split st[ADD_NT + 1];
    int32_t wsum[ADD_NT / 32];
};

template <typename V, bool FILL>
__global__ void __launch_bounds__(ADD_NT)
spadd_tile_kernel(int32_t m, const int32_t *__restrict__ Arp, const int32_t *__restrict__ Acol,
                  const V *__restrict__ Aval, const int32_t *__restrict__ Brp, const int32_t *__restrict__ Bcol,
                  const V *__restrict__ Bval, const Split *__restrict__ splits, int32_t *__restrict__ tile_count,
                  const int64_t *__restrict__ tile_off, int32_t *__restrict__ Crp_counts, int32_t *__restrict__ Ccol,
                  V *__restrict__ Cval)
{
    extern __shared__ __align__(16) char smem_raw[];
    AddSmem<V, FILL> &S = *reinterpret_cast<AddSmem<V, FILL> *>(smem_raw);
    const int tid = threadIdx.x;
    const int k = blockIdx.x;
    const Split s0 = splits[k], s1 = splits[k + 1];
    const int r0 = s0.r, r1 = s1.r;
    const int ga0 = s0.a, gb0 = s0.b;
    const int nA = s1.a - ga0, nB = s1.b - gb0;
    const int nrw = min(r1, m - 1) - r0 + 2;  // row offsets r0 .. min(r1, m-1)+1
    // ---- stage the tile (coalesced asynchronous copies, all in flight) ----
    for (int i = tid; i < nA; i += ADD_NT) cp_async<4>(&S.acol[i], Acol + ga0 + i);
    for (int i = tid; i < nB; i += ADD_NT) cp_async<4>(&S.bcol[i], Bcol + gb0 + i);
    for (int i = tid; i < nrw; i += ADD_NT) {
        cp_async<4>(&S.arp[i], Arp + r0 + i);
        cp_async<4>(&S.brp[i], Brp + r0 + i);
    }
    cp_async_wait_all();
    __syncthreads();
    for (int i = tid; i < nrw; i += ADD_NT) {  // tile-relative row offsets
        S.arp[i] -= ga0;
        S.brp[i] -= gb0;
    }
    __syncthreads();
    const int nrows = r1 - r0;  // row-end items in the tile
    const int items = nrows + nA + nB;
    auto a_lo = [&](int r) { return max(S.arp[r - r0], 0); };
    auto a_hi = [&](int r) { return min(S.arp[r - r0 + 1], nA); };
    auto b_lo = [&](int r) { return max(S.brp[r - r0], 0); };
    auto b_hi = [&](int r) { return min(S.brp[r - r0 + 1], nB); };
    auto acol = [&](int i) { return S.acol[i]; };
    auto bcol = [&](int i) { return S.bcol[i]; };
    // ---- this thread's split ----
    {
        const int dt = min(tid * ADD_IPT, items);
        int lo = max(0, dt - (nA + nB)), hi = min(dt, nrows);
        while (lo < hi) {
            const int mid = (lo + hi) >> 1;
            const int rend = min(S.arp[mid + 1], nA) + min(S.brp[mid + 1], nB);
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
            if (ia > al && ib < bh && S.acol[ia - 1] == S.bcol[ib]) ++ib;  // balanced path
            st.a = ia;
            st.b = ib;
        }
        S.st[tid] = st;
        if (tid == 0) S.st[ADD_NT] = Split{r1, nA, nB};
    }
    __syncthreads();
    const Split beg = S.st[tid], end = S.st[tid + 1];

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
            if (ra && (!rb || S.acol[ia] <= S.bcol[ib])) {
                if (rb && S.acol[ia] == S.bcol[ib]) {
                    on_out(S.acol[ia], ia, ib);
                    ++ia;
                    ++ib;
                } else {
                    on_out(S.acol[ia], ia, -1);
                    ++ia;
                }
            } else {
                on_out(S.bcol[ib], -1, ib);
                ++ib;
            }
        }
        return r;
    };

    if (!FILL) {
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
        if ((tid & 31) == 0) S.wsum[tid >> 5] = wsum;
        __syncthreads();
        if (tid == 0) {
            int t = 0;
            for (int w = 0; w < ADD_NT / 32; ++w) t += S.wsum[w];
            tile_count[k] = t;
        }
    } else {
        int cnt = 0;
        walk([&](int, int, int) { ++cnt; }, [&](int) {});
        int tot;
        const int off = block_exclusive_sum<int, ADD_NT / 32>(cnt, S.wsum, 0, &tot);
        // outputs of this thread are consecutive in C: store them directly
        // (values read from global at the matched positions, L1-resident)
        const int64_t base = tile_off[k] + off;
        int o = 0;
        walk(
            [&](int c, int ia, int ib) {
                V v;
                if (ia >= 0 && ib >= 0) v = Aval[ga0 + ia] + Bval[gb0 + ib];  // one rounding, A first
                else v = (ia >= 0) ? Aval[ga0 + ia] : Bval[gb0 + ib];
                Ccol[base + o] = c;
                Cval[base + o] = v;
                ++o;
            },
            [&](int) {});
        (void)tot;
    }
}

struct AddWs {
    Split *splits;
    int32_t *tile_count;
    int64_t *tile_off;  // [ntiles + 1]
    int64_t *totals;    // [4]
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
    w.scan_bytes = scan_ws_bytes(std::max<int64_t>(A->nrows, w.ntiles));
    w.scan = cv.take<char>(w.scan_bytes);
    w.bytes = cv.off;
    *ok = cv.ok();
    return w;
}

template <typename V, bool FILL>
msp_status launch_tiles(const msp_csr *A, const msp_csr *B, const AddWs &w, int32_t *Crp, int32_t *Ccol, void *Cval,
                        cudaStream_t s)
{
    auto kern = spadd_tile_kernel<V, FILL>;
    const int smem = int(sizeof(AddSmem<V, FILL>));
    static int configured = 0;
    if (!configured) {
        msp_status st = cuda_check(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem),
                                   "spadd: smem");
        if (st != MSP_OK) return st;
        configured = 1;
    }
    kern<<<unsigned(w.ntiles), ADD_NT, smem, s>>>(
        A->nrows, A->row_offsets, A->col_idx, static_cast<const V *>(A->vals), B->row_offsets, B->col_idx,
        static_cast<const V *>(B->vals), w.splits, w.tile_count, w.tile_off, Crp ? Crp + 1 : nullptr, Ccol,
        static_cast<V *>(Cval));
    return last_launch(FILL ? "spadd_tile_kernel<fill>" : "spadd_tile_kernel<count>");
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
    {
        const int64_t n = w.ntiles + 1;
        const unsigned blocks = unsigned(std::min<int64_t>(ceil_div(n, 256), 148 * 8));
        spadd_partition_kernel<<<blocks, 256, 0, s>>>(m, A->nnz, B->nnz, A->row_offsets, A->col_idx, B->row_offsets,
                                                      B->col_idx, w.ntiles, w.splits);
        st = last_launch("spadd_partition_kernel");
        if (st != MSP_OK) return st;
    }
    st = (A->dtype == MSP_F64) ? launch_tiles<double, false>(A, B, w, Crp, nullptr, nullptr, s)
                               : launch_tiles<float, false>(A, B, w, Crp, nullptr, nullptr, s);
    if (st != MSP_OK) return st;
    // row counts -> C.row_offsets (in place, Crp[0] stays 0); tile counts -> offsets
    st = scan_counts_to_offsets_i32(Crp + 1, m, &w.totals[0], w.scan, w.scan_bytes, s);
    if (st != MSP_OK) return st;
    st = scan_i32_to_i64(w.tile_count, w.tile_off, w.ntiles, w.scan, w.scan_bytes, s);
    if (st != MSP_OK) return st;
    int64_t h[2] = {0, 0};
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
    return (A->dtype == MSP_F64) ? launch_tiles<double, true>(A, B, w, nullptr, Ccol, Cval, s)
                                 : launch_tiles<float, true>(A, B, w, nullptr, Ccol, Cval, s);
}

}  // namespace msp
