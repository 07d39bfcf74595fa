// spmv_nnz.cu -- the paper's own SpMV decomposition as an ablation (SURVEY
// §8(f) f4(i)): a nonzero-only split with CSR row compaction, sm_100a.
//
// Paper: P:396-470 (Section III-A) and P:1326-1334 (Section IV-A):
//   * "assigning a fixed number of nonzeros, Nprods, per CTA";
//   * partition: "one binary search per CTA segment to locate the last
//     offset in the row offsets array processed by each CTA", stored in a
//     global buffer S;
//   * reduction: CTA i processes nonzeros [i*Nprods, min(|A|,(i+1)*Nprods))
//     (reading Z14: half-open), loads the row offsets S[i..i+1] into shared
//     memory, loads col/val "in strided order", gathers x, forms the products,
//     transposes them "from strided to blocked order using shared memory",
//     runs a CTA-wide segmented scan, stores row results to y and the CTA
//     remainder to a buffer r;
//   * update: a segmented scan of r adds each CTA's carry to the first row
//     of the next CTA (reading Z21: carries are (row, partial)
//     pairs, so a row spanning several CTAs sums all of them);
//   * empty rows: "compacts the CSR row offsets prior to performing each
//     SpMV": a scan over the nonempty-row flags gives the
//     compacted offsets and row ids; y is zero-filled, so empty rows read
//     +0.0 (Z6).
// Compared with the 2-D merge grid (spmv.cu / spmv_wt.cu) this split balances
// nonzeros only; a CTA whose range holds many short rows does more row work,
// and the compaction costs two extra passes over row_offsets.
#include <algorithm>
#include <climits>
#include <cstdint>

#include "common.cuh"
#include "internal.h"

namespace msp {
namespace {

constexpr int NZ_NT = 256;
constexpr int NZ_VT = 8;
constexpr int NZ_NP = NZ_NT * NZ_VT;  // nonzeros per CTA (the paper's Nprods)

struct NzCarry {
    int32_t row;  // original row id of the CTA's trailing partial (-1: none)
    int32_t pad;
    double val;
};

// compacted rows: crow[k] = k-th nonempty row, crp[k] = its first nonzero,
// crp[mc] = nnz
__global__ void nz_compact_kernel(int32_t m, int64_t nnz, const int32_t *__restrict__ rp,
                                  const int64_t *__restrict__ pos, int32_t *__restrict__ crow,
                                  int32_t *__restrict__ crp)
{
    for (int64_t r = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; r < m; r += int64_t(gridDim.x) * blockDim.x) {
        const int32_t a = rp[r], b = rp[r + 1];
        if (b > a) {
            const int64_t k = pos[r];
            crow[k] = int32_t(r);
            crp[k] = a;
        }
        if (r == m - 1) crp[pos[m]] = int32_t(nnz);
    }
}

// partition: S[i] = compacted row holding nonzero i*NP (the last row offset
// <= i*NP), one binary search per CTA segment
__global__ void nz_partition_kernel(int64_t G, int64_t nnz, const int32_t *__restrict__ crp,
                                    const int64_t *__restrict__ mc_dev, int32_t *__restrict__ S)
{
    const int64_t mc = *mc_dev;
    for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i <= G; i += int64_t(gridDim.x) * blockDim.x) {
        const int64_t j = i * NZ_NP < nnz ? i * NZ_NP : nnz;
        int64_t lo = 0, hi = mc;  // largest k in [0, mc) with crp[k] <= j  (j == nnz -> mc - 1 at most)
        while (hi - lo > 1) {
            const int64_t mid = (lo + hi) >> 1;
            if (crp[mid] <= j) lo = mid;
            else hi = mid;
        }
        S[i] = int32_t(lo);
    }
}

template <typename V>
__global__ void __launch_bounds__(NZ_NT)
nz_reduce_kernel(int64_t nnz, const int32_t *__restrict__ crp, const int32_t *__restrict__ crow,
                 const int32_t *__restrict__ col, const V *__restrict__ val, const V *__restrict__ x,
                 V *__restrict__ y, const int32_t *__restrict__ S, NzCarry *__restrict__ carries)
{
    __shared__ double prod[NZ_NP];
    __shared__ int32_t rowend[NZ_NP];  // compacted row + 1 ending at this position, 0 if none
    __shared__ SegPair<double> wsum[NZ_NT / 32];
    const int tid = threadIdx.x;
    const int64_t i = blockIdx.x;
    const int64_t j0 = i * NZ_NP;
    const int n = int(min(int64_t(NZ_NP), nnz - j0));
    const int k0 = S[i], k1 = S[i + 1];
    for (int p = tid; p < NZ_NP; p += NZ_NT) rowend[p] = 0;
    __syncthreads();
    // row ends of the CTA's rows (offsets S[i..i+1])
    for (int k = k0 + tid; k <= k1; k += NZ_NT) {
        const int64_t e = int64_t(crp[k + 1]) - j0 - 1;  // last nonzero of row k, CTA-relative
        if (e >= 0 && e < n) rowend[e] = k + 1;
    }
    // strided (coalesced) loads, x gathers, products -> blocked order in smem
#pragma unroll
    for (int u = 0; u < NZ_VT; ++u) {
        const int p = u * NZ_NT + tid;
        double v = 0.0;
        if (p < n) v = double(val[j0 + p]) * double(__ldg(x + col[j0 + p]));
        prod[p] = v;
    }
    __syncthreads();
    // thread-serial segmented sum over its blocked positions
    double run = 0.0, first_v = 0.0;
    int first_k = -1;
#pragma unroll
    for (int u = 0; u < NZ_VT; ++u) {
        const int p = tid * NZ_VT + u;
        run += prod[p];
        const int re = rowend[p];
        if (re) {
            if (first_k < 0) {
                first_k = re - 1;
                first_v = run;
            } else {
                y[crow[re - 1]] = V(run);
            }
            run = 0.0;
        }
    }
    // CTA-wide segmented scan: carry into each thread's first row
    SegPair<double> tot;
    const SegPair<double> ex =
        block_seg_exclusive<double, NZ_NT / 32>(SegPair<double>{first_k >= 0, run}, SegPair<double>{0, 0.0}, wsum, 1,
                                                &tot);
    if (first_k >= 0) y[crow[first_k]] = V(first_v + ex.v);  // the CTA's first row: update adds the carry
    if (tid == NZ_NT - 1) {
        // the remainder after the CTA's last row end
        const bool open = rowend[n - 1] == 0;
        NzCarry c;
        c.row = open ? crow[k1] : -1;
        c.pad = 0;
        c.val = open ? tot.v : 0.0;
        carries[i] = c;
    }
}

// update: a run of CTAs carrying the same row adds, in CTA
// order, to the value the CTA that ends the row wrote for it
template <typename V>
__global__ void nz_update_kernel(int64_t G, const NzCarry *__restrict__ carries, V *__restrict__ y)
{
    for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < G; i += int64_t(gridDim.x) * blockDim.x) {
        const int32_t row = carries[i].row;
        if (row < 0 || (i > 0 && carries[i - 1].row == row)) continue;  // not the head of a run
        double s = 0.0;
        int64_t k = i;
        while (k < G && carries[k].row == row) s += carries[k++].val;
        // the row's stored part plus the carries: two roundings for a row
        // spanning CTAs (the paper's update; within the BJ:5 tolerance, and
        // exact in integer mode)
        y[row] = V(double(y[row]) + s);
    }
}

struct NzWs {
    int64_t *pos;
    int32_t *crow, *crp, *S;
    NzCarry *carries;
    void *scan;
    size_t scan_bytes;
    int64_t G;
    size_t bytes;
};

NzWs carve_nz(const msp_csr *A, void *ws, size_t cap, bool *ok)
{
    NzWs w;
    const int64_t m = A->nrows;
    w.G = ceil_div(A->nnz > 0 ? A->nnz : 1, NZ_NP);
    Carve cv(ws, cap);
    w.pos = cv.take<int64_t>(size_t(m + 1));
    w.crow = cv.take<int32_t>(size_t(m > 0 ? m : 1));
    w.crp = cv.take<int32_t>(size_t(m + 1));
    w.S = cv.take<int32_t>(size_t(w.G + 1));
    w.carries = cv.take<NzCarry>(size_t(w.G));
    w.scan_bytes = scan_ws_bytes(m > 0 ? m : 1);
    w.scan = cv.take<char>(w.scan_bytes);
    w.bytes = cv.off;
    *ok = cv.ok();
    return w;
}

template <typename V>
msp_status run_nz(const msp_csr *A, const void *x, void *y, const NzWs &w, cudaStream_t s)
{
    const int32_t m = A->nrows;
    const int64_t nnz = A->nnz;
    msp_status st = cuda_check(cudaMemsetAsync(y, 0, size_t(m) * sizeof(V), s), "spmv_nnz: zero y");
    if (st != MSP_OK || nnz == 0) return st;
    // compaction
    st = scan_nonempty_rows(A->row_offsets, m, w.pos, w.scan, w.scan_bytes, s);
    if (st != MSP_OK) return st;
    const unsigned cb = unsigned(std::min<int64_t>(ceil_div(m, 256), 148 * 16));
    nz_compact_kernel<<<cb, 256, 0, s>>>(m, nnz, A->row_offsets, w.pos, w.crow, w.crp);
    st = last_launch("nz_compact_kernel");
    if (st != MSP_OK) return st;
    // partition
    nz_partition_kernel<<<unsigned(std::min<int64_t>(ceil_div(w.G + 1, 256), 148 * 8)), 256, 0, s>>>(
        w.G, nnz, w.crp, w.pos + m, w.S);
    st = last_launch("nz_partition_kernel");
    if (st != MSP_OK) return st;
    // reduction
    nz_reduce_kernel<V><<<unsigned(w.G), NZ_NT, 0, s>>>(nnz, w.crp, w.crow, A->col_idx,
                                                        static_cast<const V *>(A->vals), static_cast<const V *>(x),
                                                        static_cast<V *>(y), w.S, w.carries);
    st = last_launch("nz_reduce_kernel");
    if (st != MSP_OK) return st;
    // update
    nz_update_kernel<V><<<unsigned(std::min<int64_t>(ceil_div(w.G, 256), 148 * 4)), 256, 0, s>>>(
        w.G, w.carries, static_cast<V *>(y));
    return last_launch("nz_update_kernel");
}

}  // namespace

size_t spmv_nnz_ws_bytes(const msp_csr *A)
{
    bool ok;
    return carve_nz(A, nullptr, SIZE_MAX, &ok).bytes + 256;
}

msp_status spmv_nnz_run(const msp_csr *A, const void *x, void *y, void *ws, size_t ws_bytes, cudaStream_t s)
{
    bool ok;
    const NzWs w = carve_nz(A, ws, ws_bytes, &ok);
    if (!ok) return MSP_ERR_WORKSPACE;
    if (A->nrows == 0) return MSP_OK;
    return A->dtype == MSP_F64 ? run_nz<double>(A, x, y, w, s) : run_nz<float>(A, x, y, w, s);
}

}  // namespace msp
