// check.cu -- CSR input validation (the CSR contract of P:316-322 and the
// "sorted by row and row-wise internally sorted by column" precondition of
// the union formulation) and a row-offset rebase helper used for
// multi-GPU row-block views.
#include <algorithm>

#include "common.cuh"
#include "internal.h"

namespace msp {
namespace {

__global__ void csr_check_kernel(int32_t m, int32_t ncols, int64_t nnz, const int32_t *__restrict__ rp,
                                 const int32_t *__restrict__ col, int sorted_unique, int32_t *flags)
{
    const int lane = threadIdx.x & 31;
    const int64_t warp = (int64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = (int64_t(gridDim.x) * blockDim.x) >> 5;
    int f = 0;
    if (warp == 0 && lane == 0) {
        if (rp[0] != 0 || int64_t(rp[m]) != nnz) f |= 1;
    }
    for (int64_t r = warp; r < m; r += nwarps) {
        const int32_t a = rp[r], b = rp[r + 1];
        // a malformed row is flagged and skipped before col is touched, so the
        // validator never reads outside col[0, nnz) on the input it rejects
        if (a < 0 || b < a || int64_t(b) > nnz) {
            f |= 1;
            continue;
        }
        for (int64_t j = a + lane; j < b; j += 32) {
            const int32_t c = col[j];
            if (c < 0 || c >= ncols) f |= 2;
            if (sorted_unique && j + 1 < b && col[j + 1] <= c) f |= 4;
        }
    }
    f = __reduce_or_sync(0xffffffffu, f);
    if (lane == 0 && f) atomicOr(flags, f);
}

__global__ void rebase_kernel(const int32_t *__restrict__ in, int32_t *__restrict__ out, int64_t n, int64_t base)
{
    const int32_t first = in[0];
    for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n; i += int64_t(gridDim.x) * blockDim.x)
        out[i] = int32_t(int64_t(in[i]) - first + base);
}

}  // namespace

msp_status csr_check_run(const msp_csr *A, int sorted_unique, int32_t *flags_host, void *ws, size_t ws_bytes,
                         cudaStream_t s)
{
    if (ws_bytes < 16) return MSP_ERR_WORKSPACE;
    int32_t *flags = static_cast<int32_t *>(ws);
    msp_status st = cuda_check(cudaMemsetAsync(flags, 0, sizeof(int32_t), s), "csr_check: clear");
    if (st != MSP_OK) return st;
    const int threads = 256;
    int64_t blocks = ceil_div(int64_t(A->nrows) * 32, threads);
    if (blocks < 1) blocks = 1;
    if (blocks > 4 * 148 * 8) blocks = 4 * 148 * 8;
    csr_check_kernel<<<unsigned(blocks), threads, 0, s>>>(A->nrows, A->ncols, A->nnz, A->row_offsets, A->col_idx,
                                                          sorted_unique, flags);
    st = last_launch("csr_check_kernel");
    if (st != MSP_OK) return st;
    int32_t h = 0;
    st = cuda_check(cudaMemcpyAsync(&h, flags, sizeof(int32_t), cudaMemcpyDeviceToHost, s), "csr_check: copy");
    if (st != MSP_OK) return st;
    st = cuda_check(cudaStreamSynchronize(s), "csr_check: sync");
    if (st != MSP_OK) return st;
    if (flags_host) *flags_host = h;
    return h ? MSP_ERR_INPUT : MSP_OK;
}

msp_status rebase_run(const int32_t *in, int32_t *out, int64_t n, int64_t base, cudaStream_t s)
{
    if (n <= 0) return MSP_OK;
    int64_t blocks = ceil_div(n, 256);
    if (blocks > 148 * 16) blocks = 148 * 16;
    rebase_kernel<<<unsigned(blocks), 256, 0, s>>>(in, out, n, base);
    return last_launch("rebase_kernel");
}

}  // namespace msp

// ---------------------------------------------------------------- gather
namespace msp {
namespace {

template <typename T>
__global__ void gather_kernel(const T *__restrict__ src, const int32_t *__restrict__ idx, int64_t n,
                              T *__restrict__ dst)
{
    for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n; i += int64_t(gridDim.x) * blockDim.x)
        dst[i] = src[idx[i]];
}

}  // namespace

msp_status gather_run(const void *src, const int32_t *idx, int64_t n, int value_bytes, void *dst, cudaStream_t s)
{
    if (n <= 0) return MSP_OK;
    const unsigned blocks = unsigned(std::min<int64_t>(ceil_div(n, 256), 148 * 16));
    if (value_bytes == 8)
        gather_kernel<uint64_t><<<blocks, 256, 0, s>>>(static_cast<const uint64_t *>(src), idx, n,
                                                       static_cast<uint64_t *>(dst));
    else
        gather_kernel<uint32_t><<<blocks, 256, 0, s>>>(static_cast<const uint32_t *>(src), idx, n,
                                                       static_cast<uint32_t *>(dst));
    return last_launch("gather_kernel");
}

}  // namespace msp
