// internal.h -- host-side declarations shared by the libmsp translation units.
#pragma once

#include <cstddef>
#include <cstdint>
#include <cuda_runtime.h>

#include "../../include/msp.h"

namespace msp {

// thread-local error text (api.cu)
void set_error(const char *fmt, ...);
void clear_error();

// device properties of the current device (cached)
int sm_count();
int64_t l2_bytes();  // L2 cache size of the current device

// returns MSP_OK or MSP_ERR_CUDA with the error text recorded
msp_status cuda_check(cudaError_t e, const char *where);
msp_status last_launch(const char *where);  // also counts the launch
uint64_t launch_count();
// 16 pinned int64 words per host thread (NULL if pinned allocation failed)
int64_t *pinned_scratch();
// cudaFuncAttributeMaxDynamicSharedMemorySize (and, with threads > 0, the
// max carveout + occupancy query) once per (device, kernel).
// fit_l1: then shrink the carveout to the occupancy's shared memory, the rest
// of the SM's unified 256 KB staying L1.
msp_status set_smem_attr(const void *func, int smem_bytes, const char *where, int threads = 0, int *occ = nullptr,
                         bool fit_l1 = false);

inline size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

// Simple bump allocator over a caller-provided workspace.
struct Carve {
    char *base;
    size_t cap, off;
    Carve(void *b, size_t c) : base(static_cast<char *>(b)), cap(c), off(0) {}
    template <typename T>
    T *take(size_t n, size_t align = 256)
    {
        off = align_up(off, align);
        T *p = reinterpret_cast<T *>(base ? base + off : nullptr);
        off += n * sizeof(T);
        return p;
    }
    bool ok() const { return off <= cap; }
};

inline size_t value_size(int32_t dt) { return dt == MSP_F64 ? 8 : 4; }

// ---------------------------------------------------------------- scan ---
// Device-wide exclusive scans (decoupled look-back, scan.cu).
size_t scan_ws_bytes(int64_t n);
// out[i] = sum_{k<i} in[k] for i in [0, n]  (n+1 outputs; out[n] = total).
msp_status scan_i32_to_i64(const int32_t *in, int64_t *out, int64_t n, void *ws, size_t ws_bytes,
                           cudaStream_t s);
msp_status scan_i64_to_i64(const int64_t *in, int64_t *out, int64_t n, void *ws, size_t ws_bytes, cudaStream_t s);
// In place: counts c[0..n) -> exclusive offsets with c_out[n] = total, int32
// result; *overflow_dev set to 1 if the total exceeds INT32_MAX.
msp_status scan_counts_to_offsets_i32(int32_t *counts, int64_t n, int64_t *total_dev, void *ws,
                                      size_t ws_bytes, cudaStream_t s);
// pos[i] = number of nonempty rows before row i, i in [0, m] (row compaction)
msp_status scan_nonempty_rows(const int32_t *rp, int64_t m, int64_t *pos, void *ws, size_t ws_bytes, cudaStream_t s);
// S[j] = sum_{k<j} (Brp[Acol[k]+1] - Brp[Acol[k]]), j in [0, nnzA] (SpGEMM setup)
msp_status scan_widths_to_S(const int32_t *Acol, const int32_t *Brp, int64_t nnzA, int64_t *S, void *ws,
                            size_t ws_bytes, cudaStream_t s);
// the same, also recording bstart[j] = Brp[Acol[j]] (the B row each A nonzero expands)
msp_status scan_widths_to_S_bstart(const int32_t *Acol, const int32_t *Brp, int64_t nnzA, int64_t *S, int32_t *bstart,
                                   void *ws, size_t ws_bytes, cudaStream_t s);

// ---------------------------------------------------------------- ops ----
size_t spmv_ws_bytes(const msp_csr *A);
msp_status spmv_run(const msp_csr *A, const void *x, void *y, void *ws, size_t ws_bytes, cudaStream_t s);
// warp-tile row-aligned SpMV (spmv_wt.cu), K odd in 15..31
msp_status spmv_wt_run(int K, const msp_csr *A, const void *x, void *y, void *ws, size_t ws_bytes, cudaStream_t s);

// the paper's own SpMV decomposition (nnz-only split + row compaction), f4
size_t spmv_nnz_ws_bytes(const msp_csr *A);
msp_status spmv_nnz_run(const msp_csr *A, const void *x, void *y, void *ws, size_t ws_bytes, cudaStream_t s);

size_t spadd_ws_bytes(const msp_csr *A, const msp_csr *B);
msp_status spadd_symbolic_run(const msp_csr *A, const msp_csr *B, int32_t *Crp, int64_t *nnzC, void *ws,
                              size_t ws_bytes, cudaStream_t s);
msp_status spadd_numeric_run(const msp_csr *A, const msp_csr *B, const int32_t *Crp, int32_t *Ccol, void *Cval,
                             void *ws, size_t ws_bytes, cudaStream_t s);
msp_status spadd_fused_run(const msp_csr *A, const msp_csr *B, int32_t *Crp, int32_t *Ccol, void *Cval, int64_t cap,
                           int64_t *nnzC, void *ws, size_t ws_bytes, cudaStream_t s);

size_t spgemm_setup_ws_bytes(const msp_csr *A, const msp_csr *B);
msp_status spgemm_setup_run(const msp_csr *A, const msp_csr *B, void *ws1, size_t b1, msp_spgemm_info *info,
                            cudaStream_t s);
msp_status spgemm_symbolic_run(const msp_csr *A, const msp_csr *B, const void *ws1, size_t b1, void *ws2,
                               size_t b2, msp_spgemm_info *info, int32_t *Crp, int64_t *nnzC, cudaStream_t s);
msp_status spgemm_numeric_run(const msp_csr *A, const msp_csr *B, const void *ws1, size_t b1, void *ws2,
                              size_t b2, const msp_spgemm_info *info, const int32_t *Crp, int32_t *Ccol, void *Cval,
                              cudaStream_t s);

// COO rows of A's nonzeros and the product prefix S (both in setup_ws)
msp_status spgemm_setup_arrays(const msp_csr *A, const void *ws1, size_t b1, const int32_t **arow, const int64_t **S);
// the paper's own SpGEMM sort pipeline (spgemm_radix.cu)
size_t spgemm_radix_ws_bytes(const msp_csr *A, const msp_csr *B, int64_t nprods);
msp_status spgemm_radix_symbolic_run(const msp_csr *A, const msp_csr *B, const void *ws1, size_t b1, void *ws,
                                     size_t bytes, int64_t nprods, int32_t *Crp, int64_t *nnzC, cudaStream_t s);
msp_status spgemm_radix_numeric_run(const msp_csr *A, const msp_csr *B, const void *ws1, size_t b1, void *ws,
                                    size_t bytes, int64_t nprods, const int32_t *Crp, int32_t *Ccol, void *Cval,
                                    cudaStream_t s);

msp_status csr_check_run(const msp_csr *A, int sorted_unique, int32_t *flags_host, void *ws, size_t ws_bytes,
                         cudaStream_t s);
size_t set_op_ws_bytes(int64_t na, int64_t nb);
msp_status set_op_run(int op, const void *A, const void *Av, int64_t na, const void *B, const void *Bv, int64_t nb,
                      int key_bytes, int val_bytes, void *C, void *Cv, int64_t cap, int64_t *nC_host, int64_t *nC_dev,
                      void *ws, size_t ws_bytes, cudaStream_t s);
msp_status gather_run(const void *src, const int32_t *idx, int64_t n, int value_bytes, void *dst, cudaStream_t s);
msp_status rebase_run(const int32_t *in, int32_t *out, int64_t n, int64_t base, cudaStream_t s);

}  // namespace msp
