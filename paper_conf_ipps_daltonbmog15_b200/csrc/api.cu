// api.cu -- the extern "C" boundary of libmsp (include/msp.h).
//
// Host-side argument, shape and dtype validation happens here, before any
// launch; the kernels live in spmv.cu / spadd.cu / spgemm.cu / scan.cu /
// check.cu.  No call allocates device memory: every buffer is the caller's.
#include <cstdarg>
#include <cstdlib>
#include <cstdio>
#include <cstring>
#include <atomic>
#include <mutex>

#include "internal.h"

namespace msp {

static thread_local char g_err[512] = "";

void set_error(const char *fmt, ...)
{
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(g_err, sizeof(g_err), fmt, ap);
    va_end(ap);
}

void clear_error() { g_err[0] = 0; }

msp_status cuda_check(cudaError_t e, const char *where)
{
    if (e == cudaSuccess) return MSP_OK;
    set_error("%s: %s (%s)", where, cudaGetErrorString(e), cudaGetErrorName(e));
    return MSP_ERR_CUDA;
}

static std::atomic<uint64_t> g_launches{0};

msp_status last_launch(const char *where)
{
    g_launches.fetch_add(1, std::memory_order_relaxed);
    return cuda_check(cudaGetLastError(), where);
}

uint64_t launch_count() { return g_launches.load(std::memory_order_relaxed); }

int sm_count()
{
    static int cache[64] = {0};
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) return 148;
    if (dev < 0 || dev >= 64) return 148;
    if (!cache[dev]) {
        int n = 0;
        if (cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || n <= 0) n = 148;
        cache[dev] = n;
    }
    return cache[dev];
}

int64_t l2_bytes()
{
    static int64_t cache[64] = {0};
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return int64_t(126) << 20;
    if (!cache[dev]) {
        int n = 0;
        if (cudaDeviceGetAttribute(&n, cudaDevAttrL2CacheSize, dev) != cudaSuccess || n <= 0) n = 126 << 20;
        cache[dev] = n;
    }
    return cache[dev];
}

// Pinned host words per host thread for the synchronising size read-backs
// (a pageable destination would stage each small copy through a driver
// buffer).  Never freed: one small allocation per host thread.
int64_t *pinned_scratch()
{
    static thread_local int64_t *p = nullptr;
    if (!p && cudaMallocHost(reinterpret_cast<void **>(&p), 16 * sizeof(int64_t)) != cudaSuccess) p = nullptr;
    return p;
}

// Large-shared-memory opt-in, once per (device, kernel): the attribute is a
// per-device property, so a process driving several GPUs sets it on each.
// Returns the occupancy (resident CTAs per SM) when `threads` > 0.
msp_status set_smem_attr(const void *func, int smem_bytes, const char *where, int threads, int *occ, bool fit_l1)
{
    struct Entry {
        int dev;
        const void *func;
        int occ;
    };
    static std::mutex mu;
    static Entry table[1024];
    static int n = 0;
    int dev = 0;
    msp_status st = cuda_check(cudaGetDevice(&dev), where);
    if (st != MSP_OK) return st;
    std::lock_guard<std::mutex> lk(mu);
    for (int i = 0; i < n; ++i)
        if (table[i].dev == dev && table[i].func == func) {
            if (occ) *occ = table[i].occ;
            return MSP_OK;
        }
    st = cuda_check(cudaFuncSetAttribute(func, cudaFuncAttributeMaxDynamicSharedMemorySize, smem_bytes), where);
    if (st != MSP_OK) return st;
    int o = 1;
    if (threads > 0) {
        st = cuda_check(cudaFuncSetAttribute(func, cudaFuncAttributePreferredSharedMemoryCarveout, 100), where);
        if (st != MSP_OK) return st;
        st = cuda_check(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o, func, threads, size_t(smem_bytes)), where);
        if (st != MSP_OK) return st;
        if (o < 1) o = 1;
        if (fit_l1) {
            // shrink the carveout to what `o` CTAs need (+1 KB reserved per
            // CTA): the rest of the SM's 256 KB stays L1, whose lines also
            // hold the in-flight misses of the gathers
            int max_smem = 0;
            if (cudaDeviceGetAttribute(&max_smem, cudaDevAttrMaxSharedMemoryPerMultiprocessor, dev) != cudaSuccess ||
                max_smem <= 0)
                max_smem = 228 * 1024;
            const int64_t need = int64_t(o) * (smem_bytes + 1024);
            int pct = int((need * 100 + max_smem - 1) / max_smem);
            if (pct < 100) {
                st = cuda_check(cudaFuncSetAttribute(func, cudaFuncAttributePreferredSharedMemoryCarveout, pct), where);
                if (st != MSP_OK) return st;
                int o2 = 0;
                st = cuda_check(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o2, func, threads, size_t(smem_bytes)),
                                where);
                if (st != MSP_OK) return st;
                if (o2 < o) {  // the driver's carveout steps did not fit: keep the full carveout
                    st = cuda_check(cudaFuncSetAttribute(func, cudaFuncAttributePreferredSharedMemoryCarveout, 100),
                                    where);
                    if (st != MSP_OK) return st;
                }
            }
        }
    }
    if (n < 1024) table[n++] = Entry{dev, func, o};
    if (occ) *occ = o;
    return MSP_OK;
}

}  // namespace msp

using namespace msp;

namespace {

msp_status check_csr(const msp_csr *A, const char *name)
{
    if (!A) {
        set_error("%s is NULL", name);
        return MSP_ERR_ARG;
    }
    if (A->nrows < 0 || A->ncols < 0 || A->nnz < 0) {
        set_error("%s: negative size", name);
        return MSP_ERR_ARG;
    }
    if (A->nnz > INT32_MAX) {
        set_error("%s: nnz exceeds int32 indices", name);
        return MSP_ERR_OVERFLOW;
    }
    if (A->dtype != MSP_F32 && A->dtype != MSP_F64) {
        set_error("%s: dtype %d not supported", name, int(A->dtype));
        return MSP_ERR_DTYPE;
    }
    if (!A->row_offsets || (A->nnz > 0 && (!A->col_idx || !A->vals))) {
        set_error("%s: NULL array", name);
        return MSP_ERR_ARG;
    }
    return MSP_OK;
}

inline cudaStream_t as_stream(void *s) { return static_cast<cudaStream_t>(s); }

// Every *_workspace size carries kValidateBytes of tail room for the
// MSP_DEBUG_VALIDATE input check (a flag word; the library never allocates).
constexpr size_t kValidateBytes = 512;

bool debug_validate_on()
{
    static int v = -1;
    if (v < 0) {
        const char *e = getenv("MSP_DEBUG_VALIDATE");
        v = (e && *e && atoi(e) != 0) ? 1 : 0;
    }
    return v != 0;
}

// With MSP_DEBUG_VALIDATE=1 in the environment, the entry points run
// msp_csr_check on their inputs first (synchronising) and return
// MSP_ERR_INPUT on a malformed matrix instead of computing on it.
msp_status debug_validate(const msp_csr *A, int sorted_unique, void *ws, size_t ws_bytes, size_t used, cudaStream_t s,
                          const char *what)
{
    if (!debug_validate_on()) return MSP_OK;
    const size_t off = align_up(used, 256);
    if (off + 16 > ws_bytes) return MSP_ERR_WORKSPACE;
    int32_t flags = 0;
    msp_status st = csr_check_run(A, sorted_unique, &flags, static_cast<char *>(ws) + off, 16, s);
    if (st == MSP_ERR_INPUT) set_error("%s: MSP_DEBUG_VALIDATE: malformed CSR (flags %d)", what, flags);
    return st;
}

}  // namespace

extern "C" {

const char *msp_status_string(int status)
{
    switch (status) {
    case MSP_OK: return "MSP_OK";
    case MSP_ERR_ARG: return "MSP_ERR_ARG";
    case MSP_ERR_DTYPE: return "MSP_ERR_DTYPE";
    case MSP_ERR_SHAPE: return "MSP_ERR_SHAPE";
    case MSP_ERR_WORKSPACE: return "MSP_ERR_WORKSPACE";
    case MSP_ERR_OVERFLOW: return "MSP_ERR_OVERFLOW";
    case MSP_ERR_INPUT: return "MSP_ERR_INPUT";
    case MSP_ERR_CUDA: return "MSP_ERR_CUDA";
    case MSP_ERR_NCCL: return "MSP_ERR_NCCL";
    case MSP_ERR_UNSUPPORTED: return "MSP_ERR_UNSUPPORTED";
    default: return "MSP_ERR_UNKNOWN";
    }
}

const char *msp_last_error(void) { return g_err; }

int msp_version(void) { return MSP_VERSION; }

uint64_t msp_launch_count(void) { return launch_count(); }

// ------------------------------------------------------------------ SpMV
msp_status msp_spmv_workspace(const msp_csr *A, size_t *bytes)
{
    clear_error();
    msp_status st = check_csr(A, "A");
    if (st != MSP_OK) return st;
    if (!bytes) return MSP_ERR_ARG;
    *bytes = spmv_ws_bytes(A) + kValidateBytes;
    return MSP_OK;
}

msp_status msp_spmv(const msp_csr *A, const void *x, void *y, void *ws, size_t ws_bytes, void *stream)
{
    clear_error();
    msp_status st = check_csr(A, "A");
    if (st != MSP_OK) return st;
    if ((A->ncols > 0 && !x) || (A->nrows > 0 && !y) || !ws) {
        set_error("spmv: NULL x, y or workspace");
        return MSP_ERR_ARG;
    }
    if (ws_bytes < spmv_ws_bytes(A)) {
        set_error("spmv: workspace %zu < %zu bytes", ws_bytes, spmv_ws_bytes(A));
        return MSP_ERR_WORKSPACE;
    }
    st = debug_validate(A, 0, ws, ws_bytes, spmv_ws_bytes(A), as_stream(stream), "spmv A");
    if (st != MSP_OK) return st;
    return spmv_run(A, x, y, ws, ws_bytes, as_stream(stream));
}

msp_status msp_spmv_nnz_split_workspace(const msp_csr *A, size_t *bytes)
{
    clear_error();
    msp_status st = check_csr(A, "A");
    if (st != MSP_OK) return st;
    if (!bytes) return MSP_ERR_ARG;
    *bytes = spmv_nnz_ws_bytes(A) + kValidateBytes;
    return MSP_OK;
}

msp_status msp_spmv_nnz_split(const msp_csr *A, const void *x, void *y, void *ws, size_t ws_bytes, void *stream)
{
    clear_error();
    msp_status st = check_csr(A, "A");
    if (st != MSP_OK) return st;
    if ((A->ncols > 0 && !x) || (A->nrows > 0 && !y) || !ws) {
        set_error("spmv_nnz_split: NULL x, y or workspace");
        return MSP_ERR_ARG;
    }
    if (ws_bytes < spmv_nnz_ws_bytes(A)) {
        set_error("spmv_nnz_split: workspace %zu < %zu bytes", ws_bytes, spmv_nnz_ws_bytes(A));
        return MSP_ERR_WORKSPACE;
    }
    st = debug_validate(A, 0, ws, ws_bytes, spmv_nnz_ws_bytes(A), as_stream(stream), "spmv_nnz_split A");
    if (st != MSP_OK) return st;
    return spmv_nnz_run(A, x, y, ws, ws_bytes, as_stream(stream));
}

// ------------------------------------------------------------------ SpAdd
static msp_status check_pair_add(const msp_csr *A, const msp_csr *B)
{
    msp_status st = check_csr(A, "A");
    if (st == MSP_OK) st = check_csr(B, "B");
    if (st != MSP_OK) return st;
    if (A->nrows != B->nrows || A->ncols != B->ncols) {
        set_error("spadd: shapes %dx%d and %dx%d differ", A->nrows, A->ncols, B->nrows, B->ncols);
        return MSP_ERR_SHAPE;
    }
    if (A->dtype != B->dtype) {
        set_error("spadd: dtypes differ");
        return MSP_ERR_DTYPE;
    }
    return MSP_OK;
}

msp_status msp_spadd_workspace(const msp_csr *A, const msp_csr *B, size_t *bytes)
{
    clear_error();
    msp_status st = check_pair_add(A, B);
    if (st != MSP_OK) return st;
    if (!bytes) return MSP_ERR_ARG;
    *bytes = spadd_ws_bytes(A, B) + kValidateBytes;
    return MSP_OK;
}

msp_status msp_spadd_symbolic(const msp_csr *A, const msp_csr *B, int32_t *C_row_offsets, int64_t *nnzC_host,
                              void *ws, size_t ws_bytes, void *stream)
{
    clear_error();
    msp_status st = check_pair_add(A, B);
    if (st != MSP_OK) return st;
    if (!C_row_offsets || !nnzC_host || !ws) return MSP_ERR_ARG;
    if (ws_bytes < spadd_ws_bytes(A, B)) return MSP_ERR_WORKSPACE;
    st = debug_validate(A, 1, ws, ws_bytes, spadd_ws_bytes(A, B), as_stream(stream), "spadd A");
    if (st == MSP_OK) st = debug_validate(B, 1, ws, ws_bytes, spadd_ws_bytes(A, B), as_stream(stream), "spadd B");
    if (st != MSP_OK) return st;
    return spadd_symbolic_run(A, B, C_row_offsets, nnzC_host, ws, ws_bytes, as_stream(stream));
}

msp_status msp_spadd_numeric(const msp_csr *A, const msp_csr *B, const int32_t *C_row_offsets, int32_t *C_col_idx,
                             void *C_vals, void *ws, size_t ws_bytes, void *stream)
{
    clear_error();
    msp_status st = check_pair_add(A, B);
    if (st != MSP_OK) return st;
    if (!C_row_offsets || !ws) return MSP_ERR_ARG;
    if (ws_bytes < spadd_ws_bytes(A, B)) return MSP_ERR_WORKSPACE;
    return spadd_numeric_run(A, B, C_row_offsets, C_col_idx, C_vals, ws, ws_bytes, as_stream(stream));
}

msp_status msp_spadd_fused(const msp_csr *A, const msp_csr *B, int32_t *C_row_offsets, int32_t *C_col_idx,
                           void *C_vals, int64_t C_capacity, int64_t *nnzC_host, void *ws, size_t ws_bytes,
                           void *stream)
{
    clear_error();
    msp_status st = check_pair_add(A, B);
    if (st != MSP_OK) return st;
    if (!C_row_offsets || !nnzC_host || !ws) return MSP_ERR_ARG;
    if (C_capacity < A->nnz + B->nnz) {
        set_error("spadd fused: C capacity %lld below nnz(A) + nnz(B) = %lld", (long long)C_capacity,
                  (long long)(A->nnz + B->nnz));
        return MSP_ERR_SHAPE;
    }
    if (C_capacity > 0 && (!C_col_idx || !C_vals)) return MSP_ERR_ARG;
    if (ws_bytes < spadd_ws_bytes(A, B)) return MSP_ERR_WORKSPACE;
    st = debug_validate(A, 1, ws, ws_bytes, spadd_ws_bytes(A, B), as_stream(stream), "spadd A");
    if (st == MSP_OK) st = debug_validate(B, 1, ws, ws_bytes, spadd_ws_bytes(A, B), as_stream(stream), "spadd B");
    if (st != MSP_OK) return st;
    return spadd_fused_run(A, B, C_row_offsets, C_col_idx, C_vals, C_capacity, nnzC_host, ws, ws_bytes,
                           as_stream(stream));
}

// ------------------------------------------------------------------ SpGEMM
static msp_status check_pair_mul(const msp_csr *A, const msp_csr *B)
{
    msp_status st = check_csr(A, "A");
    if (st == MSP_OK) st = check_csr(B, "B");
    if (st != MSP_OK) return st;
    if (A->ncols != B->nrows) {
        set_error("spgemm: A is %dx%d but B is %dx%d", A->nrows, A->ncols, B->nrows, B->ncols);
        return MSP_ERR_SHAPE;
    }
    if (A->dtype != B->dtype) {
        set_error("spgemm: dtypes differ");
        return MSP_ERR_DTYPE;
    }
    return MSP_OK;
}

msp_status msp_spgemm_setup_workspace(const msp_csr *A, const msp_csr *B, size_t *bytes)
{
    clear_error();
    msp_status st = check_pair_mul(A, B);
    if (st != MSP_OK) return st;
    if (!bytes) return MSP_ERR_ARG;
    *bytes = spgemm_setup_ws_bytes(A, B) + kValidateBytes;
    return MSP_OK;
}

msp_status msp_spgemm_setup(const msp_csr *A, const msp_csr *B, void *setup_ws, size_t setup_ws_bytes,
                            msp_spgemm_info *info_host, void *stream)
{
    clear_error();
    msp_status st = check_pair_mul(A, B);
    if (st != MSP_OK) return st;
    if (!setup_ws || !info_host) return MSP_ERR_ARG;
    if (setup_ws_bytes < spgemm_setup_ws_bytes(A, B)) return MSP_ERR_WORKSPACE;
    st = debug_validate(A, 1, setup_ws, setup_ws_bytes, spgemm_setup_ws_bytes(A, B), as_stream(stream), "spgemm A");
    if (st == MSP_OK)
        st = debug_validate(B, 1, setup_ws, setup_ws_bytes, spgemm_setup_ws_bytes(A, B), as_stream(stream), "spgemm B");
    if (st != MSP_OK) return st;
    return spgemm_setup_run(A, B, setup_ws, setup_ws_bytes, info_host, as_stream(stream));
}

msp_status msp_spgemm_symbolic(const msp_csr *A, const msp_csr *B, const void *setup_ws, size_t setup_ws_bytes,
                               void *main_ws, size_t main_ws_bytes, msp_spgemm_info *info_host,
                               int32_t *C_row_offsets, int64_t *nnzC_host, void *stream)
{
    clear_error();
    msp_status st = check_pair_mul(A, B);
    if (st != MSP_OK) return st;
    if (!setup_ws || !main_ws || !info_host || !C_row_offsets || !nnzC_host) return MSP_ERR_ARG;
    if (main_ws_bytes < size_t(info_host->main_ws_bytes)) return MSP_ERR_WORKSPACE;
    return spgemm_symbolic_run(A, B, setup_ws, setup_ws_bytes, main_ws, main_ws_bytes, info_host, C_row_offsets,
                               nnzC_host, as_stream(stream));
}

msp_status msp_spgemm_numeric(const msp_csr *A, const msp_csr *B, const void *setup_ws, size_t setup_ws_bytes,
                              void *main_ws, size_t main_ws_bytes, const msp_spgemm_info *info_host,
                              const int32_t *C_row_offsets, int32_t *C_col_idx, void *C_vals, void *stream)
{
    clear_error();
    msp_status st = check_pair_mul(A, B);
    if (st != MSP_OK) return st;
    if (!setup_ws || !main_ws || !info_host || !C_row_offsets) return MSP_ERR_ARG;
    if (main_ws_bytes < size_t(info_host->main_ws_bytes)) return MSP_ERR_WORKSPACE;
    return spgemm_numeric_run(A, B, setup_ws, setup_ws_bytes, main_ws, main_ws_bytes, info_host, C_row_offsets,
                              C_col_idx, C_vals, as_stream(stream));
}

msp_status msp_spgemm_radix_workspace(const msp_csr *A, const msp_csr *B, const msp_spgemm_info *info_host,
                                      size_t *bytes)
{
    clear_error();
    msp_status st = check_pair_mul(A, B);
    if (st != MSP_OK) return st;
    if (!info_host || !bytes) return MSP_ERR_ARG;
    *bytes = spgemm_radix_ws_bytes(A, B, info_host->nprods);
    return MSP_OK;
}

msp_status msp_spgemm_radix_symbolic(const msp_csr *A, const msp_csr *B, const void *setup_ws, size_t setup_ws_bytes,
                                     void *ws, size_t ws_bytes, const msp_spgemm_info *info_host,
                                     int32_t *C_row_offsets, int64_t *nnzC_host, void *stream)
{
    clear_error();
    msp_status st = check_pair_mul(A, B);
    if (st != MSP_OK) return st;
    if (!setup_ws || !ws || !info_host || !C_row_offsets || !nnzC_host) return MSP_ERR_ARG;
    if (info_host->nprods >= (int64_t(1) << 32)) {
        set_error("spgemm_radix: Nprods >= 2^32 (32-bit reduced-entry indices)");
        return MSP_ERR_OVERFLOW;
    }
    if (ws_bytes < spgemm_radix_ws_bytes(A, B, info_host->nprods)) return MSP_ERR_WORKSPACE;
    return spgemm_radix_symbolic_run(A, B, setup_ws, setup_ws_bytes, ws, ws_bytes, info_host->nprods, C_row_offsets,
                                     nnzC_host, as_stream(stream));
}

msp_status msp_spgemm_radix_numeric(const msp_csr *A, const msp_csr *B, const void *setup_ws, size_t setup_ws_bytes,
                                    void *ws, size_t ws_bytes, const msp_spgemm_info *info_host,
                                    const int32_t *C_row_offsets, int32_t *C_col_idx, void *C_vals, void *stream)
{
    clear_error();
    msp_status st = check_pair_mul(A, B);
    if (st != MSP_OK) return st;
    if (!setup_ws || !ws || !info_host || !C_row_offsets) return MSP_ERR_ARG;
    if (ws_bytes < spgemm_radix_ws_bytes(A, B, info_host->nprods)) return MSP_ERR_WORKSPACE;
    return spgemm_radix_numeric_run(A, B, setup_ws, setup_ws_bytes, ws, ws_bytes, info_host->nprods, C_row_offsets,
                                    C_col_idx, C_vals, as_stream(stream));
}

// ------------------------------------------------------------------ misc
msp_status msp_csr_check(const msp_csr *A, int require_sorted_unique, int32_t *flags_host, void *ws,
                         size_t ws_bytes, void *stream)
{
    clear_error();
    msp_status st = check_csr(A, "A");
    if (st != MSP_OK) return st;
    if (!ws) return MSP_ERR_ARG;
    return csr_check_run(A, require_sorted_unique, flags_host, ws, ws_bytes, as_stream(stream));
}

msp_status msp_row_split(const int32_t *rp, int32_t nrows, int32_t P, int32_t *starts)
{
    clear_error();
    if (!rp || !starts || nrows < 0 || P < 1) return MSP_ERR_ARG;
    const int64_t nnz = rp[nrows];
    starts[0] = 0;
    for (int32_t r = 1; r < P; ++r) {
        const int64_t target = (int64_t(r) * nnz + P - 1) / P;
        // lower_bound(rp[0..nrows], target)
        int32_t lo = 0, hi = nrows;
        while (lo < hi) {
            const int32_t mid = lo + (hi - lo) / 2;
            if (int64_t(rp[mid]) < target) lo = mid + 1;
            else hi = mid;
        }
        starts[r] = lo;
    }
    starts[P] = nrows;
    return MSP_OK;
}

msp_status msp_rebase_offsets(const int32_t *in, int32_t *out, int64_t n, int64_t base, void *stream)
{
    clear_error();
    if (n < 0 || (n > 0 && (!in || !out))) return MSP_ERR_ARG;
    if (in == out && n > 0) {
        set_error("rebase: in and out alias");
        return MSP_ERR_ARG;
    }
    return rebase_run(in, out, n, base, as_stream(stream));
}

msp_status msp_gather_values(const void *src, const int32_t *idx, int64_t n, int32_t value_bytes, void *dst,
                             void *stream)
{
    clear_error();
    if (n < 0 || (n > 0 && (!src || !idx || !dst))) return MSP_ERR_ARG;
    if (value_bytes != 4 && value_bytes != 8) {
        set_error("gather: value_bytes must be 4 or 8");
        return MSP_ERR_DTYPE;
    }
    return gather_run(src, idx, n, value_bytes, dst, as_stream(stream));
}

msp_status msp_set_op_workspace(int64_t nA, int64_t nB, size_t *bytes)
{
    clear_error();
    if (!bytes || nA < 0 || nB < 0) return MSP_ERR_ARG;
    *bytes = set_op_ws_bytes(nA, nB);
    return MSP_OK;
}

namespace {
msp_status set_op_args(msp_set_op op, const void *A_keys, const void *A_vals, int64_t nA, const void *B_keys,
                       const void *B_vals, int64_t nB, int32_t key_bytes, int32_t val_bytes, void *C_keys,
                       void *C_vals, int64_t C_capacity, void *ws)
{
    if (nA < 0 || nB < 0 || int(op) < 0 || int(op) > 3) return MSP_ERR_ARG;
    if (key_bytes != 4 && key_bytes != 8) {
        set_error("set op: key_bytes must be 4 or 8");
        return MSP_ERR_DTYPE;
    }
    if (val_bytes != 0 && val_bytes != 4 && val_bytes != 8) {
        set_error("set op: val_bytes must be 0, 4 or 8");
        return MSP_ERR_DTYPE;
    }
    if ((nA > 0 && !A_keys) || (nB > 0 && !B_keys) || (val_bytes && ((nA > 0 && !A_vals) || (nB > 0 && !B_vals)))) {
        set_error("set op: NULL input");
        return MSP_ERR_ARG;
    }
    if (nA + nB > (int64_t(1) << 40)) {
        set_error("set op: inputs too large");
        return MSP_ERR_OVERFLOW;
    }
    const int64_t bound = op == MSP_SET_INTERSECTION ? (nA < nB ? nA : nB) : op == MSP_SET_DIFFERENCE ? nA : nA + nB;
    if (C_capacity < bound) {
        set_error("set op: C capacity %lld below the result bound %lld", (long long)C_capacity, (long long)bound);
        return MSP_ERR_SHAPE;
    }
    if (bound > 0 && (!C_keys || (val_bytes && !C_vals))) {
        set_error("set op: NULL output");
        return MSP_ERR_ARG;
    }
    if (!ws && nA + nB > 0) return MSP_ERR_ARG;
    return MSP_OK;
}
}  // namespace

msp_status msp_set_operation(msp_set_op op, const void *A_keys, const void *A_vals, int64_t nA, const void *B_keys,
                             const void *B_vals, int64_t nB, int32_t key_bytes, int32_t val_bytes, void *C_keys,
                             void *C_vals, int64_t C_capacity, int64_t *nC_host, void *ws, size_t ws_bytes,
                             void *stream)
{
    clear_error();
    if (!nC_host) return MSP_ERR_ARG;
    msp_status st = set_op_args(op, A_keys, A_vals, nA, B_keys, B_vals, nB, key_bytes, val_bytes, C_keys, C_vals,
                                C_capacity, ws);
    if (st != MSP_OK) return st;
    return set_op_run(int(op), A_keys, A_vals, nA, B_keys, B_vals, nB, key_bytes, val_bytes, C_keys, C_vals, C_capacity,
                      nC_host, nullptr, ws, ws_bytes, as_stream(stream));
}

msp_status msp_set_operation_async(msp_set_op op, const void *A_keys, const void *A_vals, int64_t nA,
                                   const void *B_keys, const void *B_vals, int64_t nB, int32_t key_bytes,
                                   int32_t val_bytes, void *C_keys, void *C_vals, int64_t C_capacity, int64_t *nC_dev,
                                   void *ws, size_t ws_bytes, void *stream)
{
    clear_error();
    if (!nC_dev || (reinterpret_cast<uintptr_t>(nC_dev) & 7)) return MSP_ERR_ARG;
    msp_status st = set_op_args(op, A_keys, A_vals, nA, B_keys, B_vals, nB, key_bytes, val_bytes, C_keys, C_vals,
                                C_capacity, ws);
    if (st != MSP_OK) return st;
    return set_op_run(int(op), A_keys, A_vals, nA, B_keys, B_vals, nB, key_bytes, val_bytes, C_keys, C_vals, C_capacity,
                      nullptr, nC_dev, ws, ws_bytes, as_stream(stream));
}

}  // extern "C"
