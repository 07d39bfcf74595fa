// temporary: SpGEMM entry points before its kernels land
#include "internal.h"
namespace msp {
size_t spgemm_setup_ws_bytes(const msp_csr *, const msp_csr *) { return 256; }
msp_status spgemm_setup_run(const msp_csr *, const msp_csr *, void *, size_t, msp_spgemm_info *, cudaStream_t) { set_error("spgemm not built yet"); return MSP_ERR_UNSUPPORTED; }
msp_status spgemm_symbolic_run(const msp_csr *, const msp_csr *, const void *, size_t, void *, size_t, int32_t *, int64_t *, cudaStream_t) { return MSP_ERR_UNSUPPORTED; }
msp_status spgemm_numeric_run(const msp_csr *, const msp_csr *, const void *, size_t, void *, size_t, const int32_t *, int32_t *, void *, cudaStream_t) { return MSP_ERR_UNSUPPORTED; }
}
