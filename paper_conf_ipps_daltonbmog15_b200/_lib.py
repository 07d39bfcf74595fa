"""ctypes declarations of the libmsp C ABI (include/msp.h).

Argument marshalling only: every step of the hot path runs in the CUDA
kernels of libmsp.so.  If the library is missing or cannot be loaded, import
fails loudly -- there is no CPU or PyTorch fallback.
"""
from __future__ import annotations

import ctypes
import os
from pathlib import Path

_PKG = Path(__file__).resolve().parent
LIB_PATH = Path(os.environ.get("MSP_LIB", _PKG / "libmsp.so"))

MSP_F32, MSP_F64 = 0, 1
MSP_OK = 0
STATUS = {0: "MSP_OK", 1: "MSP_ERR_ARG", 2: "MSP_ERR_DTYPE", 3: "MSP_ERR_SHAPE", 4: "MSP_ERR_WORKSPACE",
          5: "MSP_ERR_OVERFLOW", 6: "MSP_ERR_INPUT", 7: "MSP_ERR_CUDA", 8: "MSP_ERR_NCCL",
          9: "MSP_ERR_UNSUPPORTED"}

# every symbol include/msp.h declares (checked by tests/test_abi.py)
EXPORTS = [
    "msp_status_string", "msp_last_error", "msp_version", "msp_launch_count",
    "msp_spmv_workspace", "msp_spmv", "msp_spmv_nnz_split_workspace", "msp_spmv_nnz_split",
    "msp_spadd_workspace", "msp_spadd_symbolic", "msp_spadd_numeric", "msp_spadd_fused",
    "msp_spgemm_setup_workspace", "msp_spgemm_setup", "msp_spgemm_symbolic", "msp_spgemm_numeric",
    "msp_spgemm_radix_workspace", "msp_spgemm_radix_symbolic", "msp_spgemm_radix_numeric",
    "msp_csr_check", "msp_row_split", "msp_rebase_offsets", "msp_gather_values",
    "msp_set_op_workspace", "msp_set_operation", "msp_set_operation_async",
]


class MspError(RuntimeError):
    def __init__(self, fn: str, status: int, detail: str):
        self.status = status
        super().__init__(f"{fn} -> {STATUS.get(status, status)}: {detail}")


class msp_csr(ctypes.Structure):
    _fields_ = [("nrows", ctypes.c_int32), ("ncols", ctypes.c_int32), ("nnz", ctypes.c_int64),
                ("row_offsets", ctypes.c_void_p), ("col_idx", ctypes.c_void_p), ("vals", ctypes.c_void_p),
                ("dtype", ctypes.c_int32)]


class msp_spgemm_info(ctypes.Structure):
    _fields_ = [("nprods", ctypes.c_int64), ("ntiles", ctypes.c_int64), ("long_rows", ctypes.c_int64),
                ("long_products", ctypes.c_int64), ("max_row_products", ctypes.c_int64),
                ("main_ws_bytes", ctypes.c_int64), ("long_chunks", ctypes.c_int64),
                ("max_tile_span", ctypes.c_int64), ("segmented_rows", ctypes.c_int64),
                ("row_accumulator", ctypes.c_int64), ("small_rows", ctypes.c_int64),
                ("bitmap_rows", ctypes.c_int64)]


_P = ctypes.POINTER
_csr_p = _P(msp_csr)
_vp = ctypes.c_void_p
_sz = ctypes.c_size_t
_i32 = ctypes.c_int32
_i64 = ctypes.c_int64

_SIGS = {
    "msp_status_string": (ctypes.c_char_p, [ctypes.c_int]),
    "msp_last_error": (ctypes.c_char_p, []),
    "msp_version": (ctypes.c_int, []),
    "msp_launch_count": (ctypes.c_uint64, []),
    "msp_spmv_workspace": (ctypes.c_int, [_csr_p, _P(_sz)]),
    "msp_spmv": (ctypes.c_int, [_csr_p, _vp, _vp, _vp, _sz, _vp]),
    "msp_spmv_nnz_split_workspace": (ctypes.c_int, [_csr_p, _P(_sz)]),
    "msp_spmv_nnz_split": (ctypes.c_int, [_csr_p, _vp, _vp, _vp, _sz, _vp]),
    "msp_spadd_workspace": (ctypes.c_int, [_csr_p, _csr_p, _P(_sz)]),
    "msp_spadd_symbolic": (ctypes.c_int, [_csr_p, _csr_p, _vp, _P(_i64), _vp, _sz, _vp]),
    "msp_spadd_numeric": (ctypes.c_int, [_csr_p, _csr_p, _vp, _vp, _vp, _vp, _sz, _vp]),
    "msp_spadd_fused": (ctypes.c_int, [_csr_p, _csr_p, _vp, _vp, _vp, _i64, _P(_i64), _vp, _sz, _vp]),
    "msp_spgemm_setup_workspace": (ctypes.c_int, [_csr_p, _csr_p, _P(_sz)]),
    "msp_spgemm_setup": (ctypes.c_int, [_csr_p, _csr_p, _vp, _sz, _P(msp_spgemm_info), _vp]),
    "msp_spgemm_symbolic": (ctypes.c_int, [_csr_p, _csr_p, _vp, _sz, _vp, _sz, _P(msp_spgemm_info), _vp, _P(_i64),
                                           _vp]),
    "msp_spgemm_numeric": (ctypes.c_int, [_csr_p, _csr_p, _vp, _sz, _vp, _sz, _P(msp_spgemm_info), _vp, _vp, _vp,
                                          _vp]),
    "msp_spgemm_radix_workspace": (ctypes.c_int, [_csr_p, _csr_p, _P(msp_spgemm_info), _P(_sz)]),
    "msp_spgemm_radix_symbolic": (ctypes.c_int, [_csr_p, _csr_p, _vp, _sz, _vp, _sz, _P(msp_spgemm_info), _vp,
                                                 _P(_i64), _vp]),
    "msp_spgemm_radix_numeric": (ctypes.c_int, [_csr_p, _csr_p, _vp, _sz, _vp, _sz, _P(msp_spgemm_info), _vp, _vp,
                                                _vp, _vp]),
    "msp_csr_check": (ctypes.c_int, [_csr_p, ctypes.c_int, _P(_i32), _vp, _sz, _vp]),
    "msp_row_split": (ctypes.c_int, [_vp, _i32, _i32, _vp]),
    "msp_rebase_offsets": (ctypes.c_int, [_vp, _vp, _i64, _i64, _vp]),
    "msp_gather_values": (ctypes.c_int, [_vp, _vp, _i64, _i32, _vp, _vp]),
    "msp_set_op_workspace": (ctypes.c_int, [_i64, _i64, _P(_sz)]),
    "msp_set_operation": (ctypes.c_int, [ctypes.c_int, _vp, _vp, _i64, _vp, _vp, _i64, _i32, _i32, _vp, _vp, _i64,
                                          _P(_i64), _vp, _sz, _vp]),
    "msp_set_operation_async": (ctypes.c_int, [ctypes.c_int, _vp, _vp, _i64, _vp, _vp, _i64, _i32, _i32, _vp, _vp,
                                                _i64, _vp, _vp, _sz, _vp]),
}

_lib = None


def lib():
    """Load libmsp.so (raises if it is missing: no fallback path exists)."""
    global _lib
    if _lib is None:
        if not LIB_PATH.exists():
            raise ImportError(f"libmsp.so not found at {LIB_PATH}; run __graft_entry__.build() "
                              "(python -m paper_conf_ipps_daltonbmog15_b200._build)")
        L = ctypes.CDLL(str(LIB_PATH))
        for name, (res, args) in _SIGS.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def check(fn: str, status: int):
    if status != MSP_OK:
        detail = lib().msp_last_error().decode(errors="replace")
        raise MspError(fn, status, detail)
