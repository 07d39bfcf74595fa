"""PyTorch-facing wrappers of the libmsp C ABI (argument marshalling only).

Tensors live on a CUDA device; outputs and workspaces are allocated with
torch and passed to libmsp by pointer together with the current CUDA stream.
Every computation happens in the sm_100a kernels of libmsp.so; there is no
CPU path.  Names follow the paper: spmv (Section III-A), spadd (III-B),
spgemm (III-C).
"""
from __future__ import annotations

import ctypes
import itertools
from dataclasses import dataclass

import torch

from ._lib import MSP_F32, MSP_F64, check, lib, msp_csr, msp_spgemm_info

_DT = {torch.float32: MSP_F32, torch.float64: MSP_F64}


@dataclass
class CsrTensor:
    """CSR matrix on a CUDA device: row_offsets int32[m+1], col_idx int32[nnz],
    vals float32/float64[nnz]; columns sorted within each row."""
    rp: torch.Tensor
    col: torch.Tensor
    val: torch.Tensor
    shape: tuple[int, int]

    @property
    def nnz(self) -> int:
        return int(self.col.numel())

    @property
    def dtype(self):
        return self.val.dtype

    @property
    def device(self):
        return self.val.device

    @classmethod
    def from_arrays(cls, rp, col, val, shape, device="cuda") -> "CsrTensor":
        t = lambda a, dt=None: torch.as_tensor(a, dtype=dt, device=device).contiguous()  # noqa: E731
        return cls(t(rp, torch.int32), t(col, torch.int32), t(val), (int(shape[0]), int(shape[1])))

    def c(self) -> msp_csr:
        if self.val.dtype not in _DT:
            raise TypeError(f"unsupported dtype {self.val.dtype}")
        for t in (self.rp, self.col, self.val):
            if not t.is_contiguous():
                raise ValueError("CSR arrays must be contiguous")
        return msp_csr(self.shape[0], self.shape[1], self.nnz, self.rp.data_ptr(),
                       self.col.data_ptr() if self.nnz else 0, self.val.data_ptr() if self.nnz else 0,
                       _DT[self.val.dtype])

    def numpy(self):
        return (self.rp.cpu().numpy(), self.col.cpu().numpy(), self.val.cpu().numpy())


# ----------------------------------------------------------------- workspaces

_WS: dict = {}
_OWNER: dict = {}
_TOKENS = itertools.count(1)


def _ws_key(device, slot: str, stream=None):
    dev = torch.device(device)
    s = stream if stream is not None else torch.cuda.current_stream(dev)
    return (dev.index, s.cuda_stream, slot)


def workspace(nbytes: int, device, slot: str, stream=None) -> torch.Tensor:
    """Zero-initialised byte workspace cached per (device, stream, slot).  Each
    slot is only ever used by one kind of call, whose kernels leave their
    counters zeroed, so reuse needs no re-clearing.  Symbolic -> numeric
    state kept in a slot belongs to the plan that last ran its symbolic
    phase there (see _claim / _owns)."""
    key = _ws_key(device, slot, stream)
    buf = _WS.get(key)
    if buf is None or buf.numel() < nbytes:
        buf = torch.zeros(max(int(nbytes), 256), dtype=torch.uint8, device=torch.device(device))
        _WS[key] = buf
        _OWNER.pop(key, None)
    return buf


def _claim(token: int, device, slots, stream=None) -> None:
    for sl in slots:
        _OWNER[_ws_key(device, sl, stream)] = token


def _owns(token: int, device, slots, stream=None) -> bool:
    return all(_OWNER.get(_ws_key(device, sl, stream)) == token for sl in slots)


def _stream_ptr(device, stream=None):
    s = stream if stream is not None else torch.cuda.current_stream(torch.device(device))
    return ctypes.c_void_p(s.cuda_stream)


# ----------------------------------------------------------------- SpMV

def spmv_workspace_bytes(A: CsrTensor) -> int:
    n = ctypes.c_size_t(0)
    a = A.c()
    check("msp_spmv_workspace", lib().msp_spmv_workspace(ctypes.byref(a), ctypes.byref(n)))
    return int(n.value)


def spmv(A: CsrTensor, x: torch.Tensor, out: torch.Tensor | None = None, stream=None,
         ws: torch.Tensor | None = None) -> torch.Tensor:
    """y = A x  (merge-path SpMV)."""
    if x.dtype != A.dtype or x.device != A.device or x.numel() != A.shape[1] or not x.is_contiguous():
        raise ValueError("x must be a contiguous vector of A.dtype on A.device with A.shape[1] entries")
    y = out if out is not None else torch.empty(A.shape[0], dtype=A.dtype, device=A.device)
    a = A.c()
    if ws is None:
        ws = workspace(spmv_workspace_bytes(A), A.device, "spmv", stream)
    check("msp_spmv", lib().msp_spmv(ctypes.byref(a), x.data_ptr(), y.data_ptr(), ws.data_ptr(),
                                     ws.numel(), _stream_ptr(A.device, stream)))
    return y


def spmv_nnz_split(A: CsrTensor, x: torch.Tensor, out: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    """y = A x with the paper's own decomposition (nnz-only split + row
    compaction): the f4(i) ablation of spmv()."""
    if x.dtype != A.dtype or x.device != A.device or x.numel() != A.shape[1] or not x.is_contiguous():
        raise ValueError("x must be a contiguous vector of A.dtype on A.device with A.shape[1] entries")
    y = out if out is not None else torch.empty(A.shape[0], dtype=A.dtype, device=A.device)
    a = A.c()
    n = ctypes.c_size_t(0)
    check("msp_spmv_nnz_split_workspace", lib().msp_spmv_nnz_split_workspace(ctypes.byref(a), ctypes.byref(n)))
    ws = workspace(int(n.value), A.device, "spmv_nnz", stream)
    check("msp_spmv_nnz_split", lib().msp_spmv_nnz_split(ctypes.byref(a), x.data_ptr(), y.data_ptr(), ws.data_ptr(),
                                                         ws.numel(), _stream_ptr(A.device, stream)))
    return y


# ----------------------------------------------------------------- SpAdd

class SpAddPlan:
    """Two-phase SpAdd: symbolic() counts C's rows and returns
    nnz(C); numeric() fills C with the partition symbolic() stored."""

    def __init__(self, A: CsrTensor, B: CsrTensor, stream=None):
        self.A, self.B, self.stream = A, B, stream
        self.a, self.b = A.c(), B.c()
        n = ctypes.c_size_t(0)
        check("msp_spadd_workspace", lib().msp_spadd_workspace(ctypes.byref(self.a), ctypes.byref(self.b),
                                                               ctypes.byref(n)))
        self.ws_bytes = int(n.value)
        self.ws = workspace(self.ws_bytes, A.device, "spadd", stream)
        self.rp = torch.empty(A.shape[0] + 1, dtype=torch.int32, device=A.device)
        self.nnz = None
        self.token = next(_TOKENS)

    def symbolic(self) -> int:
        nnz = ctypes.c_int64(0)
        self.ws = workspace(self.ws_bytes, self.A.device, "spadd", self.stream)
        check("msp_spadd_symbolic",
              lib().msp_spadd_symbolic(ctypes.byref(self.a), ctypes.byref(self.b), self.rp.data_ptr(),
                                       ctypes.byref(nnz), self.ws.data_ptr(), self.ws.numel(),
                                       _stream_ptr(self.A.device, self.stream)))
        _claim(self.token, self.A.device, ("spadd",), self.stream)
        self.nnz = int(nnz.value)
        return self.nnz

    def numeric(self, col: torch.Tensor | None = None, val: torch.Tensor | None = None) -> CsrTensor:
        # numeric needs the partition this plan's symbolic call left in the
        # shared workspace; if another plan has used it since, redo symbolic
        if self.nnz is None or not _owns(self.token, self.A.device, ("spadd",), self.stream):
            self.symbolic()
        dev = self.A.device
        col = col if col is not None else torch.empty(self.nnz, dtype=torch.int32, device=dev)
        val = val if val is not None else torch.empty(self.nnz, dtype=self.A.dtype, device=dev)
        check("msp_spadd_numeric",
              lib().msp_spadd_numeric(ctypes.byref(self.a), ctypes.byref(self.b), self.rp.data_ptr(),
                                      col.data_ptr() if self.nnz else None, val.data_ptr() if self.nnz else None,
                                      self.ws.data_ptr(), self.ws.numel(), _stream_ptr(dev, self.stream)))
        return CsrTensor(self.rp, col, val, self.A.shape)


def spadd(A: CsrTensor, B: CsrTensor, stream=None) -> CsrTensor:
    """C = A + B (balanced-path union)."""
    p = SpAddPlan(A, B, stream)
    p.symbolic()
    return p.numeric()


def spadd_fused(A: CsrTensor, B: CsrTensor, stream=None, col: torch.Tensor | None = None,
                val: torch.Tensor | None = None) -> CsrTensor:
    """C = A + B in one pass (msp_spadd_fused; same result as spadd() bit for
    bit).  col / val, if given, need nnz(A) + nnz(B) entries; the returned
    C.col / C.vals are views of their first nnz(C) entries."""
    a, b = A.c(), B.c()
    if A.shape != B.shape:
        raise ValueError("A and B differ in shape")
    dev = A.device
    cap = A.nnz + B.nnz
    n = ctypes.c_size_t(0)
    check("msp_spadd_workspace", lib().msp_spadd_workspace(ctypes.byref(a), ctypes.byref(b), ctypes.byref(n)))
    ws = workspace(int(n.value), dev, "spadd", stream)
    _claim(next(_TOKENS), dev, ("spadd",), stream)  # any SpAddPlan's partition in this slot is gone
    rp = torch.empty(A.shape[0] + 1, dtype=torch.int32, device=dev)
    col = col if col is not None else torch.empty(max(cap, 1), dtype=torch.int32, device=dev)
    val = val if val is not None else torch.empty(max(cap, 1), dtype=A.dtype, device=dev)
    if col.numel() < cap or val.numel() < cap:
        raise ValueError("col / val need nnz(A) + nnz(B) entries")
    nnz = ctypes.c_int64(0)
    check("msp_spadd_fused", lib().msp_spadd_fused(ctypes.byref(a), ctypes.byref(b), rp.data_ptr(), col.data_ptr(),
                                                   val.data_ptr(), cap, ctypes.byref(nnz), ws.data_ptr(), ws.numel(),
                                                   _stream_ptr(dev, stream)))
    k = int(nnz.value)
    return CsrTensor(rp, col[:k], val[:k], A.shape)


# ----------------------------------------------------------------- SpGEMM

class SpGemmPlan:
    """ESC SpGEMM: setup() -> Nprods and sizes, symbolic() ->
    C.row_offsets and nnz(C), numeric() -> C.col / C.vals."""

    def __init__(self, A: CsrTensor, B: CsrTensor, stream=None):
        if A.shape[1] != B.shape[0]:
            raise ValueError("inner dimensions differ")
        self.A, self.B, self.stream = A, B, stream
        self.a, self.b = A.c(), B.c()
        n = ctypes.c_size_t(0)
        check("msp_spgemm_setup_workspace",
              lib().msp_spgemm_setup_workspace(ctypes.byref(self.a), ctypes.byref(self.b), ctypes.byref(n)))
        self.ws1_bytes = int(n.value)
        self.ws1 = workspace(self.ws1_bytes, A.device, "spgemm_setup", stream)
        self.info = None
        self.ws2 = None
        self.rp = torch.empty(A.shape[0] + 1, dtype=torch.int32, device=A.device)
        self.nnz = None
        self.token = next(_TOKENS)

    _SLOTS = ("spgemm_setup", "spgemm_main")

    def setup(self) -> msp_spgemm_info:
        info = msp_spgemm_info()
        self.ws1 = workspace(self.ws1_bytes, self.A.device, "spgemm_setup", self.stream)
        check("msp_spgemm_setup",
              lib().msp_spgemm_setup(ctypes.byref(self.a), ctypes.byref(self.b), self.ws1.data_ptr(),
                                     self.ws1.numel(), ctypes.byref(info), _stream_ptr(self.A.device, self.stream)))
        self.info = info
        self.ws2 = workspace(int(info.main_ws_bytes), self.A.device, "spgemm_main", self.stream)
        _claim(self.token, self.A.device, self._SLOTS[:1], self.stream)
        self.nnz = None  # symbolic must follow a setup
        return info

    @property
    def nprods(self) -> int:
        if self.info is None:
            self.setup()
        return int(self.info.nprods)

    def symbolic(self) -> int:
        if self.info is None or not _owns(self.token, self.A.device, self._SLOTS[:1], self.stream):
            self.setup()
        nnz = ctypes.c_int64(0)
        check("msp_spgemm_symbolic",
              lib().msp_spgemm_symbolic(ctypes.byref(self.a), ctypes.byref(self.b), self.ws1.data_ptr(),
                                        self.ws1.numel(), self.ws2.data_ptr(), self.ws2.numel(),
                                        ctypes.byref(self.info), self.rp.data_ptr(), ctypes.byref(nnz),
                                        _stream_ptr(self.A.device, self.stream)))
        _claim(self.token, self.A.device, self._SLOTS, self.stream)
        self.nnz = int(nnz.value)
        return self.nnz

    def numeric(self, col: torch.Tensor | None = None, val: torch.Tensor | None = None) -> CsrTensor:
        # numeric reads the setup arrays and the tile permutations this plan's
        # symbolic call left in the shared workspaces; redo them if another
        # plan has used those workspaces since
        if self.nnz is None or not _owns(self.token, self.A.device, self._SLOTS, self.stream):
            self.symbolic()
        dev = self.A.device
        col = col if col is not None else torch.empty(self.nnz, dtype=torch.int32, device=dev)
        val = val if val is not None else torch.empty(self.nnz, dtype=self.A.dtype, device=dev)
        check("msp_spgemm_numeric",
              lib().msp_spgemm_numeric(ctypes.byref(self.a), ctypes.byref(self.b), self.ws1.data_ptr(),
                                       self.ws1.numel(), self.ws2.data_ptr(), self.ws2.numel(),
                                       ctypes.byref(self.info), self.rp.data_ptr(),
                                       col.data_ptr() if self.nnz else None, val.data_ptr() if self.nnz else None,
                                       _stream_ptr(dev, self.stream)))
        return CsrTensor(self.rp, col, val, (self.A.shape[0], self.B.shape[1]))


class SpGemmRadixPlan(SpGemmPlan):
    """SpGEMM with the paper's own sort pipeline (the f2
    ablation): setup() as SpGemmPlan, then radix symbolic / numeric."""

    def symbolic(self) -> int:
        if self.info is None or not _owns(self.token, self.A.device, self._SLOTS[:1], self.stream):
            self.setup()
        n = ctypes.c_size_t(0)
        check("msp_spgemm_radix_workspace",
              lib().msp_spgemm_radix_workspace(ctypes.byref(self.a), ctypes.byref(self.b), ctypes.byref(self.info),
                                               ctypes.byref(n)))
        self.wsr = workspace(int(n.value), self.A.device, "spgemm_radix", self.stream)
        nnz = ctypes.c_int64(0)
        check("msp_spgemm_radix_symbolic",
              lib().msp_spgemm_radix_symbolic(ctypes.byref(self.a), ctypes.byref(self.b), self.ws1.data_ptr(),
                                              self.ws1.numel(), self.wsr.data_ptr(), self.wsr.numel(),
                                              ctypes.byref(self.info), self.rp.data_ptr(), ctypes.byref(nnz),
                                              _stream_ptr(self.A.device, self.stream)))
        _claim(self.token, self.A.device, ("spgemm_setup", "spgemm_radix"), self.stream)
        self.nnz = int(nnz.value)
        return self.nnz

    def numeric(self, col: torch.Tensor | None = None, val: torch.Tensor | None = None) -> CsrTensor:
        if self.nnz is None or not _owns(self.token, self.A.device, ("spgemm_setup", "spgemm_radix"), self.stream):
            self.symbolic()
        dev = self.A.device
        col = col if col is not None else torch.empty(self.nnz, dtype=torch.int32, device=dev)
        val = val if val is not None else torch.empty(self.nnz, dtype=self.A.dtype, device=dev)
        check("msp_spgemm_radix_numeric",
              lib().msp_spgemm_radix_numeric(ctypes.byref(self.a), ctypes.byref(self.b), self.ws1.data_ptr(),
                                             self.ws1.numel(), self.wsr.data_ptr(), self.wsr.numel(),
                                             ctypes.byref(self.info), self.rp.data_ptr(),
                                             col.data_ptr() if self.nnz else None,
                                             val.data_ptr() if self.nnz else None, _stream_ptr(dev, self.stream)))
        return CsrTensor(self.rp, col, val, (self.A.shape[0], self.B.shape[1]))


def spgemm(A: CsrTensor, B: CsrTensor, stream=None) -> CsrTensor:
    """C = A B (expand / sort / compress)."""
    p = SpGemmPlan(A, B, stream)
    p.setup()
    p.symbolic()
    return p.numeric()


# ----------------------------------------------------------------- misc

def csr_check(A: CsrTensor, sorted_unique: bool = True) -> int:
    """Validate the CSR contract on the device; returns the flag bits."""
    a = A.c()
    ws = workspace(256, A.device, "check")
    flags = ctypes.c_int32(0)
    st = lib().msp_csr_check(ctypes.byref(a), int(sorted_unique), ctypes.byref(flags), ws.data_ptr(),
                             ws.numel(), _stream_ptr(A.device))
    if st not in (0, 6):
        check("msp_csr_check", st)
    return int(flags.value)


def row_split(rp_host, P: int):
    """nnz-balanced row blocks (host): R_r = lower_bound(rp, ceil(r nnz / P))."""
    import numpy as np
    rp = np.ascontiguousarray(rp_host, dtype=np.int32)
    out = np.empty(P + 1, dtype=np.int32)
    check("msp_row_split", lib().msp_row_split(rp.ctypes.data, rp.size - 1, P, out.ctypes.data))
    return out


def rebase_offsets(rp: torch.Tensor, base: int, out: torch.Tensor | None = None) -> torch.Tensor:
    out = out if out is not None else torch.empty_like(rp)
    check("msp_rebase_offsets", lib().msp_rebase_offsets(rp.data_ptr(), out.data_ptr(), rp.numel(), int(base),
                                                         _stream_ptr(rp.device)))
    return out


def gather_values(src: torch.Tensor, idx: torch.Tensor, out: torch.Tensor | None = None) -> torch.Tensor:
    """out[i] = src[idx[i]] on the device (msp_gather_values; halo packing)."""
    if idx.dtype != torch.int32 or not idx.is_contiguous() or not src.is_contiguous():
        raise ValueError("idx int32 and contiguous tensors required")
    out = out if out is not None else torch.empty(idx.numel(), dtype=src.dtype, device=src.device)
    check("msp_gather_values", lib().msp_gather_values(src.data_ptr(), idx.data_ptr(), idx.numel(),
                                                       src.element_size(), out.data_ptr(),
                                                       _stream_ptr(src.device)))
    return out


# ----------------------------------------------------------------- set operations

SET_OPS = {"union": 0, "intersection": 1, "difference": 2, "symmetric_difference": 3}
_KEY_T = {torch.int32: 4, torch.int64: 8, torch.uint32: 4, torch.uint64: 8}


def set_operation(op: str, a_keys: torch.Tensor, b_keys: torch.Tensor, a_vals: torch.Tensor | None = None,
                  b_vals: torch.Tensor | None = None, stream=None, sync: bool = True):
    """Balanced-path set operation on sorted key lists: keys are
    compared as unsigned 32/64-bit integers (int32/int64 tensors are
    reinterpreted), duplicates are key-rank pairs.  Returns (keys, vals or
    None), trimmed to the result size (msp_set_operation synchronises).

    sync=False calls msp_set_operation_async instead and returns (keys, vals
    or None, count): untrimmed output buffers of the result bound and a
    device int64[2] tensor holding [result size, unsorted-input flag],
    written in stream order -- no host round trip."""
    code = SET_OPS[op]
    if a_keys.dtype != b_keys.dtype or a_keys.dtype not in _KEY_T:
        raise ValueError("keys must share a 32/64-bit integer dtype")
    if not (a_keys.is_contiguous() and b_keys.is_contiguous()) or a_keys.device != b_keys.device:
        raise ValueError("keys must be contiguous tensors on one device")
    kb = _KEY_T[a_keys.dtype]
    vb = 0
    if a_vals is not None:
        if b_vals is None or a_vals.dtype != b_vals.dtype or a_vals.element_size() not in (4, 8):
            raise ValueError("values: both sides, one 4/8-byte dtype")
        if a_vals.numel() != a_keys.numel() or b_vals.numel() != b_keys.numel():
            raise ValueError("one value per key")
        vb = a_vals.element_size()
    na, nb = a_keys.numel(), b_keys.numel()
    bound = min(na, nb) if op == "intersection" else na if op == "difference" else na + nb
    dev = a_keys.device
    ck = torch.empty(max(bound, 1), dtype=a_keys.dtype, device=dev)
    cv = torch.empty(max(bound, 1), dtype=a_vals.dtype, device=dev) if vb else None
    n = ctypes.c_size_t(0)
    check("msp_set_op_workspace", lib().msp_set_op_workspace(na, nb, ctypes.byref(n)))
    ws = workspace(int(n.value), dev, "setop", stream)
    if not sync:
        count = torch.empty(2, dtype=torch.int64, device=dev)
        check("msp_set_operation_async", lib().msp_set_operation_async(
            code, a_keys.data_ptr(), a_vals.data_ptr() if vb else None, na, b_keys.data_ptr(),
            b_vals.data_ptr() if vb else None, nb, kb, vb, ck.data_ptr(), cv.data_ptr() if vb else None, bound,
            count.data_ptr(), ws.data_ptr(), ws.numel(), _stream_ptr(dev, stream)))
        return ck, cv, count
    nc = ctypes.c_int64(0)
    check("msp_set_operation", lib().msp_set_operation(
        code, a_keys.data_ptr(), a_vals.data_ptr() if vb else None, na, b_keys.data_ptr(),
        b_vals.data_ptr() if vb else None, nb, kb, vb, ck.data_ptr(), cv.data_ptr() if vb else None, bound,
        ctypes.byref(nc), ws.data_ptr(), ws.numel(), _stream_ptr(dev, stream)))
    k = int(nc.value)
    return ck[:k], (cv[:k] if vb else None)
