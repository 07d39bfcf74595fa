"""CPU oracle (TEST INFRASTRUCTURE ONLY).

Only ``tests/``, ``__graft_entry__.smoke()`` and bench.py's ``cpu_baseline`` /
``--impl reference`` legs may import this package.  The product path
(``paper_conf_ipps_daltonbmog15_b200``) never imports it and shares no code
with it; see ``msp_oracle.c`` for the algorithms and their paper citations.

Pins: tests/test_oracle_*.py (run with ``-m "not gpu"``).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from pathlib import Path

import numpy as np

from gen import CSR

_HERE = Path(__file__).resolve().parent
_SRC = _HERE / "msp_oracle.c"
_LIB = _HERE / "liboracle.so"
_lib = None

_i32p = np.ctypeslib.ndpointer(np.int32, flags="C_CONTIGUOUS")
_i64p = np.ctypeslib.ndpointer(np.int64, flags="C_CONTIGUOUS")
_f64p = np.ctypeslib.ndpointer(np.float64, flags="C_CONTIGUOUS")
_u64p = np.ctypeslib.ndpointer(np.uint64, flags="C_CONTIGUOUS")
_vp = ctypes.c_void_p


def build(force: bool = False) -> Path:
    """Compile the oracle with gcc -O2 -ffp-contract=off (no FMA contraction)."""
    if force or not _LIB.exists() or _LIB.stat().st_mtime < _SRC.stat().st_mtime:
        tmp = _LIB.with_suffix(f".so.{os.getpid()}")
        subprocess.check_call(["gcc", "-O2", "-ffp-contract=off", "-fno-fast-math", "-fPIC",
                               "-shared", "-o", str(tmp), str(_SRC), "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(str(_LIB))
        L.oracle_spmv.restype = None
        L.oracle_spmv.argtypes = [ctypes.c_int32, _i32p, _i32p, _vp, _vp, ctypes.c_int,
                                  ctypes.c_int64, _vp, _vp, _vp]
        L.oracle_spadd.restype = ctypes.c_int64
        L.oracle_spadd.argtypes = [ctypes.c_int32, _i32p, _i32p, _vp, _i32p, _i32p, _vp,
                                   ctypes.c_int, _i64p, _vp, _vp]
        L.oracle_spadd_rows.restype = None
        L.oracle_spadd_rows.argtypes = [ctypes.c_int64, _i32p, _i32p, _i32p, _vp, _i32p, _i32p,
                                        _vp, ctypes.c_int, _i64p, _vp, _vp]
        L.oracle_spgemm.restype = ctypes.c_int64
        L.oracle_spgemm.argtypes = [ctypes.c_int32, ctypes.c_int32, _i32p, _i32p, _vp, _i32p,
                                    _i32p, _vp, ctypes.c_int, _i64p, _vp, _vp, _vp,
                                    ctypes.POINTER(ctypes.c_int64)]
        L.oracle_spgemm_rows.restype = ctypes.c_int64
        L.oracle_spgemm_rows.argtypes = [ctypes.c_int64, _i32p, ctypes.c_int32, _i32p, _i32p,
                                         _vp, _i32p, _i32p, _vp, ctypes.c_int, _i64p, _vp,
                                         _vp, _vp]
        L.oracle_nprods.restype = ctypes.c_int64
        L.oracle_nprods.argtypes = [ctypes.c_int64, _i32p, _i32p]
        L.oracle_set_op.restype = ctypes.c_int64
        L.oracle_set_op.argtypes = [ctypes.c_int, _u64p, _vp, ctypes.c_int64, _u64p, _vp, ctypes.c_int64, _vp, _vp]
        L.oracle_row_split.restype = None
        L.oracle_row_split.argtypes = [ctypes.c_int32, _i32p, ctypes.c_int32, _i32p]
        _lib = L
    return _lib


def _dt(a: np.ndarray) -> int:
    if a.dtype == np.float64:
        return 1
    if a.dtype == np.float32:
        return 0
    raise TypeError(f"oracle supports float32/float64 values, got {a.dtype}")


def _ptr(a: np.ndarray | None):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def _c(a, dt=None):
    return np.ascontiguousarray(a if dt is None else a.astype(dt, copy=False))


def spmv(A: CSR, x: np.ndarray, rows: np.ndarray | None = None):
    """y = A x (scalar CSR); returns (y, scale) with scale_i =
    sum_j |a_ij||x_j| in fp64.  With `rows`, only those rows (in that order)."""
    dt = _dt(A.val)
    x = _c(x, A.val.dtype)
    rp, col, val = _c(A.rp), _c(A.col), _c(A.val)
    if rows is None:
        y = np.empty(A.m, dtype=A.val.dtype)
        s = np.empty(A.m, dtype=np.float64)
        lib().oracle_spmv(A.m, rp, col, _ptr(val), _ptr(x), dt, 0, None, _ptr(y), _ptr(s))
    else:
        rows = _c(rows, np.int32)
        y = np.empty(rows.size, dtype=A.val.dtype)
        s = np.empty(rows.size, dtype=np.float64)
        lib().oracle_spmv(A.m, rp, col, _ptr(val), _ptr(x), dt, rows.size, _ptr(rows),
                          _ptr(y), _ptr(s))
    return y, s


def spadd(A: CSR, B: CSR) -> CSR:
    """C = A + B (two-pointer row merge, Alg. 1 tie rule; symbolic union)."""
    assert A.m == B.m and A.n == B.n and A.val.dtype == B.val.dtype
    dt = _dt(A.val)
    args = [_c(A.rp), _c(A.col), _ptr(_c(A.val)), _c(B.rp), _c(B.col), _ptr(_c(B.val)), dt]
    keep = (args[2], args[5])  # noqa: F841  (keep buffers alive)
    rpC = np.empty(A.m + 1, dtype=np.int64)
    nnz = lib().oracle_spadd(A.m, *args, rpC, None, None)
    col = np.empty(nnz, dtype=np.int32)
    val = np.empty(nnz, dtype=A.val.dtype)
    lib().oracle_spadd(A.m, *args, rpC, _ptr(col), _ptr(val))
    return CSR(A.m, A.n, _rp32(rpC), col, val)


def spadd_rows(A: CSR, B: CSR, rows: np.ndarray):
    """Selected rows of A + B -> (offsets int64[len(rows)+1], col, val)."""
    dt = _dt(A.val)
    rows = _c(rows, np.int32)
    Av, Bv = _c(A.val), _c(B.val)
    off = np.empty(rows.size + 1, dtype=np.int64)
    L = lib()
    L.oracle_spadd_rows(rows.size, rows, _c(A.rp), _c(A.col), _ptr(Av), _c(B.rp), _c(B.col),
                        _ptr(Bv), dt, off, None, None)
    col = np.empty(int(off[-1]), dtype=np.int32)
    val = np.empty(int(off[-1]), dtype=A.val.dtype)
    L.oracle_spadd_rows(rows.size, rows, _c(A.rp), _c(A.col), _ptr(Av), _c(B.rp), _c(B.col),
                        _ptr(Bv), dt, off, _ptr(col), _ptr(val))
    return off, col, val


def _rp32(rp64: np.ndarray) -> np.ndarray:
    if rp64[-1] > np.iinfo(np.int32).max:
        raise OverflowError("nnz(C) exceeds int32")
    return rp64.astype(np.int32)


def spgemm(A: CSR, B: CSR, with_scale: bool = True):
    """C = A B (Gustavson, dense accumulator).  Returns (C, scale, nprods);
    scale_ij = sum_k |a_ik||b_kj| (fp64) is the tolerance scale (Z18)."""
    assert A.n == B.m and A.val.dtype == B.val.dtype
    dt = _dt(A.val)
    Av, Bv = _c(A.val), _c(B.val)
    args = [_c(A.rp), _c(A.col), _ptr(Av), _c(B.rp), _c(B.col), _ptr(Bv), dt]
    rpC = np.empty(A.m + 1, dtype=np.int64)
    npr = ctypes.c_int64(0)
    L = lib()
    nnz = L.oracle_spgemm(A.m, B.n, *args, rpC, None, None, None, ctypes.byref(npr))
    if nnz < 0:
        raise MemoryError("oracle_spgemm: allocation failed")
    col = np.empty(nnz, dtype=np.int32)
    val = np.empty(nnz, dtype=A.val.dtype)
    sc = np.empty(nnz, dtype=np.float64) if with_scale else None
    L.oracle_spgemm(A.m, B.n, *args, rpC, _ptr(col), _ptr(val), _ptr(sc), ctypes.byref(npr))
    return CSR(A.m, B.n, _rp32(rpC), col, val), sc, int(npr.value)


def spgemm_rows(A: CSR, B: CSR, rows: np.ndarray):
    """Selected rows of A B -> (offsets int64[len+1], col, val, scale)."""
    dt = _dt(A.val)
    rows = _c(rows, np.int32)
    Av, Bv = _c(A.val), _c(B.val)
    args = [_c(A.rp), _c(A.col), _ptr(Av), _c(B.rp), _c(B.col), _ptr(Bv), dt]
    off = np.empty(rows.size + 1, dtype=np.int64)
    L = lib()
    tot = L.oracle_spgemm_rows(rows.size, rows, B.n, *args, off, None, None, None)
    if tot < 0:
        raise MemoryError("oracle_spgemm_rows: allocation failed")
    col = np.empty(tot, dtype=np.int32)
    val = np.empty(tot, dtype=A.val.dtype)
    sc = np.empty(tot, dtype=np.float64)
    L.oracle_spgemm_rows(rows.size, rows, B.n, *args, off, _ptr(col), _ptr(val), _ptr(sc))
    return off, col, val, sc


def nprods(A: CSR, B: CSR) -> int:
    return int(lib().oracle_nprods(A.nnz, _c(A.col), _c(B.rp)))


def row_split(rp: np.ndarray, P: int) -> np.ndarray:
    """Rank r owns rows [R_r, R_{r+1}), R_r = lower_bound(rp, ceil(r nnz / P))."""
    rp = _c(rp, np.int32)
    out = np.empty(P + 1, dtype=np.int32)
    lib().oracle_row_split(rp.size - 1, rp, P, out)
    return out


# ----------------------------------------------------------------------------
# Comparison rule (BJ:5; SURVEY §8(c) "Comparison rule")
# ----------------------------------------------------------------------------

TOL = {np.dtype(np.float64): 1e-12, np.dtype(np.float32): 1e-5}


def check_values(got: np.ndarray, want: np.ndarray, scale: np.ndarray, dtype) -> tuple[bool, str]:
    """|got - want| <= tau * scale per entry; scale == 0 -> got must be exactly
    0; NaN positions must match (Z19)."""
    tau = TOL[np.dtype(dtype)]
    g = got.astype(np.float64)
    w = want.astype(np.float64)
    gn, wn = np.isnan(g), np.isnan(w)
    if not np.array_equal(gn, wn):
        return False, "NaN positions differ"
    # an infinity propagates (Z19): where either side is infinite both must be
    # the same infinity (|inf - -inf| <= tau * inf would otherwise pass)
    inf = (np.isinf(g) | np.isinf(w)) & ~gn
    if np.any(g[inf] != w[inf]):
        return False, "infinities differ"
    ok = ~gn & ~inf
    err = np.abs(g[ok] - w[ok])
    # fp32 results are rounded once from an fp64 accumulator on both sides
    # (Z4); a one-ulp difference of the stored value is <= 2^-23 |y| <=
    # 2^-23 scale < 1e-5 scale, so no extra allowance is needed.
    lim = tau * scale[ok]
    bad = err > lim
    zero_scale = scale[ok] == 0
    bad |= zero_scale & (g[ok] != 0)
    if bad.any():
        i = int(np.flatnonzero(bad)[0])
        return False, (f"{int(bad.sum())} entries out of tolerance; first at {i}: "
                       f"got {g[ok][i]!r} want {w[ok][i]!r} scale {scale[ok][i]!r}")
    return True, "ok"


SET_OPS = {"union": 0, "intersection": 1, "difference": 2, "symmetric_difference": 3}


def set_op(op: str, a_keys, b_keys, a_vals=None, b_vals=None):
    """Multiset operation on sorted keys (key-rank pairs, msp_oracle.c
    oracle_set_op).  Keys: unsigned 32/64-bit arrays; values: optional arrays
    of the same length (any 4/8-byte dtype, carried bit-for-bit).
    Returns (keys, vals or None) in the input dtypes."""
    kd = np.asarray(a_keys).dtype
    A = np.ascontiguousarray(np.asarray(a_keys).astype(np.uint64))
    B = np.ascontiguousarray(np.asarray(b_keys).astype(np.uint64))
    has_v = a_vals is not None
    if has_v:
        vd = np.asarray(a_vals).dtype
        ut = np.uint32 if vd.itemsize == 4 else np.uint64
        Av = np.ascontiguousarray(np.asarray(a_vals).view(ut).astype(np.uint64))
        Bv = np.ascontiguousarray(np.asarray(b_vals).view(ut).astype(np.uint64))
    L = lib()
    code = SET_OPS[op]
    n = L.oracle_set_op(code, A, _ptr(Av) if has_v else None, A.size, B, _ptr(Bv) if has_v else None, B.size,
                        None, None)
    C = np.empty(n, dtype=np.uint64)
    Cv = np.empty(n, dtype=np.uint64) if has_v else None
    L.oracle_set_op(code, A, _ptr(Av) if has_v else None, A.size, B, _ptr(Bv) if has_v else None, B.size,
                    _ptr(C), _ptr(Cv) if has_v else None)
    keys = C.astype(kd)
    vals = Cv.astype(ut).view(vd) if has_v else None
    return keys, vals
