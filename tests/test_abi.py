"""CPU-only checks of the C-ABI boundary: the library loads, exports every
symbol include/msp.h declares, and rejects bad arguments on the host before
any launch.  No compute call is made (there is no GPU here)."""
import ctypes
import re
from pathlib import Path

import numpy as np

import oracle
from paper_conf_ipps_daltonbmog15_b200 import _lib

ROOT = Path(__file__).resolve().parents[1]


def declared_symbols():
    txt = (ROOT / "include" / "msp.h").read_text()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(msp_[a-z0-9_]+)\s*\(", txt)))


def test_header_matches_binding_table():
    assert declared_symbols() == sorted(_lib.EXPORTS)


def test_library_exports_every_declared_symbol():
    L = _lib.lib()
    for name in declared_symbols():
        assert hasattr(L, name), name
    assert L.msp_version() == 6


def test_only_abi_symbols_exported():
    import subprocess
    out = subprocess.run(["nm", "-D", "--defined-only", str(_lib.LIB_PATH)], capture_output=True,
                         text=True).stdout
    names = [ln.split()[-1] for ln in out.splitlines() if ln.strip()]
    assert names and all(n.startswith("msp_") for n in names), names


def test_status_strings():
    L = _lib.lib()
    for code, name in _lib.STATUS.items():
        assert L.msp_status_string(code).decode() == name


def test_host_argument_checks():
    L = _lib.lib()
    n = ctypes.c_size_t(0)
    assert L.msp_spmv_workspace(None, ctypes.byref(n)) == 1                      # MSP_ERR_ARG
    a = _lib.msp_csr(4, 4, 6, 0, 0, 0, 1)                                         # NULL arrays
    assert L.msp_spmv_workspace(ctypes.byref(a), ctypes.byref(n)) == 1
    a = _lib.msp_csr(4, 4, 6, 8, 8, 8, 7)                                         # bad dtype
    assert L.msp_spmv_workspace(ctypes.byref(a), ctypes.byref(n)) == 2
    a = _lib.msp_csr(4, 5, 6, 8, 8, 8, 1)
    b = _lib.msp_csr(4, 4, 6, 8, 8, 8, 1)
    assert L.msp_spadd_workspace(ctypes.byref(a), ctypes.byref(b), ctypes.byref(n)) == 3   # shape
    b = _lib.msp_csr(4, 5, 6, 8, 8, 8, 0)
    assert L.msp_spadd_workspace(ctypes.byref(a), ctypes.byref(b), ctypes.byref(n)) == 2   # dtype
    c = _lib.msp_csr(4, 4, 6, 8, 8, 8, 1)
    assert L.msp_spgemm_setup_workspace(ctypes.byref(a), ctypes.byref(c), ctypes.byref(n)) == 3
    a = _lib.msp_csr(4, 4, 6, 8, 8, 8, 1)
    assert L.msp_spmv(ctypes.byref(a), None, None, None, 0, None) == 1
    assert "NULL" in L.msp_last_error().decode()
    assert L.msp_rebase_offsets(8, 8, 3, 0, None) == 1                           # aliasing


def test_row_split_matches_oracle():
    import gen
    L = _lib.lib()
    for A in (gen.config("C1"), gen.random_csr(500, 30, 3, density=0.1, empty_frac=0.4, dense_rows=2)):
        for P in (1, 2, 3, 4, 8):
            out = np.empty(P + 1, dtype=np.int32)
            rp = np.ascontiguousarray(A.rp)
            assert L.msp_row_split(rp.ctypes.data, A.m, P, out.ctypes.data) == 0
            assert np.array_equal(out, oracle.row_split(A.rp, P))
