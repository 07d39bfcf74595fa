"""Helpers for the -m gpu parity tests (CUDA path through the C ABI vs the
oracle on the same seeded inputs)."""
import numpy as np
import torch

import gen
import oracle


def dev(A: gen.CSR, device="cuda"):
    from paper_conf_ipps_daltonbmog15_b200 import CsrTensor
    return CsrTensor.from_arrays(A.rp, A.col, A.val, (A.m, A.n), device)


def assert_spmv(A: gen.CSR, x: np.ndarray, y_gpu: np.ndarray, rows=None, label=""):
    want, scale = oracle.spmv(A, x, rows)
    got = y_gpu if rows is None else y_gpu[rows]
    ok, msg = oracle.check_values(got, want, scale, A.val.dtype)
    assert ok, f"{label}: {msg}"


def assert_csr_equal_structure(rp, col, C: gen.CSR, label=""):
    assert np.array_equal(np.asarray(rp, dtype=np.int64), C.rp.astype(np.int64)), f"{label}: row_offsets differ"
    assert np.array_equal(np.asarray(col), C.col), f"{label}: col_idx differ"


def tile_edge_matrix(row_lens, n=None, seed=0, dtype=np.float64, mode="int"):
    """CSR with prescribed row lengths (random sorted unique columns) -- used to
    place row ends exactly on / next to tile boundaries."""
    rng = np.random.default_rng(seed)
    row_lens = np.asarray(row_lens, dtype=np.int64)
    n = int(n if n is not None else max(1, int(row_lens.max(initial=1)) + 3))
    cols = [np.sort(rng.choice(n, size=int(k), replace=False)) for k in row_lens]
    col = np.concatenate(cols).astype(np.int32) if cols else np.zeros(0, np.int32)
    rp = np.zeros(row_lens.size + 1, dtype=np.int64)
    np.cumsum(row_lens, out=rp[1:])
    val = gen.matrices.int_values(col.size, seed + 1, dtype) if mode == "int" else \
        gen.matrices.random_values(col.size, seed + 1, dtype)
    return gen.CSR(row_lens.size, n, rp.astype(np.int32), col, val)


def sync():
    torch.cuda.synchronize()
