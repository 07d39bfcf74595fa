"""SpAdd parity: CUDA balanced-path union (C ABI) vs the oracle's two-pointer
row merge.  Structure must be bit-exact; values too (a matched pair is one
IEEE addition, A's value first; unmatched entries are copied)."""
import numpy as np
import pytest

import gen
import oracle
from tests.conftest import csr_from_dense
from tests.gpu_util import dev, tile_edge_matrix

pytestmark = pytest.mark.gpu


def run(A: gen.CSR, B: gen.CSR, fused=False):
    from paper_conf_ipps_daltonbmog15_b200 import spadd, spadd_fused
    C = (spadd_fused if fused else spadd)(dev(A), dev(B))
    rp, col, val = C.numpy()
    return rp, col, val


def check(A, B, label=""):
    """Both forms -- two-phase (symbolic + numeric) and the fused
    one-pass msp_spadd_fused -- against the oracle, bit-exact."""
    W = oracle.spadd(A, B)
    for fused in (False, True):
        rp, col, val = run(A, B, fused)
        form = "fused" if fused else "two-phase"
        assert np.array_equal(rp, W.rp), f"{label} ({form}): row_offsets differ"
        assert np.array_equal(col, W.col), f"{label} ({form}): col_idx differ"
        assert np.array_equal(val.view(np.uint8), W.val.view(np.uint8)), f"{label} ({form}): values differ"


def test_paper_example(paper_example):
    A = csr_from_dense(paper_example["A_dense"])
    B = csr_from_dense(paper_example["B_dense"])
    check(A, B, "A+B")
    check(A, gen.transpose(A), "A+A^T")


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_fuzz(dtype):
    shapes = [(1, 1), (1, 50), (50, 1), (7, 9), (64, 64), (300, 200), (1000, 40)]
    for si, (m, n) in enumerate(shapes):
        for seed in range(3):
            for kw in (dict(density=0.2), dict(density=0.03, empty_frac=0.5), dict(density=0.01, dense_rows=2)):
                A = gen.random_csr(m, n, 10 * si + seed, dtype=dtype, mode="random", **kw)
                B = gen.random_csr(m, n, 10 * si + seed + 5, dtype=dtype, mode="random", **kw)
                check(A, B, f"{m}x{n} {kw}")
                check(A, A, "A+A")                               # every key matched
                check(A, A.with_values(-A.val), "A-A")           # explicit zeros kept (Z1)


def test_empty():
    for m, n in [(0, 0), (0, 4), (4, 4)]:
        Z = gen.CSR(m, n, np.zeros(m + 1, np.int32), np.zeros(0, np.int32), np.zeros(0))
        check(Z, Z, f"empty {m}x{n}")
    A = gen.random_csr(30, 30, 1, density=0.2)
    Z = gen.CSR(30, 30, np.zeros(31, np.int32), np.zeros(0, np.int32), np.zeros(0))
    check(A, Z, "A+0")
    check(Z, A, "0+A")


def test_tile_boundaries():
    """Long rows over several tiles (2048 merge items per tile) with matched
    pairs landing on tile and thread boundaries; runs of empty rows."""
    T = 2048
    for i, lens in enumerate([[T] * 3, [T // 2 + 1] * 7, [3 * T + 5, 0, 0, 7] * 3, [0] * 5000 + [9] * 40,
                              list(np.random.default_rng(3).integers(0, 60, 5000))]):
        n = max(lens) + 50
        A = tile_edge_matrix(lens, n=n, seed=i, mode="random")
        # B shares about half of A's keys per row (matched pairs everywhere)
        rng = np.random.default_rng(100 + i)
        keep = rng.random(A.nnz) < 0.5
        rows = A.row_ids()
        extra = tile_edge_matrix([max(0, l // 3) for l in lens], n=n, seed=200 + i, mode="random")
        keys = np.unique(np.concatenate([rows[keep] * n + A.col[keep], extra.row_ids() * n + extra.col]))
        r = keys // n
        c = (keys % n).astype(np.int32)
        rp = np.zeros(A.m + 1, dtype=np.int64)
        np.cumsum(np.bincount(r, minlength=A.m), out=rp[1:])
        B = gen.CSR(A.m, n, rp.astype(np.int32), c, gen.matrices.random_values(c.size, 7 + i))
        check(A, B, f"case {i}")
        check(B, A, f"case {i} swapped")


@pytest.mark.parametrize("mode", ["int", "random"])
def test_c1_a_plus_at(mode):
    A = gen.config("C1", mode)
    check(A, gen.transpose(A), f"C1 {mode}")


def test_c3_scaled_a_plus_at():
    A = gen.config("C3", "random", scale=1 / 16)
    check(A, gen.transpose(A), "C3/16 A+A^T")


def test_c4_scaled():
    A = gen.config("C4", "random", scale=0.1)
    check(A, gen.transpose(A), "C4/10 A+A^T")


def test_deterministic():
    A = gen.config("C3", "random", scale=1 / 64)
    B = gen.transpose(A)
    r1, c1, v1 = run(A, B)
    r2, c2, v2 = run(A, B)
    assert np.array_equal(v1.view(np.uint8), v2.view(np.uint8))


def test_fused_capacity_and_unsorted():
    """msp_spadd_fused: capacity below nnz(A) + nnz(B) is MSP_ERR_SHAPE; an
    unsorted row is MSP_ERR_INPUT (row-end and tile totals disagree) or a
    structure that differs from the oracle's, never an out-of-bounds store."""
    import torch
    from paper_conf_ipps_daltonbmog15_b200 import MspError, spadd_fused
    import ctypes
    from paper_conf_ipps_daltonbmog15_b200 import lib
    A = gen.random_csr(400, 300, 3, density=0.05)
    with pytest.raises(ValueError):   # the binding checks the capacity first
        spadd_fused(dev(A), dev(A), col=torch.empty(A.nnz, dtype=torch.int32, device="cuda"),
                    val=torch.empty(A.nnz, dtype=torch.float64, device="cuda"))
    dA = dev(A)
    a = dA.c()
    n = ctypes.c_size_t(0)
    assert lib().msp_spadd_workspace(ctypes.byref(a), ctypes.byref(a), ctypes.byref(n)) == 0
    ws = torch.zeros(int(n.value), dtype=torch.uint8, device="cuda")
    rp = torch.empty(A.m + 1, dtype=torch.int32, device="cuda")
    c = torch.empty(2 * A.nnz, dtype=torch.int32, device="cuda")
    v = torch.empty(2 * A.nnz, dtype=torch.float64, device="cuda")
    nnz = ctypes.c_int64(0)
    st = lib().msp_spadd_fused(ctypes.byref(a), ctypes.byref(a), rp.data_ptr(), c.data_ptr(), v.data_ptr(),
                               2 * A.nnz - 1, ctypes.byref(nnz), ws.data_ptr(), ws.numel(), None)
    assert st == 3  # MSP_ERR_SHAPE: capacity below nnz(A) + nnz(B)
    st = lib().msp_spadd_fused(ctypes.byref(a), ctypes.byref(a), rp.data_ptr(), c.data_ptr(), v.data_ptr(),
                               2 * A.nnz, ctypes.byref(nnz), ws.data_ptr(), ws.numel(), None)
    assert st == 0 and nnz.value == A.nnz
    bad = A.col.copy()
    r = int(np.argmax(np.diff(A.rp)))
    bad[A.rp[r]:A.rp[r + 1]] = bad[A.rp[r]:A.rp[r + 1]][::-1]
    U = gen.CSR(A.m, A.n, A.rp, bad, A.val)
    guard = 4096
    col = torch.full((2 * A.nnz + guard,), -7, dtype=torch.int32, device="cuda")
    val = torch.zeros(2 * A.nnz + guard, dtype=torch.float64, device="cuda")
    try:
        spadd_fused(dev(U), dev(A), col=col[:2 * A.nnz], val=val[:2 * A.nnz])
    except MspError as err:
        assert err.status == 6
    torch.cuda.synchronize()
    assert (col[2 * A.nnz:] == -7).all(), "store past C_capacity"
