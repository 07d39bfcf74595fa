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


def run(A: gen.CSR, B: gen.CSR):
    from paper_conf_ipps_daltonbmog15_b200 import spadd
    C = spadd(dev(A), dev(B))
    rp, col, val = C.numpy()
    return rp, col, val


def check(A, B, label=""):
    rp, col, val = run(A, B)
    W = oracle.spadd(A, B)
    assert np.array_equal(rp, W.rp), f"{label}: row_offsets differ"
    assert np.array_equal(col, W.col), f"{label}: col_idx differ"
    assert np.array_equal(val.view(np.uint8), W.val.view(np.uint8)), f"{label}: values differ"


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
