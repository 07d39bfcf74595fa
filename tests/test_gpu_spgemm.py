"""SpGEMM parity: CUDA ESC (C ABI) vs Gustavson's dense-accumulator oracle.
Structure bit-exact (structural zeros kept, Z1); values within
1e-12 (fp64) / 1e-5 (fp32) of sum_k |a_ik||b_kj| (BJ:5, Z18); integer-valued
inputs are exact in any order, so they must match bit for bit."""
import numpy as np
import pytest

import gen
import oracle
from tests.conftest import csr_from_dense
from tests.gpu_util import dev, tile_edge_matrix

pytestmark = pytest.mark.gpu


def run(A: gen.CSR, B: gen.CSR):
    from paper_conf_ipps_daltonbmog15_b200 import SpGemmPlan
    p = SpGemmPlan(dev(A), dev(B))
    info = p.setup()
    C = p.numeric()
    rp, col, val = C.numpy()
    return rp, col, val, info


def check(A, B, label="", exact=None):
    rp, col, val, info = run(A, B)
    W, scale, npr = oracle.spgemm(A, B)
    assert info.nprods == npr, f"{label}: nprods {info.nprods} != {npr}"
    assert np.array_equal(rp, W.rp), f"{label}: row_offsets differ"
    assert np.array_equal(col, W.col), f"{label}: col_idx differ"
    ok, msg = oracle.check_values(val, W.val, scale, A.val.dtype)
    assert ok, f"{label}: {msg}"
    if exact:
        assert np.array_equal(val, W.val), f"{label}: integer mode must be exact"
    return info


def test_paper_example(paper_example):
    A = csr_from_dense(paper_example["A_dense"])
    B = csr_from_dense(paper_example["B_dense"])
    rp, col, val, info = run(A, B)
    assert info.nprods == 11
    C = gen.CSR(4, 4, rp, col, val)
    assert np.array_equal(C.dense(), np.array(paper_example["C_dense"], dtype=float))


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_fuzz(dtype):
    shapes = [(1, 1, 1), (1, 9, 4), (9, 1, 5), (13, 11, 17), (64, 64, 64), (300, 120, 250), (500, 40, 30)]
    for si, (m, k, n) in enumerate(shapes):
        for seed in range(3):
            for kw in (dict(density=0.2), dict(density=0.05, empty_frac=0.4)):
                A = gen.random_csr(m, k, 10 * si + seed, dtype=dtype, **kw)
                B = gen.random_csr(k, n, 10 * si + seed + 3, dtype=dtype, **kw)
                check(A, B, f"{m}x{k}x{n} {kw}", exact=True)
                Ar = A.with_values(gen.matrices.random_values(A.nnz, seed, dtype))
                Br = B.with_values(gen.matrices.random_values(B.nnz, seed + 1, dtype))
                check(Ar, Br, f"{m}x{k}x{n} {kw} random")


def test_structural_zero():
    A = csr_from_dense([[1.0, 1.0]])
    B = csr_from_dense([[1.0], [-1.0]])
    rp, col, val, _ = run(A, B)
    assert rp.tolist() == [0, 1] and col.tolist() == [0] and val.tolist() == [0.0]


def test_empty():
    Z = gen.CSR(5, 6, np.zeros(6, np.int32), np.zeros(0, np.int32), np.zeros(0))
    B = gen.random_csr(6, 7, 1, density=0.3)
    rp, col, val, info = run(Z, B)
    assert info.nprods == 0 and np.all(rp == 0) and col.size == 0
    A = gen.random_csr(5, 6, 2, density=0.3)
    Zb = gen.CSR(6, 7, np.zeros(7, np.int32), np.zeros(0, np.int32), np.zeros(0))
    rp, col, val, info = run(A, Zb)
    assert info.nprods == 0 and np.all(rp == 0)


def test_long_rows_and_tile_edges():
    """Rows whose items exceed T/4 (long path, several chunks and merge
    passes) next to short rows; row lengths around the snapping points."""
    n = 3000
    for i, lens in enumerate([[5] * 300 + [2500] + [5] * 300, [60] * 200, [1] * 2000 + [n] * 2 + [0] * 10,
                              list(np.random.default_rng(4).integers(0, 40, 3000))]):
        A = tile_edge_matrix(lens, n=n, seed=i)
        B = tile_edge_matrix(list(np.random.default_rng(9 + i).integers(0, 12, n)), n=n, seed=50 + i)
        info = check(A, B, f"case {i}", exact=True)
        if i == 0:  # the long row: ESC long-row pass or (narrow span) the segmented path
            assert info.long_rows + info.segmented_rows >= 1


@pytest.mark.parametrize("mode", ["int", "random"])
def test_c1(mode):
    A = gen.config("C1", mode)
    info = check(A, A, f"C1 {mode}", exact=(mode == "int"))
    assert info.nprods == 100_104


def test_c2_scaled():
    A = gen.poisson3d_27pt(30)
    A = A.with_values(gen.matrices.random_values(A.nnz, 3))
    info = check(A, A, "27pt 30^3")
    assert info.nprods == (9 * 30 - 10) ** 3


def test_c4_scaled():
    A = gen.config("C4", "int", scale=0.05)
    info = check(A, A, "C4/20", exact=True)
    assert info.long_rows >= 1


def test_c5_scaled():
    A = gen.config("C5", "random", scale=0.005)
    check(A, A, "C5/200")


def test_deterministic():
    A = gen.config("C4", "random", scale=0.02)
    _, _, v1, _ = run(A, A)
    _, _, v2, _ = run(A, A)
    assert np.array_equal(v1.view(np.uint8), v2.view(np.uint8))


def check_sampled(A, B, rows, label):
    """Full-size run in the bench's launch configuration; structure of the
    whole C checked against its closed forms / totals, sampled rows element
    by element against the oracle."""
    rp, col, val, info = run(A, B)
    off, wcol, wval, scale = oracle.spgemm_rows(A, B, rows)
    for k, r in enumerate(rows):
        a, b = int(rp[r]), int(rp[r + 1])
        lo, hi = int(off[k]), int(off[k + 1])
        assert b - a == hi - lo, f"{label}: row {r} length"
        assert np.array_equal(col[a:b], wcol[lo:hi]), f"{label}: row {r} columns"
        ok, msg = oracle.check_values(val[a:b], wval[lo:hi], scale[lo:hi], A.val.dtype)
        assert ok, f"{label}: row {r}: {msg}"
    return rp, info


def test_c2_full_sampled():
    """C2 A*A at full size (BJ:8): Nprods = 890^3, nnz(C) = 494^3."""
    A = gen.config("C2", "random")
    rows = np.unique(np.concatenate([np.arange(0, 200), np.linspace(0, A.m - 1, 300).astype(np.int64),
                                     np.arange(A.m - 200, A.m)]))
    rp, info = check_sampled(A, A, rows, "C2 full")
    assert info.nprods == 890 ** 3 and int(rp[-1]) == 494 ** 3


def test_c4_full_sampled():
    """C4 A*A at full size (BJ:10), including the 1M-nnz dense row (long-row
    path: chunk sorts + CTA merge passes) and empty rows."""
    A = gen.config("C4", "int")
    dense = int(np.argmax(np.diff(A.rp)))
    rows = np.unique(np.concatenate([[dense, dense - 1, dense + 1], np.linspace(0, A.m - 1, 400).astype(np.int64),
                                     np.arange(A.m - 50, A.m)]))
    rp, info = check_sampled(A, A, rows, "C4 full")
    assert info.long_rows >= 1 and int(rp[-1]) <= info.nprods
