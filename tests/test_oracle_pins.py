"""Pins of the CPU oracle against values that do not come from the oracle
itself: the paper's worked example (tests/golden, cited there), dense brute
force on integer matrices (exact), algebraic identities, and scipy as a third
opinion on positive matrices.  All CPU-only (-m "not gpu").
"""
import numpy as np
import pytest
import scipy.sparse as sp

import gen
import oracle
from tests.conftest import csr_from_dense, csr_from_tuples


def _sp(A):
    return sp.csr_matrix((A.val.astype(np.float64), A.col, A.rp), shape=(A.m, A.n))


# ---------------------------------------------------------------- paper example

def test_paper_example_spgemm(paper_example):
    """C = A x B as printed at P:880-884; Nprods = 11 products;
    the 8 reduced tuples of P:868-874 are exactly C's CSR entries."""
    A = csr_from_dense(paper_example["A_dense"])
    B = csr_from_dense(paper_example["B_dense"])
    # tuple forms printed at P:338-354 describe the same matrices
    At = csr_from_tuples(paper_example["A_tuples"], 4, 4)
    Bt = csr_from_tuples(paper_example["B_tuples"], 4, 4)
    for X, Y in ((A, At), (B, Bt)):
        assert np.array_equal(X.rp, Y.rp) and np.array_equal(X.col, Y.col)
        assert np.array_equal(X.val, Y.val)
    C, scale, npr = oracle.spgemm(A, B)
    assert npr == paper_example["nprods"] == len(paper_example["products_paper_order"])
    assert np.array_equal(C.dense(), np.array(paper_example["C_dense"], dtype=float))
    got = [[int(r), int(c), float(v)] for r, c, v in zip(C.row_ids(), C.col, C.val)]
    assert got == [[r, c, float(v)] for r, c, v in paper_example["reduced"]]
    # the sorted product list reduces (sum of equal keys) to the same tuples
    red = {}
    for r, c, v in paper_example["products_sorted"]:
        red[(r, c)] = red.get((r, c), 0) + v
    assert sorted([k[0], k[1], v] for k, v in red.items()) == paper_example["reduced"]
    # products_sorted is a permutation of products_paper_order
    assert sorted(map(tuple, paper_example["products_sorted"])) == \
        sorted(map(tuple, paper_example["products_paper_order"]))
    assert oracle.nprods(A, B) == 11


def test_paper_example_spmv_spadd(paper_example):
    A = csr_from_dense(paper_example["A_dense"])
    B = csr_from_dense(paper_example["B_dense"])
    one = np.ones(4)
    y, s = oracle.spmv(A, one)
    assert y.tolist() == [10.0, 90.0, 50.0, 60.0]           # row sums of P:330-336
    y, s = oracle.spmv(B, one)
    assert y.tolist() == [1.0, 5.0, 9.0, 13.0]
    C = oracle.spadd(A, B)
    want = np.array(paper_example["A_dense"]) + np.array(paper_example["B_dense"])
    assert np.array_equal(C.dense(), want)
    assert C.nnz == 9
    At = gen.transpose(A)
    assert oracle.spadd(A, At).nnz == 8


# ---------------------------------------------------------------- brute force

SHAPES = [(0, 0, 0), (1, 1, 1), (1, 7, 5), (7, 1, 3), (5, 6, 7), (13, 11, 17), (40, 33, 29),
          (64, 64, 64), (3, 200, 2)]


def _rand(m, n, seed, dtype=np.float64, **kw):
    kw.setdefault("density", 0.25)
    return gen.random_csr(m, n, seed, dtype=dtype, **kw)


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
@pytest.mark.parametrize("shape", SHAPES)
def test_bruteforce_spmv(shape, dtype):
    m, k, _ = shape
    for seed in range(3):
        A = _rand(m, k, seed, dtype, empty_frac=0.2, dense_rows=1 if m > 3 else 0)
        x = gen.x_vector(k, "int", dtype=dtype)
        y, s = oracle.spmv(A, x)
        d = A.dense()
        assert np.array_equal(y.astype(np.float64), d @ x.astype(np.float64))
        assert np.array_equal(s, np.abs(d) @ np.abs(x.astype(np.float64)))
        assert y.dtype == dtype


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
@pytest.mark.parametrize("shape", SHAPES)
def test_bruteforce_spadd(shape, dtype):
    m, n, _ = shape
    for seed in range(3):
        A = _rand(m, n, seed, dtype, empty_frac=0.1)
        B = _rand(m, n, seed + 100, dtype, density=0.3)
        C = oracle.spadd(A, B)
        pa, pb = A.dense() != 0, B.dense() != 0
        pc = np.zeros((m, n), dtype=bool)
        if C.nnz:
            pc[C.row_ids(), C.col] = True
        assert np.array_equal(pc, pa | pb)                 # structure = symbolic union
        assert np.array_equal(C.dense(), A.dense() + B.dense())
        assert np.all(np.diff(C.rp) >= 0)
        for i in range(m):                                 # columns sorted, unique
            cs = C.col[C.rp[i]:C.rp[i + 1]]
            assert np.all(np.diff(cs) > 0)


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
@pytest.mark.parametrize("shape", SHAPES)
def test_bruteforce_spgemm(shape, dtype):
    m, k, n = shape
    for seed in range(3):
        A = _rand(m, k, seed, dtype, empty_frac=0.2)
        B = _rand(k, n, seed + 50, dtype, density=0.3, empty_frac=0.1)
        C, scale, npr = oracle.spgemm(A, B)
        Pa = (A.dense() != 0).astype(np.int64)
        Pb = (B.dense() != 0).astype(np.int64)
        struct = (Pa @ Pb) > 0
        pc = np.zeros((m, n), dtype=bool)
        if C.nnz:
            pc[C.row_ids(), C.col] = True
        assert np.array_equal(pc, struct)                  # structural zeros kept (Z1)
        assert np.array_equal(C.dense(), A.dense() @ B.dense())
        assert npr == int(Pa.sum(axis=0) @ Pb.sum(axis=1))   # sum_k nnz(A[:,k]) nnz(B[k,:])
        assert npr == oracle.nprods(A, B)
        absd = np.abs(A.dense()) @ np.abs(B.dense())
        if C.nnz:
            assert np.array_equal(scale, absd[C.row_ids(), C.col])
        for i in range(m):
            cs = C.col[C.rp[i]:C.rp[i + 1]]
            assert np.all(np.diff(cs) > 0)


def test_structural_zero_kept():
    """[[1, 1]] x [[1], [-1]] has one structural entry with value 0 (Z1);
    scipy drops it, the oracle must keep it."""
    A = csr_from_dense([[1.0, 1.0]])
    B = csr_from_dense([[1.0], [-1.0]])
    C, _, npr = oracle.spgemm(A, B)
    assert C.nnz == 1 and C.val[0] == 0.0 and npr == 2
    assert (_sp(A) @ _sp(B)).nnz == 0
    D = oracle.spadd(A, A.with_values(-A.val))
    assert D.nnz == 2 and np.all(D.val == 0.0)


# ---------------------------------------------------------------- identities

@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_identities(dtype):
    for seed in range(4):
        A = gen.random_csr(37, 37, seed, density=0.15, mode="random", dtype=dtype, empty_frac=0.1)
        B = gen.random_csr(37, 37, seed + 9, density=0.2, mode="random", dtype=dtype)
        I = gen.identity(37, dtype)
        for C in (oracle.spgemm(A, I)[0], oracle.spgemm(I, A)[0]):   # A I = I A = A, bitwise
            assert np.array_equal(C.rp, A.rp) and np.array_equal(C.col, A.col)
            assert np.array_equal(C.val, A.val)
        Z = gen.CSR(37, 37, np.zeros(38, np.int32), np.zeros(0, np.int32), np.zeros(0, dtype))
        C = oracle.spadd(A, Z)                                       # A + 0 = A
        assert np.array_equal(C.col, A.col) and np.array_equal(C.val, A.val)
        C1, C2 = oracle.spadd(A, B), oracle.spadd(B, A)               # A + B = B + A
        assert np.array_equal(C1.rp, C2.rp) and np.array_equal(C1.col, C2.col)
        assert np.array_equal(C1.val, C2.val)
        N = oracle.spadd(A, A.with_values(-A.val))                   # A + (-A)
        assert np.array_equal(N.col, A.col) and np.all(N.val == 0)
        for j in (0, 5, 36):                                         # A e_j = column j
            e = np.zeros(37, dtype=dtype); e[j] = 1
            y, _ = oracle.spmv(A, e)
            assert np.array_equal(y, A.dense()[:, j].astype(dtype))


def test_linearity_int_mode():
    for seed in range(4):
        A = gen.random_csr(50, 40, seed, density=0.2)
        B = gen.random_csr(50, 40, seed + 1, density=0.2)
        Bk = gen.random_csr(40, 30, seed + 2, density=0.2)
        x = gen.x_vector(40)
        z = gen.x_vector(30)
        ab, _ = oracle.spmv(oracle.spadd(A, B), x)
        assert np.array_equal(ab, oracle.spmv(A, x)[0] + oracle.spmv(B, x)[0])   # (A+B)x
        C, _, _ = oracle.spgemm(A, Bk)
        assert np.array_equal(oracle.spmv(C, z)[0], oracle.spmv(A, oracle.spmv(Bk, z)[0])[0])


# ---------------------------------------------------------------- scipy, rows

def test_scipy_third_opinion_positive():
    for seed in range(3):
        A = gen.random_csr(120, 90, seed, density=0.05, mode="random")
        A = A.with_values(np.abs(A.val) + 0.5)
        B = gen.random_csr(90, 70, seed + 3, density=0.08, mode="random")
        B = B.with_values(np.abs(B.val) + 0.5)
        C, _, _ = oracle.spgemm(A, B)
        S = (_sp(A) @ _sp(B)).tocsr(); S.sort_indices()
        assert np.array_equal(C.rp, S.indptr) and np.array_equal(C.col, S.indices)
        assert np.allclose(C.val, S.data, rtol=1e-14)
        At = gen.transpose(A)
        St = _sp(A).T.tocsr(); St.sort_indices()
        assert np.array_equal(At.rp, St.indptr) and np.array_equal(At.col, St.indices)
        D = oracle.spadd(A, A.with_values(A.val * 2))
        assert np.array_equal(D.val, A.val * 3)


def test_row_subsets_match_full():
    A = gen.random_csr(80, 60, 3, density=0.1, mode="random", empty_frac=0.2)
    B = gen.random_csr(60, 50, 4, density=0.1, mode="random")
    B2 = gen.random_csr(80, 60, 5, density=0.1, mode="random")
    rows = np.array([79, 0, 13, 13, 41], dtype=np.int32)
    x = gen.x_vector(60, "random")
    y, s = oracle.spmv(A, x)
    yr, sr = oracle.spmv(A, x, rows)
    assert np.array_equal(yr, y[rows]) and np.array_equal(sr, s[rows])
    C, sc, _ = oracle.spgemm(A, B)
    off, col, val, scl = oracle.spgemm_rows(A, B, rows)
    for q, r in enumerate(rows):
        a, b = C.rp[r], C.rp[r + 1]
        assert np.array_equal(col[off[q]:off[q + 1]], C.col[a:b])
        assert np.array_equal(val[off[q]:off[q + 1]], C.val[a:b])
        assert np.array_equal(scl[off[q]:off[q + 1]], sc[a:b])
    D = oracle.spadd(A, B2)
    off, col, val = oracle.spadd_rows(A, B2, rows)
    for q, r in enumerate(rows):
        a, b = D.rp[r], D.rp[r + 1]
        assert np.array_equal(col[off[q]:off[q + 1]], D.col[a:b])
        assert np.array_equal(val[off[q]:off[q + 1]], D.val[a:b])


def test_fp32_accumulates_in_fp64():
    """Z4: fp32 SpMV rounds once from an fp64 accumulator.  A row where
    sequential fp32 summation loses the small terms pins the precision."""
    n = 4097
    A = gen.CSR(1, n, np.array([0, n], np.int32), np.arange(n, dtype=np.int32),
                np.concatenate([[2.0 ** 24], np.ones(n - 1)]).astype(np.float32))
    x = np.ones(n, dtype=np.float32)
    y, s = oracle.spmv(A, x)
    assert y[0] == np.float32(2.0 ** 24 + 4096)         # fp32 sequential would give 2^24
    C, _, _ = oracle.spgemm(A, gen.CSR(n, 1, np.arange(n + 1, dtype=np.int32),
                                       np.zeros(n, np.int32), np.ones(n, np.float32)))
    assert C.val[0] == np.float32(2.0 ** 24 + 4096)
