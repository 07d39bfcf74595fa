"""Closed forms of the Poisson stencils pinning the oracle
and the generators of C1/C2.  The 27-point pattern is P1 (x) P1 (x) P1 with
P1 the k x k tridiagonal pattern, so for a k^3 grid: nnz = (3k-2)^3,
Nprods(A*A) = (9k-10)^3, nnz(A*A) = (5k-6)^3 (pentadiagonal P1^2).  For the
5-point k x k stencil: nnz = 5k^2 - 4k."""
import numpy as np
import pytest

import gen
import oracle


def test_c1_closed_forms():
    A = gen.config("C1")
    k = 64
    assert A.m == 4096 and A.nnz == 5 * k * k - 4 * k == 20224
    lens = np.diff(A.rp)
    assert set(lens.tolist()) == {3, 4, 5}
    y, _ = oracle.spmv(A, np.ones(A.n))
    vals, cnt = np.unique(y, return_counts=True)
    assert dict(zip(vals.tolist(), cnt.tolist())) == {0.0: 3844, 1.0: 248, 2.0: 4}
    C, _, npr = oracle.spgemm(A, A)
    assert npr == 100_104 and C.nnz == 51_972
    assert set(np.unique(C.val).tolist()) == {-8.0, 1.0, 2.0, 18.0, 19.0, 20.0}
    diag = C.dense().diagonal()
    assert np.array_equal(diag, 16 + (lens - 1))          # 16 + degree
    T = gen.transpose(A)
    S = oracle.spadd(A, T)                                # Poisson A + A^T = 2A
    assert np.array_equal(S.col, A.col) and np.array_equal(S.val, 2 * A.val)


@pytest.mark.parametrize("k", [2, 3, 7, 20])
def test_27pt_closed_forms(k):
    A = gen.poisson3d_27pt(k)
    assert A.nnz == (3 * k - 2) ** 3
    assert oracle.nprods(A, A) == (9 * k - 10) ** 3
    lens = np.diff(A.rp)
    y, s = oracle.spmv(A, np.ones(A.n))
    assert np.array_equal(y, 27.0 - lens)                 # A*1 = 26 - (len - 1)
    assert np.array_equal(s, 25.0 + lens)                 # 26 + (len - 1)
    C, _, npr = oracle.spgemm(A, A, with_scale=False)
    assert npr == (9 * k - 10) ** 3
    assert C.nnz == (5 * k - 6) ** 3


def test_c2_sizes():
    """Full C2 sizes (SURVEY size sheet): nnz = 298^3, Nprods = 890^3; row
    lengths {8, 12, 18, 27}; A*1 histogram."""
    A = gen.poisson3d_27pt(100)
    assert A.nnz == 298 ** 3 == 26_463_592
    assert oracle.nprods(A, A) == 890 ** 3 == 704_969_000
    lens = np.diff(A.rp)
    assert set(np.unique(lens).tolist()) == {8, 12, 18, 27}
    y, _ = oracle.spmv(A, np.ones(A.n))
    vals, cnt = np.unique(y, return_counts=True)
    assert dict(zip(vals.tolist(), cnt.tolist())) == {0.0: 941_192, 9.0: 57_624,
                                                      15.0: 1_176, 19.0: 8}


def test_row_split_oracle_vs_model():
    from oracle.partition_model import row_split as model_split
    for A in (gen.config("C1"), gen.random_csr(300, 50, 1, density=0.05, empty_frac=0.3)):
        for P in (1, 2, 3, 4, 8):
            s = oracle.row_split(A.rp, P)
            assert np.array_equal(s, model_split(A.rp, P))
            assert s[0] == 0 and s[-1] == A.m and np.all(np.diff(s) >= 0)
