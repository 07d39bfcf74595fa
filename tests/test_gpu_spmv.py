"""SpMV parity: CUDA path (C ABI) vs the CPU oracle, element by element.

Tolerance (BJ:5): |y_gpu - y| <= tau * sum_j |a_ij||x_j|, tau = 1e-12 (fp64)
or 1e-5 (fp32); integer-valued inputs are exact in any summation order
 so they must match bit for bit."""
import numpy as np
import pytest
import torch

import gen
import oracle
from tests.conftest import csr_from_dense
from tests.gpu_util import assert_spmv, dev, tile_edge_matrix

pytestmark = pytest.mark.gpu

T_F64 = 256 * 8     # merge items per tile of the fp64 kernel (spmv.cu Cfg)


def run(A: gen.CSR, x: np.ndarray) -> np.ndarray:
    from paper_conf_ipps_daltonbmog15_b200 import spmv
    Ad = dev(A)
    y = spmv(Ad, torch.as_tensor(x, device="cuda"))
    return y.cpu().numpy()


def test_paper_example(paper_example):
    A = csr_from_dense(paper_example["A_dense"])
    y = run(A, np.ones(4))
    assert y.tolist() == [10.0, 90.0, 50.0, 60.0]


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_fuzz_small(dtype):
    shapes = [(1, 1), (1, 9), (9, 1), (5, 7), (37, 41), (300, 300), (1000, 17), (17, 1000)]
    for si, (m, n) in enumerate(shapes):
        for seed in range(3):
            for kw in (dict(density=0.2), dict(density=0.05, empty_frac=0.5),
                       dict(density=0.01, dense_rows=2), dict(density=0.0)):
                A = gen.random_csr(m, n, 100 * si + seed, dtype=dtype, **kw)
                x = gen.x_vector(n, "int", dtype=dtype)
                y = run(A, x)
                assert_spmv(A, x, y, label=f"{m}x{n} {kw}")
                assert np.array_equal(y, oracle.spmv(A, x)[0]), "integer mode must be exact"


def test_empty_shapes():
    for m, n in [(0, 0), (0, 5), (5, 0), (3, 3)]:
        A = gen.CSR(m, n, np.zeros(m + 1, np.int32), np.zeros(0, np.int32), np.zeros(0))
        y = run(A, np.ones(n))
        assert y.shape == (m,) and np.all(y == 0)


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_tile_boundaries(dtype):
    """Row ends exactly on, before and after tile boundaries; rows spanning 1,
    2 and many tiles; runs of empty rows across a boundary (Z21, H2)."""
    T = T_F64
    cases = [
        [T - 1] * 6,                         # row + its row-end item = one tile
        [T] * 5, [T + 1] * 5, [T - 2] * 5,
        [0] * 3000 + [5] * 10 + [0] * 5000,  # empty runs spanning tiles
        [3 * T + 17, 0, 0, 1, 2 * T, 0] * 3,
        [20 * T + 5],                        # one row over many tiles / CTAs
        list(np.random.default_rng(5).integers(0, 40, 20000)),
    ]
    for i, lens in enumerate(cases):
        for mode in ("int", "random"):
            A = tile_edge_matrix(lens, n=max(64, max(lens) + 7), seed=i, dtype=dtype, mode=mode)
            x = gen.x_vector(A.n, mode, seed=7, dtype=dtype)
            assert_spmv(A, x, run(A, x), label=f"case {i} {mode}")


@pytest.mark.parametrize("mode", ["int", "random"])
def test_c1_c2(mode):
    for name in ("C1", "C2"):
        A = gen.config(name, mode)
        x = gen.x_vector(A.n, mode, seed=1000 + int(name[1]), dtype=A.val.dtype)
        y = run(A, x)
        assert_spmv(A, x, y, label=f"{name} {mode}")
        if mode == "int":
            assert np.array_equal(y, oracle.spmv(A, x)[0])


def test_c3_scaled_fp32():
    A = gen.config("C3", "random", scale=1 / 16)        # R-MAT scale 18, same recipe
    x = gen.x_vector(A.n, "random", seed=1003, dtype=np.float32)
    assert_spmv(A, x, run(A, x), label="C3/16 fp32")
    Ai = gen.config("C3", "int", scale=1 / 16)
    xi = gen.x_vector(A.n, "int", dtype=np.float32)
    assert np.array_equal(run(Ai, xi), oracle.spmv(Ai, xi)[0])


def test_c4_full():
    A = gen.config("C4", "int")
    x = gen.x_vector(A.n, "int")
    y = run(A, x)
    assert np.array_equal(y, oracle.spmv(A, x)[0])
    # the dense row equals a single dot product
    r = 1_000_003
    a, b = A.rp[r], A.rp[r + 1]
    assert y[r] == float(np.dot(A.val[a:b], x[A.col[a:b]]))
    Ar = gen.config("C4", "random")
    xr = gen.x_vector(A.n, "random", seed=1004)
    assert_spmv(Ar, xr, run(Ar, xr), label="C4 random")


def test_c5_scaled():
    A = gen.config("C5", "random", scale=0.02)          # 2M rows, same recipe
    x = gen.x_vector(A.n, "random", seed=1005)
    assert_spmv(A, x, run(A, x), label="C5/50")


def test_deterministic():
    A = gen.config("C4", "random", scale=0.25)
    x = gen.x_vector(A.n, "random", seed=3)
    y1, y2 = run(A, x), run(A, x)
    assert np.array_equal(y1.view(np.int64), y2.view(np.int64))


def test_fp32_long_row_accumulates_in_fp64():
    """Z4 pin on the GPU: 2^24 followed by 4096 ones in one fp32 row."""
    n = 4097
    A = gen.CSR(1, n, np.array([0, n], np.int32), np.arange(n, dtype=np.int32),
                np.concatenate([[2.0 ** 24], np.ones(n - 1)]).astype(np.float32))
    y = run(A, np.ones(n, np.float32))
    assert y[0] == np.float32(2.0 ** 24 + 4096)


@pytest.mark.parametrize("L", [3, 5, 7, 27])
def test_cta_boundary_before_row_end(L):
    """Uniform rows of L nonzeros: the persistent grid's diagonal split
    b*(m+nnz)/G falls, for about one CTA in L+1, between a row's last nonzero
    and its row-end item, so the CTA's trailing partial belongs to a row whose
    end the next CTA consumes first (Z21: carries are (row, partial) pairs)."""
    for m in (150_001, 200_003, 333_331):
        n = m
        rp = (np.arange(m + 1, dtype=np.int64) * L).astype(np.int32)
        col = np.tile((np.arange(L) * (n // L)).astype(np.int32), m)  # sorted, distinct per row
        val = gen.int_values(m * L, L)
        A = gen.CSR(m, n, rp, col, val)
        x = gen.x_vector(n, "int")
        y = run(A, x)
        assert np.array_equal(y, oracle.spmv(A, x)[0]), f"m={m} L={L}"


def test_warp_tiles_long_rows():
    """The warp-tile kernel (chosen when the mean row length is >= 20) on rows
    that span many warp tiles and CTAs next to stencil-length rows and empty
    rows: the decoupled look-back over tiles without row ends must give the
    exact result, run to run (a record upgraded in place once let a reader
    take an inclusive carry for an aggregate)."""
    rng = np.random.default_rng(11)
    for i, lens in enumerate([[27] * 5000 + [200_000] + [27] * 5000,
                              [300_000] + list(rng.choice([0, 27, 27, 27, 3000], 20_000)),
                              list(rng.integers(0, 3000, 400))]):
        n = 400_000
        g = np.random.default_rng(20 + i)
        cols = [np.unique(g.integers(0, n, int(L) + int(L) // 8 + 4))[:int(L)] for L in lens]
        lens = [c.size for c in cols]
        rp = np.concatenate([[0], np.cumsum(lens)]).astype(np.int32)
        col = np.concatenate(cols).astype(np.int32)
        A = gen.CSR(len(lens), n, rp, col, gen.int_values(col.size, 30 + i))
        assert A.nnz >= 20 * A.m  # the warp-tile path
        x = gen.x_vector(A.n, "int")
        want = oracle.spmv(A, x)[0]
        for _ in range(3):
            assert np.array_equal(run(A, x), want), f"case {i}"
