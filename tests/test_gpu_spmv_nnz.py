"""Parity of the paper's own SpMV decomposition (SURVEY §8(f) f4(i):
nnz-only split + CSR row compaction) against the
oracle: integer mode bit-exact, random values within BJ:5's tolerance.
Cases: empty rows (compaction), rows spanning several 2048-nonzero CTA
segments (the update phase), rows ending exactly on a segment boundary,
empty matrices, and the BJ configs."""
import numpy as np
import pytest
import torch

import gen
import oracle
from tests.gpu_util import assert_spmv, dev, tile_edge_matrix

pytestmark = pytest.mark.gpu

NP = 2048  # nonzeros per CTA segment (spmv_nnz.cu)


def run(A, x):
    from paper_conf_ipps_daltonbmog15_b200 import spmv_nnz_split
    return spmv_nnz_split(dev(A), torch.as_tensor(x, device="cuda")).cpu().numpy()


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_fuzz(dtype):
    for si, (m, n) in enumerate([(1, 1), (9, 1), (37, 41), (300, 300), (1000, 17), (17, 1000)]):
        for seed in range(3):
            for kw in (dict(density=0.2), dict(density=0.05, empty_frac=0.5), dict(density=0.01, dense_rows=2),
                       dict(density=0.0)):
                A = gen.random_csr(m, n, 100 * si + seed, dtype=dtype, **kw)
                x = gen.x_vector(n, "int", dtype=dtype)
                assert np.array_equal(run(A, x), oracle.spmv(A, x)[0]), f"{m}x{n} {kw}"
                Ar = A.with_values(gen.matrices.random_values(A.nnz, seed, dtype))
                xr = gen.x_vector(n, "random", seed=seed, dtype=dtype)
                assert_spmv(Ar, xr, run(Ar, xr), label=f"{m}x{n} {kw} random")


def test_segment_boundaries():
    for i, lens in enumerate([[NP] * 3, [NP - 1, 1] * 4, [3 * NP + 5, 0, 0, 7] * 3, [0] * 5000 + [9] * 40,
                              [1] * 5000, [NP // 2 + 1] * 9, list(np.random.default_rng(1).integers(0, 60, 4000))]):
        A = tile_edge_matrix(lens, n=max(lens) + 50, seed=i)
        x = gen.x_vector(A.n, "int")
        assert np.array_equal(run(A, x), oracle.spmv(A, x)[0]), f"case {i}"


def test_empty():
    for m, n in [(0, 0), (0, 5), (5, 0), (3, 3)]:
        A = gen.CSR(m, n, np.zeros(m + 1, np.int32), np.zeros(0, np.int32), np.zeros(0))
        y = run(A, np.ones(n))
        assert y.shape == (m,) and np.all(y == 0)


@pytest.mark.parametrize("name,scale", [("C1", 1.0), ("C2", 1.0), ("C3", 1 / 16), ("C4", 1.0), ("C5", 0.02)])
def test_configs(name, scale):
    A = gen.config(name, "int", scale=scale)
    x = gen.x_vector(A.n, "int", dtype=A.val.dtype)
    assert np.array_equal(run(A, x), oracle.spmv(A, x)[0]), name
    Ar = gen.config(name, "random", scale=scale)
    xr = gen.x_vector(A.n, "random", seed=3, dtype=A.val.dtype)
    assert_spmv(Ar, xr, run(Ar, xr), label=name)
