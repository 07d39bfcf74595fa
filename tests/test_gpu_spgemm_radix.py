"""Parity of the paper's own SpGEMM sort pipeline (SURVEY §8(f) f2:
per-tile keys-only radix by column + 16-bit permutations, global radix sort
of the reduced entries, re-expansion) against Gustavson's oracle:
structure bit-exact, values within tolerance, integer mode exact, run to run
deterministic.  Includes the paper's worked example (Fig 3) and 64-bit tile
keys (more than 21 column bits)."""
import numpy as np
import pytest

import gen
import oracle
from tests.conftest import csr_from_dense
from tests.gpu_util import dev, tile_edge_matrix

pytestmark = pytest.mark.gpu


def run(A, B):
    from paper_conf_ipps_daltonbmog15_b200 import SpGemmRadixPlan
    p = SpGemmRadixPlan(dev(A), dev(B))
    p.setup()
    p.symbolic()
    C = p.numeric()
    return C.numpy()


def check(A, B, label, exact=False):
    rp, col, val = run(A, B)
    W, sc, _ = oracle.spgemm(A, B)
    assert np.array_equal(rp, W.rp), f"{label}: row_offsets"
    assert np.array_equal(col, W.col), f"{label}: col_idx"
    ok, msg = oracle.check_values(val, W.val, sc, A.val.dtype)
    assert ok, f"{label}: {msg}"
    if exact:
        assert np.array_equal(val, W.val), f"{label}: integer mode must be exact"


def test_paper_example(paper_example):
    A = csr_from_dense(paper_example["A_dense"])
    B = csr_from_dense(paper_example["B_dense"])
    rp, col, val = run(A, B)
    C = gen.CSR(4, 4, rp, col, val)
    assert np.array_equal(C.dense(), np.array(paper_example["C_dense"], dtype=float))


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_fuzz(dtype):
    for si, (m, k, n) in enumerate([(1, 1, 1), (9, 1, 5), (13, 11, 17), (64, 64, 64), (300, 120, 250),
                                    (500, 40, 30)]):
        for seed in range(2):
            for kw in (dict(density=0.2), dict(density=0.05, empty_frac=0.4)):
                A = gen.random_csr(m, k, 10 * si + seed, dtype=dtype, **kw)
                B = gen.random_csr(k, n, 10 * si + seed + 3, dtype=dtype, **kw)
                check(A, B, f"{m}x{k}x{n} {kw}", exact=True)


def test_rows_across_tiles():
    """Rows with many more products than a 2048-product tile (duplicates
    reduced across tiles by the global phase) next to short rows."""
    for i, lens in enumerate([[5] * 300 + [2500] + [5] * 300, [60] * 200, list(np.random.default_rng(4).integers(0, 40, 3000))]):
        A = tile_edge_matrix(lens, n=3000, seed=i)
        B = tile_edge_matrix(list(np.random.default_rng(9 + i).integers(0, 12, 3000)), n=3000, seed=50 + i)
        check(A, B, f"case {i}", exact=True)


@pytest.mark.parametrize("cfg,scale", [("C1", 1.0), ("C2", 0.027), ("C4", 0.02), ("C5", 0.002)])
def test_configs(cfg, scale):
    A = gen.config(cfg, "int", scale=scale)
    check(A, A, cfg, exact=True)
    Ar = gen.config(cfg, "random", scale=scale)
    check(Ar, Ar, cfg + " random")


def test_64bit_tile_keys():
    rng = np.random.default_rng(7)
    m, k, n = 2000, 300, 1 << 22          # 22 column bits + 11 index bits > 32
    A = gen.random_csr(m, k, 1, density=0.01)
    bl = rng.integers(0, 5, k)
    rp = np.concatenate([[0], np.cumsum(bl)]).astype(np.int32)
    col = np.concatenate([np.sort(rng.choice(n, size=int(L), replace=False)) for L in bl]).astype(np.int32)
    B = gen.CSR(k, n, rp, col, gen.int_values(col.size, 2))
    check(A, B, "64-bit keys", exact=True)


def test_deterministic():
    A = gen.config("C4", "random", scale=0.01)
    v1 = run(A, A)[2]
    v2 = run(A, A)[2]
    assert np.array_equal(v1.view(np.uint8), v2.view(np.uint8))
