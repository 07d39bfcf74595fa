"""SpGEMM compare-count path for small short rows (
msp_spgemm_info.small_rows): rows with at most 64 products, in warp batches
of consecutive rows with <= 256 products; short rows with more products and
an output span wider than 65,536 columns are promoted to long rows, so the
warp-row path covers every short row.  Parity with Gustavson's oracle
(structure bit-exact, values within the BJ:5 tolerance, integer inputs and
the signed-zero case bit for bit); the round-2 behaviour (MSP_SPGEMM_SMALL=0:
one too-wide row sends every short row to the ESC tiles) stays under test in
a subprocess."""
import os
import subprocess
import sys

import numpy as np
import pytest

import gen
import oracle
from tests.gpu_util import dev
from tests.test_gpu_spgemm_rowacc import _rows, check, run

pytestmark = pytest.mark.gpu

SMALL_OFF = os.environ.get("MSP_SPGEMM_SMALL") == "0"


def _row_products(A, B):
    blen = np.diff(B.rp.astype(np.int64))
    pa = blen[A.col]
    cs = np.zeros(A.nnz + 1, np.int64)
    np.cumsum(pa, out=cs[1:])
    return cs[A.rp[1:]] - cs[A.rp[:-1]]


@pytest.mark.skipif(SMALL_OFF, reason="small path disabled")
def test_random_rows_c5_shape():
    """C5's structure (BJ:11) at 3*10^5 rows: row length uniform in 0..8,
    uniform random columns -- every row has <= 64 products and a span of
    ~all columns, so every row with products takes the small path."""
    A = gen.random_rows(300_000, seed=21)
    P = _row_products(A, A)
    for mode, Am in (("int", A.with_values(gen.int_values(A.nnz, 22))), ("random", A)):
        info = check(Am, Am, f"C5-shape {mode}", exact=(mode == "int"))
        assert info.ntiles == 0 and info.long_rows == 0
        assert info.small_rows == int(np.count_nonzero((P > 0) & (P <= 64)))
        assert info.bitmap_rows == 0
    A32 = A.with_values(A.val.astype(np.float32))
    check(A32, A32, "C5-shape fp32")


@pytest.mark.skipif(SMALL_OFF, reason="small path disabled")
def test_duplicates_batches_and_many_a_nonzeros():
    """Few columns (many duplicate products summed in k order), rows with
    exactly 64 products next to each other (batches split at 256), rows with
    more than 32 A nonzeros whose B rows are mostly empty (the expansion's
    A-nonzero chunks), empty rows in between."""
    rng = np.random.default_rng(5)
    k, n = 500, 40
    blens = np.where(rng.random(k) < 0.6, 0, rng.integers(1, 9, k))
    Brp, Bcol = _rows(blens, n, rng)
    B = gen.CSR(k, n, Brp, Bcol, gen.matrices.random_values(Bcol.size, 6))
    nz = np.flatnonzero(blens > 0)
    rows_c, rows_l = [], []
    for i in range(3000):
        kind = i % 5
        if kind == 0:
            cols = np.array([], np.int64)
        elif kind == 1:  # exactly 64 products: 8 B rows of length 8
            full = np.flatnonzero(blens == 8)
            cols = np.sort(rng.choice(full, size=min(8, full.size), replace=False))
        elif kind == 2:  # > 32 A nonzeros, mostly empty B rows
            cols = np.sort(rng.choice(k, size=45, replace=False))
        else:
            cols = np.sort(rng.choice(nz, size=int(rng.integers(1, 7)), replace=False))
        rows_c.append(cols)
        rows_l.append(cols.size)
    Arp = np.zeros(len(rows_l) + 1, np.int64)
    np.cumsum(rows_l, out=Arp[1:])
    Acol = np.concatenate(rows_c).astype(np.int32)
    A = gen.CSR(len(rows_l), k, Arp.astype(np.int32), Acol, gen.matrices.random_values(Acol.size, 7))
    P = _row_products(A, B)
    small = (P > 0) & (P <= 64)
    info = check(A, B, "duplicates")
    assert info.small_rows == int(np.count_nonzero(small))
    assert (P[small] == 64).sum() > 100
    Ai = A.with_values(gen.int_values(A.nnz, 8))
    Bi = B.with_values(gen.int_values(B.nnz, 9))
    check(Ai, Bi, "duplicates int", exact=True)
    check(A.with_values(A.val.astype(np.float32)), B.with_values(B.val.astype(np.float32)), "duplicates fp32")


@pytest.mark.skipif(SMALL_OFF, reason="small path disabled")
def test_mixed_small_bitmap_promoted_long():
    """One matrix with every short-row mode: small rows, rows with > 64
    products inside a 60,000-column span (bitmap), rows with 120 products
    spanning 10^6 columns (small: <= 256 products), rows with 300 products
    spanning 10^6 columns (promoted to long), and rows longer than a tile
    (long from the start)."""
    rng = np.random.default_rng(9)
    n = 1_000_000
    # B rows: 0..99 narrow (cols < 60000, length 10), 100..199 wide (length 10), 200 very long
    brows = [np.sort(rng.choice(60_000, 10, replace=False)) for _ in range(100)]
    brows += [np.sort(rng.choice(n, 10, replace=False)) for _ in range(100)]
    brows += [np.sort(rng.choice(n, 5000, replace=False))]
    Brp = np.zeros(len(brows) + 1, np.int64)
    np.cumsum([b.size for b in brows], out=Brp[1:])
    B = gen.CSR(len(brows), n, Brp.astype(np.int32), np.concatenate(brows).astype(np.int32),
                gen.matrices.random_values(int(Brp[-1]), 10))
    arows = []
    for i in range(2000):
        kind = i % 5
        if kind == 0:
            arows.append(np.sort(rng.choice(200, int(rng.integers(1, 6)), replace=False)))  # small
        elif kind == 1:
            arows.append(np.sort(rng.choice(100, 12, replace=False)))  # 120 products, narrow: bitmap
        elif kind == 2:
            arows.append(np.sort(rng.choice(np.arange(100, 200), 30, replace=False)))  # 300, wide: promoted
        elif kind == 3:
            arows.append(np.sort(rng.choice(np.arange(100, 200), 12, replace=False)))  # 120, wide: small
        else:
            arows.append(np.array([200]) if i % 400 == 4 else np.array([], np.int64))  # long / empty
    Arp = np.zeros(len(arows) + 1, np.int64)
    np.cumsum([a.size for a in arows], out=Arp[1:])
    Acol = np.concatenate(arows).astype(np.int32)
    A = gen.CSR(len(arows), B.m, Arp.astype(np.int32), Acol, gen.matrices.random_values(Acol.size, 11))
    info = check(A, B, "mixed")
    assert info.small_rows == 800 and info.bitmap_rows == 400
    assert info.long_rows == 400 + 5 and info.ntiles == 0
    check(A.with_values(gen.int_values(A.nnz, 12)), B.with_values(gen.int_values(B.nnz, 13)), "mixed int",
          exact=True)


@pytest.mark.skipif(SMALL_OFF, reason="small path disabled")
def test_wide_rows_taken():
    """The case that disabled the row path in v5 (one short row spanning
    more than 65,536 columns) now takes the small path."""
    rng = np.random.default_rng(3)
    n = 200_000
    B = gen.CSR(3, n, np.array([0, 2, 3, 4], np.int32), np.array([0, 150_000, 7, 9], np.int32), np.ones(4))
    A = gen.CSR(50, 3, *_rows(rng.integers(1, 3, 50), 3, rng), None)
    A = A.with_values(np.ones(A.col.size))
    info = check(A, B, "wide span", exact=True)
    assert info.row_accumulator > 0 and info.ntiles == 0 and info.small_rows == 50


@pytest.mark.skipif(SMALL_OFF, reason="already the small-off run")
def test_small_path_off_suite():
    """MSP_SPGEMM_SMALL=0: the v5 classification (bitmap or, if any row is
    too wide, ESC tiles for every short row) on the row-accumulator suite."""
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, MSP_SPGEMM_SMALL="0")
    r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-m", "gpu",
                        "tests/test_gpu_spgemm_rowacc.py", "tests/test_gpu_spgemm_small.py"],
                       cwd=root, env=env, capture_output=True, text=True, timeout=1800)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-2000:]
