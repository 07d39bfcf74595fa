"""SpGEMM fuzz across every row path: random shapes,
row-length mixes and column ranges chosen so that one run touches the small
rows (compare-count), the bitmap accumulator, rows promoted to the ESC
long-row pass, narrow and windowed segmented rows and long rows, in fp64
and fp32, integer values (bit-exact) and random values (BJ:5 tolerance),
against Gustavson's oracle."""
import numpy as np
import pytest

import gen
import oracle
from tests.gpu_util import dev

pytestmark = pytest.mark.gpu


def _csr(m, n, lens, rng, mode, dtype, seed, hot=None):
    rows = []
    for L in lens:
        if L <= 0:
            rows.append(np.zeros(0, np.int64))
            continue
        if hot is not None and rng.random() < 0.3:  # clustered columns (bitmap / segmented spans)
            lo = int(rng.integers(0, max(1, n - hot)))
            rows.append(np.unique(rng.integers(lo, min(n, lo + hot), int(L))))
        else:
            rows.append(np.unique(rng.integers(0, n, int(L))))
    rp = np.zeros(m + 1, np.int64)
    np.cumsum([r.size for r in rows], out=rp[1:])
    col = np.concatenate(rows).astype(np.int32) if rows else np.zeros(0, np.int32)
    val = (gen.int_values(col.size, seed, dtype) if mode == "int"
           else gen.matrices.random_values(col.size, seed, dtype))
    return gen.CSR(m, n, rp.astype(np.int32), col, val)


def _lens(count, rng):
    kind = rng.integers(0, 4)
    if kind == 0:
        L = rng.integers(0, 4, count)
    elif kind == 1:
        L = rng.integers(0, 12, count)
    elif kind == 2:
        L = rng.integers(0, 40, count)
    else:
        L = np.where(rng.random(count) < 0.05, rng.integers(200, 3000, count), rng.integers(0, 8, count))
    L[rng.random(count) < 0.1] = 0
    return L


@pytest.mark.parametrize("seed", range(12))
def test_spgemm_fuzz(seed):
    from paper_conf_ipps_daltonbmog15_b200 import SpGemmPlan
    rng = np.random.default_rng(1000 + seed)
    m = int(rng.integers(1, 2500))
    k = int(rng.integers(1, 1500))
    n = int(rng.choice([40, 3000, 70_000, 2_000_000]))
    mode = "int" if seed % 2 == 0 else "random"
    dtype = np.float32 if seed % 3 == 2 else np.float64
    hot = int(rng.choice([64, 1000, 20_000, 60_000]))
    A = _csr(m, k, _lens(m, rng), rng, mode, dtype, seed + 1)
    B = _csr(k, n, _lens(k, rng), rng, mode, dtype, seed + 2, hot=hot)
    p = SpGemmPlan(dev(A), dev(B))
    p.setup()
    C = p.numeric()
    rp, col, val = C.numpy()
    W, scale, npr = oracle.spgemm(A, B)
    info = p.info
    label = (f"seed {seed}: m={m} k={k} n={n} {mode} {np.dtype(dtype).name} small={info.small_rows} "
             f"bitmap={info.bitmap_rows} long={info.long_rows} seg={info.segmented_rows} tiles={info.ntiles}")
    assert info.nprods == npr, label
    assert np.array_equal(rp, W.rp), label + ": row offsets"
    assert np.array_equal(col, W.col), label + ": columns"
    if mode == "int":
        assert np.array_equal(val, W.val), label + ": integer values must be exact"
    else:
        ok, msg = oracle.check_values(val, W.val, scale, dtype)
        assert ok, label + ": " + msg
