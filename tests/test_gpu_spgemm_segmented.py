"""The segmented (row-wise dense accumulator) SpGEMM path (
the paper's future work, for the Dense-like rows its ESC failed
on): long rows whose output spans <= 12288 columns with >= 1
product per 4 columns are accumulated in shared memory in A's column order
-- the oracle's order -- so they match Gustavson bit for bit even with random
values.  Checked against the oracle with the path on and (subprocess, env
MSP_SPGEMM_SEGMENTED=0) off, next to short rows and a wide long row that
stays on the ESC long-row pass."""
import os
import subprocess
import sys

import numpy as np
import pytest

import gen
import oracle
from tests.gpu_util import dev

pytestmark = pytest.mark.gpu


def run(A, B):
    from paper_conf_ipps_daltonbmog15_b200 import SpGemmPlan
    p = SpGemmPlan(dev(A), dev(B))
    info = p.setup()
    C = p.numeric()
    return C.numpy(), info


def dense(n, seed, dtype=np.float64, mode="random"):
    g = np.random.default_rng(seed)
    rp = (np.arange(n + 1, dtype=np.int64) * n).astype(np.int32)
    col = np.tile(np.arange(n, dtype=np.int32), n)
    val = g.uniform(-1, 1, n * n).astype(dtype) if mode == "random" else gen.int_values(n * n, seed, dtype)
    return gen.CSR(n, n, rp, col, val)


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_dense_rows_bit_exact(dtype):
    A = dense(300, 1, dtype)
    (rp, col, val), info = run(A, A)
    assert info.segmented_rows == 300 and info.long_rows == 0
    W, sc, _ = oracle.spgemm(A, A)
    assert np.array_equal(rp, W.rp) and np.array_equal(col, W.col)
    assert np.array_equal(val, W.val), "same summation order as the oracle: bit-exact"


def mixed(seed):
    """short rows, narrow-span long rows (segmented), a wide long row (ESC)"""
    g = np.random.default_rng(seed)
    n = 200_000
    rows = []
    for r in range(3000):
        if r % 500 == 7:      # narrow span: columns in [0, 3000), B rows there are long
            rows.append(np.unique(g.integers(0, 3000, 400)))
        elif r == 1500:       # wide span: ESC long-row pass
            rows.append(np.unique(g.integers(0, n, 60_000)))
        else:
            rows.append(np.unique(g.integers(0, n, 5)))
    rp = np.concatenate([[0], np.cumsum([x.size for x in rows])]).astype(np.int32)
    A = gen.CSR(3000, n, rp, np.concatenate(rows).astype(np.int32), gen.matrices.random_values(int(rp[-1]), seed))
    brows = [np.unique(g.integers(0, 3000, 40)) if k < 3000 else np.unique(g.integers(0, n, 3)) for k in range(n)]
    brp = np.concatenate([[0], np.cumsum([x.size for x in brows])]).astype(np.int32)
    B = gen.CSR(n, n, brp, np.concatenate(brows).astype(np.int32),
                gen.matrices.random_values(int(brp[-1]), seed + 1))
    return A, B


def test_mixed_rows():
    A, B = mixed(3)
    (rp, col, val), info = run(A, B)
    assert info.segmented_rows >= 5 and info.long_rows >= 1
    W, sc, _ = oracle.spgemm(A, B)
    assert np.array_equal(rp, W.rp) and np.array_equal(col, W.col)
    ok, msg = oracle.check_values(val, W.val, sc, np.float64)
    assert ok, msg


def windowed(seed, mode="random"):
    """long rows whose output span (60,000 columns) needs 5 windows of 12,288:
    each A row references one long B row (30,000 entries over the span) and a
    few short ones -- windows x nnz(row) = 5 x 5 <= ~30,000 products"""
    g = np.random.default_rng(seed)
    n, kb = 60_000, 400
    brows = [np.sort(g.choice(n, 30_000, replace=False)) if k % 100 == 0 else np.unique(g.integers(0, n, 6))
             for k in range(kb)]
    brp = np.concatenate([[0], np.cumsum([x.size for x in brows])]).astype(np.int32)
    bcol = np.concatenate(brows).astype(np.int32)
    arows = [np.unique(np.concatenate([[100 * (r % 4)], g.integers(0, kb, 4)])) for r in range(120)]
    arp = np.concatenate([[0], np.cumsum([x.size for x in arows])]).astype(np.int32)
    acol = np.concatenate(arows).astype(np.int32)
    if mode == "int":
        return (gen.CSR(120, kb, arp, acol, gen.int_values(acol.size, seed)),
                gen.CSR(kb, n, brp, bcol, gen.int_values(bcol.size, seed + 1)))
    return (gen.CSR(120, kb, arp, acol, gen.matrices.random_values(acol.size, seed)),
            gen.CSR(kb, n, brp, bcol, gen.matrices.random_values(bcol.size, seed + 1)))


@pytest.mark.parametrize("mode", ["random", "int", "fp32"])
def test_windowed_wide_rows(mode):
    """Spans wider than 12,288 columns cut into windows, one CTA each; a
    window's output goes after the row's earlier windows' outputs."""
    A, B = windowed(8, "random" if mode == "fp32" else mode)
    if mode == "fp32":
        A = A.with_values(A.val.astype(np.float32))
        B = B.with_values(B.val.astype(np.float32))
    (rp, col, val), info = run(A, B)
    W, sc, _ = oracle.spgemm(A, B)
    spans = [(W.col[W.rp[r + 1] - 1] - W.col[W.rp[r]] + 1) for r in range(A.m)]
    assert max(spans) > 4 * 12288
    assert info.long_rows == 0 and info.segmented_rows > A.m  # several windows per row
    assert np.array_equal(rp, W.rp) and np.array_equal(col, W.col)
    assert np.array_equal(val, W.val), "k-ordered accumulation: bit-exact"


_OFF = r"""
import sys, numpy as np
sys.path.insert(0, {root!r})
import oracle
from tests.test_gpu_spgemm_segmented import dense, run
A = dense(200, 5)
(rp, col, val), info = run(A, A)
W, sc, _ = oracle.spgemm(A, A)
ok = np.array_equal(rp, W.rp) and np.array_equal(col, W.col) and oracle.check_values(val, W.val, sc, np.float64)[0]
print(info.segmented_rows, info.long_rows, ok)
"""


def test_segmented_off_uses_esc():
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, MSP_SPGEMM_SEGMENTED="0")
    r = subprocess.run([sys.executable, "-c", _OFF.format(root=root)], env=env, capture_output=True, text=True,
                       timeout=600)
    assert r.returncode == 0, r.stderr
    assert r.stdout.split()[-3:] == ["0", "200", "True"], r.stdout
