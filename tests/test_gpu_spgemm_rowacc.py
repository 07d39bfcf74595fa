"""SpGEMM row-accumulator path for short rows (msp_spgemm_info
.row_accumulator): taken when every short row's output span is at most
65,536 columns.  Parity with Gustavson's oracle (structure bit-exact, values
within the BJ:5 tolerance, integer inputs exact) on the cases that exercise
its branches, and the ESC tile path it replaces kept under test by re-running
the SpGEMM suite with the accumulator disabled (MSP_SPGEMM_ROWACC=0)."""
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
    p.setup()
    C = p.numeric()
    rp, col, val = C.numpy()
    return rp, col, val, p.info


def check(A, B, label, exact=False):
    rp, col, val, info = run(A, B)
    W, scale, npr = oracle.spgemm(A, B)
    assert info.nprods == npr, label
    assert np.array_equal(rp, W.rp), f"{label}: row_offsets differ"
    assert np.array_equal(col, W.col), f"{label}: col_idx differ"
    ok, msg = oracle.check_values(val, W.val, scale, A.val.dtype)
    assert ok, f"{label}: {msg}"
    if exact:
        assert np.array_equal(val, W.val), f"{label}: integer mode must be exact"
    return info


def _rows(lens, ncols, rng, lo=0, hi=None):
    hi = ncols if hi is None else hi
    cols = [np.sort(rng.choice(np.arange(lo, hi), size=int(L), replace=False)) for L in lens]
    col = np.concatenate(cols).astype(np.int32) if len(cols) else np.zeros(0, np.int32)
    rp = np.zeros(len(lens) + 1, np.int64)
    np.cumsum(lens, out=rp[1:])
    return rp.astype(np.int32), col


def test_taken_on_stencils():
    for name in ("C1",):
        A = gen.config(name, "int")
        info = check(A, A, name, exact=True)
        assert info.row_accumulator > 0 and info.ntiles == 0
    A = gen.config("C2", "random")
    p_rows = slice(0, 20001)
    S = gen.CSR(20000, A.n, A.rp[p_rows] - A.rp[0], A.col[:A.rp[20000]], A.val[:A.rp[20000]])
    info = check(S, A, "C2 rows [0, 20000) x A")
    assert info.row_accumulator > 0


def test_many_unique_columns_and_long_b_rows():
    """Rows with > 512 distinct output columns (the numeric accumulator runs
    several column passes), B rows longer than a warp (the per-step loop),
    empty B rows, empty A rows, every row within a 60,000-column span."""
    rng = np.random.default_rng(11)
    k, n = 300, 60_000
    blens = np.where(rng.random(k) < 0.1, 0, rng.integers(1, 70, k))
    Brp, Bcol = _rows(blens, n, rng)
    B = gen.CSR(k, n, Brp, Bcol, gen.matrices.random_values(Bcol.size, 2))
    alens = np.where(np.arange(400) % 9 == 0, 0, rng.integers(1, 30, 400))
    Arp, Acol = _rows(alens, k, rng)
    A = gen.CSR(400, k, Arp, Acol, gen.matrices.random_values(Acol.size, 3))
    info = check(A, B, "wide rows")
    assert info.row_accumulator > 0
    W, _, _ = oracle.spgemm(A, B)
    assert np.diff(W.rp).max() > 512, "no row needs a second accumulator pass"
    Ai = A.with_values(gen.int_values(A.nnz, 4))
    Bi = B.with_values(gen.int_values(B.nnz, 5))
    check(Ai, Bi, "wide rows int", exact=True)
    check(A.with_values(A.val.astype(np.float32)), B.with_values(B.val.astype(np.float32)), "wide rows fp32")


def test_signed_zero_and_cancellation():
    """-0.0 products and exact cancellations: the accumulator starts at -0.0,
    so a single product keeps its sign and a cancelled sum is +0.0 -- both
    as in the oracle (compared bit for bit)."""
    A = gen.CSR(3, 2, np.array([0, 2, 3, 4], np.int32), np.array([0, 1, 0, 1], np.int32),
                np.array([1.0, -1.0, -0.0, 2.0]))
    B = gen.CSR(2, 3, np.array([0, 2, 4], np.int32), np.array([0, 2, 0, 2], np.int32),
                np.array([3.0, 5.0, 3.0, -0.0]))
    rp, col, val, info = run(A, B)
    W, _, _ = oracle.spgemm(A, B)
    assert info.row_accumulator > 0
    assert np.array_equal(rp, W.rp) and np.array_equal(col, W.col)
    assert np.array_equal(val.view(np.uint64), W.val.view(np.uint64)), (val, W.val)


@pytest.mark.skipif(os.environ.get("MSP_SPGEMM_SMALL") != "0" and os.environ.get("MSP_SPGEMM_ROWACC") != "0",
                    reason="with the small path on, wide rows take it (test_gpu_spgemm_small.py)")
def test_not_taken_on_wide_rows():
    """Small path off (v5 behaviour): one short row spanning more than 65,536
    columns sends every short row to the ESC tile pass (the choice is
    global)."""
    rng = np.random.default_rng(3)
    n = 200_000
    B = gen.CSR(3, n, np.array([0, 2, 3, 4], np.int32), np.array([0, 150_000, 7, 9], np.int32), np.ones(4))
    A = gen.CSR(50, 3, *_rows(rng.integers(1, 3, 50), 3, rng), None)
    A = A.with_values(np.ones(A.col.size))
    info = check(A, B, "wide span", exact=True)
    assert info.row_accumulator == 0 and info.ntiles > 0


_ESC_SUITE = ["tests/test_gpu_spgemm.py", "tests/test_gpu_spgemm_segmented.py", "tests/test_gpu_spgemm_fuzz.py"]


@pytest.mark.skipif(os.environ.get("MSP_SPGEMM_ROWACC") == "0", reason="already the ESC-only run")
def test_esc_tile_path_suite():
    """The SpGEMM suite again with the row accumulator disabled, so the ESC
    tile pass (expansion, run-merge / block sort, compression) stays under
    test on the small and stencil cases the accumulator now takes."""
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, MSP_SPGEMM_ROWACC="0")
    r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-m", "gpu", *_ESC_SUITE,
                        "tests/test_gpu_spgemm_rowacc.py::test_not_taken_on_wide_rows",
                        "tests/test_gpu_fullsize.py::test_spgemm_64bit_keys"],
                       cwd=root, env=env, capture_output=True, text=True, timeout=1800)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-2000:]
