"""Full-size parity (BASELINE.json configs at their real sizes, in the launch
configuration bench.py times) and the boundary's error paths on the GPU.

* SpGEMM C2 / C4 A*A: EVERY row offset and column index bit-exact, every
  value within tau * sum_k |a_ik||b_kj| (BJ:5, Z18) against Gustavson's
  oracle on the whole matrix (not sampled rows).
* SpMV / SpAdd C3 (R-MAT scale 22, fp32) at full size; SpMV C5 (10^8 rows)
  at full size; SpGEMM C5 A*A at full size (invariants on every row, 3,000
  sampled rows exact against the oracle).
* The 64-bit-key SpGEMM tile path (tiles whose row span does not fit the
  32-bit packed key next to the column bits), forced by construction.
* msp_csr_check, MSP_ERR_INPUT (unsorted set-operation keys, malformed CSR
  under MSP_DEBUG_VALIDATE) and MSP_ERR_OVERFLOW (nnz(C) > INT32_MAX).
"""
import ctypes
import os
import subprocess
import sys

import numpy as np
import pytest

import gen
import oracle
from tests.gpu_util import dev

pytestmark = pytest.mark.gpu


def spgemm_gpu(A, B):
    from paper_conf_ipps_daltonbmog15_b200 import SpGemmPlan
    p = SpGemmPlan(dev(A), dev(B))
    info = p.setup()
    C = p.numeric()
    rp, col, val = C.numpy()
    return rp, col, val, p.info


def assert_spgemm_complete(A, B, label, exact=False):
    rp, col, val, info = spgemm_gpu(A, B)
    W, scale, npr = oracle.spgemm(A, B)
    assert info.nprods == npr, label
    assert np.array_equal(rp, W.rp), f"{label}: row_offsets differ"
    assert np.array_equal(col, W.col), f"{label}: col_idx differ"
    ok, msg = oracle.check_values(val, W.val, scale, A.val.dtype)
    assert ok, f"{label}: {msg}"
    if exact:
        assert np.array_equal(val, W.val), f"{label}: integer mode must be exact"
    return info


def test_c2_spgemm_full_complete():
    """C2 A*A (BJ:8): 704,969,000 products, 120,553,784 = 494^3 entries."""
    A = gen.config("C2", "random")
    info = assert_spgemm_complete(A, A, "C2 A*A")
    assert info.nprods == 890 ** 3
    assert info.row_accumulator == 2 * (2 + 2 * 100 + 2 * 100 ** 2) + 1  # stencil rows: accumulator path, widest span


def test_c4_spgemm_full_complete():
    """C4 A*A (BJ:10) incl. the 1M-nnz dense row (long-row path), exact."""
    A = gen.config("C4", "int")
    info = assert_spgemm_complete(A, A, "C4 A*A", exact=True)
    assert info.long_rows >= 1
    # uniform rows: <= 64 products -> small path, more (spanning ~2e6 columns) -> promoted to long
    assert info.row_accumulator > 0 and info.small_rows > 0 and info.ntiles == 0


@pytest.mark.skipif(os.environ.get("MSP_SPGEMM_ROWACC") != "0",
                    reason="tile path only: run by test_gpu_spgemm_rowacc.py::test_esc_tile_path_suite")
def test_spgemm_64bit_keys():
    """B has 2^22 columns (22 column bits), and A's few nonzero rows are
    spread over 6000 rows, so one product tile spans > 2^(32-22) = 1024 rows:
    the 32-bit packed key cannot hold (row ordinal, col) and the tile kernel
    must take its 64-bit-key instantiation."""
    rng = np.random.default_rng(64)
    m, k, n = 6000, 500, 1 << 22
    lens = np.where(np.arange(m) % 7 == 0, rng.integers(1, 4, m), 0)
    A = gen.CSR(m, k, *_rows(lens, k, rng), None)
    A = A.with_values(gen.int_values(A.col.size, 1))
    blens = rng.integers(0, 6, k)
    B = gen.CSR(k, n, *_rows(blens, n, rng), None)
    B = B.with_values(gen.int_values(B.col.size, 2))
    info = assert_spgemm_complete(A, B, "64-bit keys", exact=True)
    cbits = (n - 1).bit_length()
    assert info.max_tile_span + 2 > (1 << (32 - cbits)), "the 64-bit key path was not taken"
    Ar = A.with_values(gen.matrices.random_values(A.nnz, 3))
    Br = B.with_values(gen.matrices.random_values(B.nnz, 4))
    assert_spgemm_complete(Ar, Br, "64-bit keys random")


def _rows(lens, ncols, rng):
    cols = [np.sort(rng.choice(ncols, size=int(L), replace=False)) for L in lens]
    col = np.concatenate(cols).astype(np.int32) if len(cols) else np.zeros(0, np.int32)
    rp = np.zeros(len(lens) + 1, np.int64)
    np.cumsum(lens, out=rp[1:])
    return rp.astype(np.int32), col


@pytest.fixture(scope="module")
def c3():
    return gen.config("C3", "random"), gen.config("C3", "int")


def test_c3_spmv_full(c3):
    from paper_conf_ipps_daltonbmog15_b200 import spmv
    import torch
    Ar, Ai = c3
    x = gen.x_vector(Ar.n, "random", seed=1003, dtype=np.float32)
    y = spmv(dev(Ar), torch.as_tensor(x, device="cuda")).cpu().numpy()
    want, scale = oracle.spmv(Ar, x)
    ok, msg = oracle.check_values(y, want, scale, np.float32)
    assert ok, "C3 SpMV: " + msg
    xi = gen.x_vector(Ai.n, "int", dtype=np.float32)
    yi = spmv(dev(Ai), torch.as_tensor(xi, device="cuda")).cpu().numpy()
    assert np.array_equal(yi, oracle.spmv(Ai, xi)[0])


def test_c3_spadd_full(c3):
    """C3 A + A^T (BJ:9, the SpAdd workload): structure and values bit-exact."""
    from paper_conf_ipps_daltonbmog15_b200 import spadd
    Ar, _ = c3
    T = gen.transpose(Ar)
    C = spadd(dev(Ar), dev(T))
    rp, col, val = C.numpy()
    W = oracle.spadd(Ar, T)
    assert np.array_equal(rp, W.rp) and np.array_equal(col, W.col)
    assert np.array_equal(val.view(np.uint32), W.val.view(np.uint32))
    from paper_conf_ipps_daltonbmog15_b200 import spadd_fused
    rp, col, val = spadd_fused(dev(Ar), dev(T)).numpy()
    assert np.array_equal(rp, W.rp) and np.array_equal(col, W.col), "fused: structure"
    assert np.array_equal(val.view(np.uint32), W.val.view(np.uint32)), "fused: values"


def test_c5_spmv_full():
    """C5 (BJ:11) at full size on one GPU: 10^8 rows, ~4e8 nonzeros."""
    from paper_conf_ipps_daltonbmog15_b200 import spmv
    import torch
    A = gen.config("C5", "int")
    x = gen.x_vector(A.n, "int")
    y = spmv(dev(A), torch.as_tensor(x, device="cuda")).cpu().numpy()
    assert np.array_equal(y, oracle.spmv(A, x)[0])


def test_c5_spgemm_full_sampled():
    """C5 A*A (BJ:11) at full size: 1.6e9 products through the small-row
    path.  On the GPU: Nprods, every row's length <= its product count and
    its columns strictly increasing, C.row_offsets consistent; 3,000 rows
    spread over the matrix (plus the first and last) against Gustavson's
    oracle, exact (integer mode)."""
    import torch
    from paper_conf_ipps_daltonbmog15_b200 import SpGemmPlan
    A = gen.config("C5", "int")
    blen = np.diff(A.rp.astype(np.int64))
    pa = blen[A.col]
    cs = np.zeros(A.nnz + 1, np.int64)
    np.cumsum(pa, out=cs[1:])
    P = cs[A.rp[1:]] - cs[A.rp[:-1]]
    del pa, cs
    dA = dev(A)
    p = SpGemmPlan(dA, dA)
    info = p.setup()
    assert info.nprods == int(P.sum())
    C = p.numeric()
    assert info.small_rows == int(np.count_nonzero((P > 0) & (P <= 64))) and info.ntiles == 0
    rp = C.rp.to(torch.int64)
    lens = rp[1:] - rp[:-1]
    assert int(rp[0]) == 0 and bool((lens >= 0).all()) and int(rp[-1]) == C.nnz
    assert bool((lens <= torch.as_tensor(P, device="cuda")).all())
    col = C.col.to(torch.int64)
    inc = col[1:] > col[:-1]
    starts = rp[1:-1][lens[1:] > 0]  # first entry of every nonempty row after the first
    inc[starts - 1] = True
    assert bool(inc.all()), "columns not strictly increasing inside a row"
    rows = np.unique(np.concatenate([[0, A.m - 1], np.random.default_rng(7).integers(0, A.m, 3000)]))
    off, wcol, wval, _ = oracle.spgemm_rows(A, A, rows)
    rph = C.rp.cpu().numpy()
    for k, r in enumerate(rows):
        a, b = int(rph[r]), int(rph[r + 1])
        assert b - a == off[k + 1] - off[k], f"row {r}: length"
        assert np.array_equal(C.col[a:b].cpu().numpy(), wcol[off[k]:off[k + 1]]), f"row {r}: columns"
        assert np.array_equal(C.val[a:b].cpu().numpy(), wval[off[k]:off[k + 1]]), f"row {r}: values"


# ------------------------------------------------------------- error paths

def test_csr_check_flags():
    from paper_conf_ipps_daltonbmog15_b200 import csr_check, CsrTensor
    A = gen.config("C1", "int")
    assert csr_check(dev(A)) == 0
    # column out of range
    bad = A.col.copy(); bad[5] = A.n
    assert csr_check(dev(gen.CSR(A.m, A.n, A.rp, bad, A.val))) & 2
    # unsorted (swap two columns of one row): only with the sorted check
    bad = A.col.copy(); bad[[0, 1]] = bad[[1, 0]]
    U = gen.CSR(A.m, A.n, A.rp, bad, A.val)
    assert csr_check(dev(U)) & 4
    assert csr_check(dev(U), sorted_unique=False) == 0
    # malformed offsets: a row end past nnz -- flagged, and col is never read
    # past its end (the validator must not fault on what it rejects)
    rp = np.array([0, 5, 100, 10], np.int32)
    M = CsrTensor.from_arrays(rp, np.arange(10, dtype=np.int32), np.ones(10), (3, 200), "cuda")
    assert csr_check(M) & 1
    rp = np.array([0, 6, 4, 10], np.int32)                           # decreasing
    M = CsrTensor.from_arrays(rp, np.arange(10, dtype=np.int32), np.ones(10), (3, 200), "cuda")
    assert csr_check(M) & 1


def test_set_operation_unsorted_is_input_error():
    import torch
    from paper_conf_ipps_daltonbmog15_b200 import set_operation, MspError
    rng = np.random.default_rng(5)
    a = np.sort(rng.integers(0, 1000, 50_000)).astype(np.int32)
    b = np.sort(rng.integers(0, 1000, 40_000)).astype(np.int32)
    a[1000:1100] = a[1000:1100][::-1]                                   # a descending stretch
    with pytest.raises(MspError) as e:
        set_operation("union", torch.from_numpy(a).cuda(), torch.from_numpy(b).cuda())
    assert e.value.status == 6
    # a sorted signed tensor with negatives is unsorted as unsigned keys
    s = np.sort(rng.integers(-500, 500, 20_000)).astype(np.int32)
    with pytest.raises(MspError):
        set_operation("intersection", torch.from_numpy(s).cuda(), torch.from_numpy(s).cuda())
    # wildly unsorted (random) input: memory-safe and reported
    r = rng.integers(0, 2 ** 31, 200_000).astype(np.int32)
    for op in ("union", "intersection", "difference", "symmetric_difference"):
        with pytest.raises(MspError):
            set_operation(op, torch.from_numpy(r).cuda(), torch.from_numpy(np.sort(r)).cuda(),
                          torch.from_numpy(r.view(np.float32)).cuda(), torch.from_numpy(r.view(np.float32)).cuda())
    torch.cuda.synchronize()
    k, _ = set_operation("union", torch.from_numpy(np.sort(a)).cuda(), torch.from_numpy(b).cuda())
    assert np.array_equal(k.cpu().numpy(), oracle.set_op("union", np.sort(a).astype(np.uint32),
                                                         b.astype(np.uint32))[0].astype(np.int32))


def test_spgemm_overflow():
    """nnz(C) = 1.1e6 * 2000 = 2.2e9 > INT32_MAX: symbolic returns
    MSP_ERR_OVERFLOW (Z16), never a wrapped row_offsets array."""
    from paper_conf_ipps_daltonbmog15_b200 import SpGemmPlan, MspError
    m, w = 1_100_000, 2000
    A = gen.CSR(m, 1, np.arange(m + 1, dtype=np.int32), np.zeros(m, np.int32), np.ones(m))
    B = gen.CSR(1, w, np.array([0, w], np.int32), np.arange(w, dtype=np.int32), np.ones(w))
    p = SpGemmPlan(dev(A), dev(B))
    info = p.setup()
    assert info.nprods == m * w
    with pytest.raises(MspError) as e:
        p.symbolic()
    assert e.value.status == 5


_VALIDATE_SCRIPT = r"""
import sys, numpy as np
sys.path.insert(0, {root!r})
import gen
from tests.gpu_util import dev
from paper_conf_ipps_daltonbmog15_b200 import spadd, spgemm, spmv, MspError
import torch
A = gen.config("C1", "int")
bad = A.col.copy(); bad[[0, 1]] = bad[[1, 0]]
U = gen.CSR(A.m, A.n, A.rp, bad, A.val)
codes = []
for fn in (lambda: spadd(dev(U), dev(A)), lambda: spgemm(dev(A), dev(U))):
    try:
        fn(); codes.append(0)
    except MspError as e:
        codes.append(e.status)
oob = A.col.copy(); oob[3] = A.n + 7
try:
    spmv(dev(gen.CSR(A.m, A.n, A.rp, oob, A.val)), torch.zeros(A.n, dtype=torch.float64, device="cuda")); codes.append(0)
except MspError as e:
    codes.append(e.status)
y = spmv(dev(U), torch.ones(A.n, dtype=torch.float64, device="cuda"))   # SpMV accepts any column order
print(codes)
"""


def test_debug_validate_env():
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, MSP_DEBUG_VALIDATE="1")
    r = subprocess.run([sys.executable, "-c", _VALIDATE_SCRIPT.format(root=root)], env=env, capture_output=True,
                       text=True, timeout=300)
    assert r.returncode == 0, r.stderr
    assert r.stdout.strip().splitlines()[-1] == "[6, 6, 6]", r.stdout + r.stderr
