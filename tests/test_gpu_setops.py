"""Set operations: CUDA path (C ABI) vs the CPU
oracle, bit-exact (integer / index work), over both key widths, keys-only and
key-value pairs, all four operations, sizes spanning many tiles, and runs of
duplicates longer than a tile (the balanced-path cut then falls inside
key-rank runs, reading R4)."""
import json
from pathlib import Path

import numpy as np
import pytest
import torch

import oracle

pytestmark = pytest.mark.gpu

OPS = ["union", "intersection", "difference", "symmetric_difference"]
GOLD = json.loads((Path(__file__).parent / "golden" / "fig1_partition.json").read_text())


def run(op, a, b, av=None, bv=None):
    from paper_conf_ipps_daltonbmog15_b200 import set_operation
    sig = np.int32 if a.dtype == np.uint32 else np.int64
    ta = torch.from_numpy(a.view(sig).copy()).cuda()
    tb = torch.from_numpy(b.view(sig).copy()).cuda()
    tav = torch.from_numpy(av).cuda() if av is not None else None
    tbv = torch.from_numpy(bv).cuda() if bv is not None else None
    k, v = set_operation(op, ta, tb, tav, tbv)
    return k.cpu().numpy().view(a.dtype), (v.cpu().numpy() if v is not None else None)


def check(op, a, b, av=None, bv=None, label=""):
    gk, gv = run(op, a, b, av, bv)
    ek, ev = oracle.set_op(op, a, b, av, bv)
    assert np.array_equal(gk, ek), f"{op} {label}: keys differ (got {gk.size}, want {ek.size})"
    if av is not None:
        assert np.array_equal(gv.view(np.uint8), ev.view(np.uint8)), f"{op} {label}: values differ"


def sorted_keys(rng, n, hi, dtype):
    return np.sort(rng.integers(0, hi, size=n, dtype=np.uint64)).astype(dtype)


@pytest.mark.parametrize("op", OPS)
def test_fig1_lists(op):
    a = np.array([ord(c) for c in GOLD["A"]], np.uint32)
    b = np.array([ord(c) for c in GOLD["B"]], np.uint32)
    check(op, a, b, label="Fig 1")


@pytest.mark.parametrize("dtype", [np.uint32, np.uint64])
@pytest.mark.parametrize("op", OPS)
def test_random_sizes_and_duplication(op, dtype):
    rng = np.random.default_rng(hash((op, dtype().itemsize)) % 2**32)
    big = 2**32 - 1 if dtype == np.uint32 else 2**64 - 1
    cases = [(0, 0, 10), (0, 5, 10), (7, 0, 10), (1, 1, 2), (100, 37, 50),
             (5000, 7000, 10**9),         # mostly unique keys (the SpAdd regime)
             (40000, 30000, 10),          # runs of thousands of copies: cuts inside key-rank runs
             (25000, 25000, 5000),        # short runs
             (100000, 3, 10**6), (3, 100000, 10**6)]
    for na, nb, hi in cases:
        a = sorted_keys(rng, na, min(hi, big), dtype)
        b = sorted_keys(rng, nb, min(hi, big), dtype)
        check(op, a, b, label=f"{na}x{nb} keys<{hi}")


@pytest.mark.parametrize("op", OPS)
def test_pairs(op):
    rng = np.random.default_rng(9)
    for dtype, vdt in [(np.uint32, np.float32), (np.uint64, np.float64), (np.uint32, np.int64)]:
        for na, nb, hi in [(20000, 15000, 3000), (30000, 30000, 7), (1, 4000, 2)]:
            a = sorted_keys(rng, na, hi, dtype)
            b = sorted_keys(rng, nb, hi, dtype)
            av = rng.standard_normal(na).astype(vdt) if vdt != np.int64 else rng.integers(-9, 9, na)
            bv = rng.standard_normal(nb).astype(vdt) if vdt != np.int64 else rng.integers(-9, 9, nb)
            check(op, a, b, av, bv, label=f"pairs {dtype.__name__}/{np.dtype(vdt).name} {na}x{nb}")


def test_extreme_keys_and_identities():
    top = np.uint64(2**64 - 1)
    a = np.array([0, 5, 5, 2**63, 2**64 - 2, 2**64 - 1, 2**64 - 1], np.uint64)
    b = np.array([5, 2**63, 2**63, 2**64 - 1], np.uint64)
    for op in OPS:
        check(op, a, b, label="u64 extremes")
    a32 = np.array([0, 1, 2**31, 2**32 - 1, 2**32 - 1], np.uint32)
    for op in OPS:
        check(op, a32, a32, label="A op A")
    assert top == np.uint64(2**64 - 1)


def test_capacity_and_dtype_errors():
    from paper_conf_ipps_daltonbmog15_b200 import MspError, lib
    import ctypes
    n = ctypes.c_size_t(0)
    assert lib().msp_set_op_workspace(10, 10, ctypes.byref(n)) == 0
    ws = torch.zeros(int(n.value), dtype=torch.uint8, device="cuda")
    a = torch.arange(10, dtype=torch.int32, device="cuda")
    c = torch.empty(5, dtype=torch.int32, device="cuda")
    nc = ctypes.c_int64(0)
    st = lib().msp_set_operation(0, a.data_ptr(), None, 10, a.data_ptr(), None, 10, 4, 0, c.data_ptr(), None, 5,
                                 ctypes.byref(nc), ws.data_ptr(), ws.numel(), None)
    assert st == 3  # MSP_ERR_SHAPE: capacity below nA + nB
    st = lib().msp_set_operation(0, a.data_ptr(), None, 10, a.data_ptr(), None, 10, 2, 0, c.data_ptr(), None, 20,
                                 ctypes.byref(nc), ws.data_ptr(), ws.numel(), None)
    assert st == 2  # MSP_ERR_DTYPE
    assert MspError


@pytest.mark.parametrize("kind", ["keys-32", "pairs-64"])
def test_fig2_scale(kind):
    """The Fig 2 workload shape at 2e7 inputs (union, inputs split evenly,
    uniform keys below 2^30 as tools/setops_bench.py draws them), exact."""
    rng = np.random.default_rng(2)
    kd = np.uint32 if kind == "keys-32" else np.uint64
    n = 10**7
    a = np.sort(rng.integers(0, 2**30, size=n)).astype(kd)
    b = np.sort(rng.integers(0, 2**30, size=n)).astype(kd)
    if kind == "pairs-64":
        check("union", a, b, np.arange(n, dtype=np.int64), -np.arange(n, dtype=np.int64), label="2e7 pairs-64")
    else:
        check("union", a, b, label="2e7 keys-32")


@pytest.mark.parametrize("op", OPS)
def test_async_form(op):
    """msp_set_operation_async: same keys / values as the oracle, the size and
    the unsorted flag land in a device int64[2] in stream order; several
    calls queued back to back on one stream (shared workspace) without a
    host sync in between, including an empty one and an unsorted one."""
    from paper_conf_ipps_daltonbmog15_b200 import set_operation
    rng = np.random.default_rng(17)
    cases = []
    for na, nb, hi in [(30000, 20000, 4000), (0, 0, 10), (1, 3000, 5), (50000, 50000, 10**9)]:
        a = sorted_keys(rng, na, hi, np.uint32)
        b = sorted_keys(rng, nb, hi, np.uint32)
        av = rng.standard_normal(na)
        bv = rng.standard_normal(nb)
        cases.append((a, b, av, bv))
    bad = cases[0][0].copy()
    bad[100:200] = bad[100:200][::-1]
    outs = []
    for a, b, av, bv in cases + [(bad, cases[0][1], cases[0][2], cases[0][3])]:
        ta = torch.from_numpy(a.view(np.int32)).cuda()
        tb = torch.from_numpy(b.view(np.int32)).cuda()
        outs.append(set_operation(op, ta, tb, torch.from_numpy(av).cuda(), torch.from_numpy(bv).cuda(), sync=False))
    torch.cuda.synchronize()
    for (a, b, av, bv), (k, v, cnt) in zip(cases, outs):
        n, flag = cnt.cpu().tolist()
        ek, ev = oracle.set_op(op, a, b, av, bv)
        assert flag == 0 and n == ek.size
        assert np.array_equal(k[:n].cpu().numpy().view(np.uint32), ek)
        assert np.array_equal(v[:n].cpu().numpy().view(np.uint8), ev.view(np.uint8))
    assert outs[-1][2][1].item() != 0, "unsorted keys must raise the device flag"
