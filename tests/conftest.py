import json
import os
import sys
from pathlib import Path

import numpy as np
import pytest

ROOT = Path(__file__).resolve().parents[1]
if str(ROOT) not in sys.path:
    sys.path.insert(0, str(ROOT))

GOLDEN = ROOT / "tests" / "golden"


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA B200 (run with -m gpu on the GPU box)")
    config.addinivalue_line("markers", "slow: larger CPU cases")


def load_golden(name: str):
    with open(GOLDEN / name) as f:
        return json.load(f)


def csr_from_dense(d, dtype=np.float64):
    from gen import CSR
    d = np.asarray(d)
    m, n = d.shape
    r, c = np.nonzero(d)
    rp = np.zeros(m + 1, dtype=np.int64)
    np.cumsum(np.bincount(r, minlength=m), out=rp[1:])
    return CSR(m, n, rp.astype(np.int32), c.astype(np.int32), d[r, c].astype(dtype))


def csr_from_tuples(tuples, m, n, dtype=np.float64):
    from gen import CSR
    t = sorted(tuple(x) for x in tuples)
    r = np.array([x[0] for x in t], dtype=np.int64)
    c = np.array([x[1] for x in t], dtype=np.int32)
    v = np.array([x[2] for x in t], dtype=dtype)
    rp = np.zeros(m + 1, dtype=np.int64)
    np.cumsum(np.bincount(r, minlength=m), out=rp[1:])
    return CSR(m, n, rp.astype(np.int32), c, v)


@pytest.fixture(scope="session")
def paper_example():
    return load_golden("paper_example.json")


def has_cuda() -> bool:
    try:
        import torch
        return torch.cuda.is_available()
    except Exception:
        return False
