"""Narrow down warp-tile SpMV failures (debug aid): run with
MSP_SPMV_CFG=-1 MSP_SPMV_WT=2 [MSP_SPMV_K=7]."""
import sys
import numpy as np
import torch
sys.path.insert(0, __import__("os").path.dirname(__file__) + "/..")
import gen  # noqa: E402
import oracle  # noqa: E402
import paper_conf_ipps_daltonbmog15_b200 as msp  # noqa: E402
from tests.gpu_util import tile_edge_matrix  # noqa: E402


def check(name, A):
    x = gen.x_vector(A.n, "int", dtype=A.val.dtype)
    d = msp.CsrTensor.from_arrays(A.rp, A.col, A.val, (A.m, A.n), "cuda")
    y = msp.spmv(d, torch.as_tensor(x, device="cuda")).cpu().numpy()
    y2 = msp.spmv(d, torch.as_tensor(x, device="cuda")).cpu().numpy()
    w = oracle.spmv(A, x)[0]
    bad = np.flatnonzero(y != w)
    lens = np.diff(A.rp)
    msg = f"{name}: m={A.m} nnz={A.nnz} bad={bad.size} det={np.array_equal(y, y2)}"
    if bad.size:
        r = bad[:5]
        msg += f" rows={r.tolist()} lens={lens[r].tolist()} got={y[r].tolist()} want={w[r].tolist()}"
    print(msg, flush=True)


rng = np.random.default_rng(0)
check("uniform5", tile_edge_matrix([5] * 200000, n=5000, seed=1))
check("uniform5+empty", tile_edge_matrix(list(rng.choice([0, 5], 200000)), n=5000, seed=2))
check("long1", tile_edge_matrix([3] * 1000 + [200000] + [3] * 1000, n=300000, seed=3))
check("long_at0", tile_edge_matrix([200000] + [3] * 100000, n=300000, seed=4))
check("many_long", tile_edge_matrix(list(rng.integers(0, 3000, 300)), n=5000, seed=5))
check("C4/0.05", gen.config("C4", "int", scale=0.05))
check("C4/0.25", gen.config("C4", "int", scale=0.25))
check("C3/64", gen.config("C3", "int", scale=1 / 64))
check("emptyruns", tile_edge_matrix([0] * 50000 + [4] * 1000 + [0] * 50000 + [7] * 5000, n=5000, seed=6))
