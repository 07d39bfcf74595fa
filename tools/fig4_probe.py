"""Fig 4 reproduction aid: run
the radix SpGEMM symbolic phase on a matrix whose B has 4096 columns (12
column bits, the paper's "28 -> 12 bits" case) and enough products that the
per-tile sort dominates; the sort variant comes from MSP_RX_SORT_BITS /
MSP_RX_TWO_PASS in the environment.  Time rx_tile_kernel with ncu or CUDA
events around symbolic.  Prints symbolic ms."""
import json
import sys

import numpy as np
import torch

sys.path.insert(0, __import__("os").path.dirname(__file__) + "/..")
import gen  # noqa: E402
import paper_conf_ipps_daltonbmog15_b200 as msp  # noqa: E402

m, k, n = 200_000, 4096, 4096
rng = np.random.default_rng(4)


def rows_of(mm, nn, L, seed):
    g = np.random.default_rng(seed)
    c = np.sort(g.integers(0, nn, size=(mm, L)), axis=1).astype(np.int64)
    keep = np.ones_like(c, dtype=bool)
    keep[:, 1:] = c[:, 1:] != c[:, :-1]
    lens = keep.sum(1)
    rp = np.concatenate([[0], np.cumsum(lens)]).astype(np.int32)
    return gen.CSR(mm, nn, rp, c[keep].astype(np.int32), gen.matrices.random_values(int(lens.sum()), seed))


A = rows_of(m, k, 16, 1)
B = rows_of(k, n, 16, 2)
dA = msp.CsrTensor.from_arrays(A.rp, A.col, A.val, (A.m, A.n), "cuda")
dB = msp.CsrTensor.from_arrays(B.rp, B.col, B.val, (B.m, B.n), "cuda")
reps = int(sys.argv[1]) if len(sys.argv) > 1 else 5
ts = []
for i in range(reps + 1):
    p = msp.SpGemmRadixPlan(dA, dB)
    p.setup()
    a = torch.cuda.Event(enable_timing=True)
    b = torch.cuda.Event(enable_timing=True)
    a.record()
    p.symbolic()
    b.record()
    torch.cuda.synchronize()
    if i:
        ts.append(a.elapsed_time(b))
print(json.dumps({"nprods": p.nprods, "symbolic_ms": float(np.mean(ts)), "nnz_c": p.nnz}))
