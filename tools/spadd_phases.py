"""SpAdd A + A^T per-phase timing (tuning aid): symbolic (partition + count +
scans + nnz read-back) and numeric (fill) with CUDA events, plus the launch
list of one call via torch.profiler-free event pairs; exactness vs the oracle
on the whole result."""
import json
import sys

import numpy as np
import torch

sys.path.insert(0, __import__("os").path.dirname(__file__) + "/..")
import gen  # noqa: E402
import oracle  # noqa: E402
import paper_conf_ipps_daltonbmog15_b200 as msp  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C3"
A = gen.config(cfg, "random")
T = gen.transpose(A)
dA = msp.CsrTensor.from_arrays(A.rp, A.col, A.val, (A.m, A.n), "cuda")
dT = msp.CsrTensor.from_arrays(T.rp, T.col, T.val, (T.m, T.n), "cuda")
for _ in range(3):
    C = msp.spadd(dA, dT)
torch.cuda.synchronize()
rec = []
for _ in range(10):
    e = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
    p = msp.SpAddPlan(dA, dT)
    e[0].record()
    p.symbolic()
    e[1].record()
    C = p.numeric()
    e[2].record()
    rec.append(e)
torch.cuda.synchronize()
sym = float(np.mean([e[0].elapsed_time(e[1]) for e in rec]))
num = float(np.mean([e[1].elapsed_time(e[2]) for e in rec]))
vs = A.val.dtype.itemsize
by = (A.nnz + T.nnz) * (4 + vs) + C.nnz * (4 + vs) + 12 * (A.m + 1)
W = oracle.spadd(A, T)
rp, col, val = C.numpy()
exact = bool(np.array_equal(rp, W.rp) and np.array_equal(col, W.col) and np.array_equal(val.view(np.uint8),
                                                                                          W.val.view(np.uint8)))
print(json.dumps({"cfg": cfg, "symbolic_ms": sym, "numeric_ms": num, "total_ms": sym + num,
                  "GB_s": by / (sym + num) / 1e6, "exact": exact}))
