"""One-pass SpAdd (msp_spadd_fused) A + A^T timing on BJ configs (tuning
aid): CUDA events over 20 calls after 3 warm-up calls, C preallocated;
exactness vs the oracle on the whole result.

    python tools/spadd_fused_time.py C3 C2"""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(__file__) + "/..")
import gen  # noqa: E402
import oracle  # noqa: E402
import paper_conf_ipps_daltonbmog15_b200 as msp  # noqa: E402

for cfg in sys.argv[1:]:
    A = gen.config(cfg, "random")
    T = gen.transpose(A)
    dA = msp.CsrTensor.from_arrays(A.rp, A.col, A.val, (A.m, A.n), "cuda")
    dT = msp.CsrTensor.from_arrays(T.rp, T.col, T.val, (T.m, T.n), "cuda")
    cap = A.nnz + T.nnz
    oc = torch.empty(cap, dtype=torch.int32, device="cuda")
    ov = torch.empty(cap, dtype=dA.dtype, device="cuda")
    for _ in range(3):
        C = msp.spadd_fused(dA, dT, col=oc, val=ov)
    torch.cuda.synchronize()
    ts = []
    for _ in range(20):
        a = torch.cuda.Event(enable_timing=True)
        b = torch.cuda.Event(enable_timing=True)
        a.record()
        C = msp.spadd_fused(dA, dT, col=oc, val=ov)
        b.record()
        ts.append((a, b))
    torch.cuda.synchronize()
    ms = float(np.mean([a.elapsed_time(b) for a, b in ts]))
    vs = A.val.dtype.itemsize
    by = (A.nnz + T.nnz) * (4 + vs) + C.nnz * (4 + vs) + 12 * (A.m + 1)
    W = oracle.spadd(A, T)
    rp, col, val = C.numpy()
    exact = bool(np.array_equal(rp, W.rp) and np.array_equal(col, W.col)
                 and np.array_equal(val.view(np.uint8), W.val.view(np.uint8)))
    print(json.dumps({"cfg": cfg, "ms": ms, "GB_s": by / ms / 1e6, "exact": exact,
                      "ipt": os.environ.get("MSP_NVCC_EXTRA", "default")}), flush=True)
