"""Dense N x N A*A through the shipped SpGEMM: the paper's
failure case for sort-based SpGEMM (Dense 2000^2 ran out of memory on its
GPU).  Reports the workspace the ESC path would need (from
msp_spgemm_info), timings and products/s with the segmented path, and a
parity check of sampled rows against the oracle.  MSP_SPGEMM_SEGMENTED=0 in
the environment runs the ESC long-row path instead (ablation).

    python tools/dense_spgemm.py 1000 [2000 ...]"""
import json
import sys

import numpy as np
import torch

sys.path.insert(0, __import__("os").path.dirname(__file__) + "/..")
import gen  # noqa: E402
import oracle  # noqa: E402
import paper_conf_ipps_daltonbmog15_b200 as msp  # noqa: E402


def dense(n, seed=1):
    g = np.random.default_rng(seed)
    rp = (np.arange(n + 1, dtype=np.int64) * n).astype(np.int32)
    return gen.CSR(n, n, rp, np.tile(np.arange(n, dtype=np.int32), n), g.uniform(-1, 1, n * n))


for arg in sys.argv[1:]:
    n = int(arg)
    A = dense(n)
    dA = msp.CsrTensor.from_arrays(A.rp, A.col, A.val, (n, n), "cuda")
    p = msp.SpGemmPlan(dA, dA)
    info = p.setup()
    res = {"n": n, "nprods": int(info.nprods), "segmented_rows": int(info.segmented_rows),
           "long_rows": int(info.long_rows), "main_ws_bytes": int(info.main_ws_bytes)}
    try:
        ts = []
        for i in range(3):
            e = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
            q = msp.SpGemmPlan(dA, dA)
            e[0].record()
            q.setup()
            q.symbolic()
            C = q.numeric()
            e[1].record()
            torch.cuda.synchronize()
            if i:
                ts.append(e[0].elapsed_time(e[1]))
        ms = float(np.mean(ts))
        rows = np.array([0, n // 2, n - 1])
        off, wcol, wval, sc = oracle.spgemm_rows(A, A, rows)
        rp, col, val = C.numpy()
        ok = all(np.array_equal(col[rp[r]:rp[r + 1]], wcol[off[k]:off[k + 1]]) and
                 np.array_equal(val[rp[r]:rp[r + 1]], wval[off[k]:off[k + 1]]) for k, r in enumerate(rows))
        res.update({"ms": ms, "products_per_s": info.nprods / ms * 1e3, "nnz_c": C.nnz,
                    "sampled_rows_bit_exact": bool(ok)})
    except Exception as ex:  # noqa: BLE001  (the ESC path may exceed HBM)
        res["error"] = f"{type(ex).__name__}: {str(ex)[:200]}"
    print(json.dumps(res), flush=True)
    del dA, p
    torch.cuda.empty_cache()
