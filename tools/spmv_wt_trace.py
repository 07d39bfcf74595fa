"""Per-tile timeline of the warp-tile SpMV (experiment aid; libmsp built with
MSP_NVCC_EXTRA=-DMSP_SPMV_TRACE): clock64 stamps in microseconds at the max
SM clock.  slots: 0 split known, 1 slot free (producer) | 2 worker ready,
3 landed, 4 released, 5 walked, 6 published + previous tile finished."""
import ctypes
import sys

import numpy as np
import torch

sys.path.insert(0, __import__("os").path.dirname(__file__) + "/..")
import gen  # noqa: E402
import paper_conf_ipps_daltonbmog15_b200 as msp  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C2"
A = gen.config(cfg, "random")
dA = msp.CsrTensor.from_arrays(A.rp, A.col, A.val, (A.m, A.n), "cuda")
x = torch.as_tensor(gen.x_vector(A.n, "random", dtype=A.val.dtype), device="cuda")
for _ in range(5):
    msp.spmv(dA, x)
torch.cuda.synchronize()
buf = np.zeros((4, 256, 8), dtype=np.int64)
L = msp.lib()
assert L.msp_debug_spmv_wt_trace(buf.ctypes.data_as(ctypes.c_void_p)) == 0
mhz = 1965.0
print("  t   split  free   ready  land   rel    walk   done  (us)")
for c in range(2):
    print(f"CTA {c}")
    for t in range(256):
        row = buf[c, t, :7]
        if not row.any():
            continue
        print(f"{t:3d} " + " ".join(f"{v / mhz:6.2f}" for v in row))
