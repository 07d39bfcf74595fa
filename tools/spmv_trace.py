"""SpMV per-tile timeline (experiment aid; needs a libmsp built with
MSP_NVCC_EXTRA=-DMSP_SPMV_TRACE): clock64 stamps per tile and role of CTAs
0..3, printed in microseconds at the max SM clock.

slots: 0 split searched, 1 TMA issued (producer) | 2 landed, 3 row map built
(row warp) | 4/8 stage seen, 5/9 gathers issued, 6/10 walk done, 7/11 tile
finished, 12/13 row map seen, 14/15 last gather returned (worker warps 0 / NW-1)."""
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
buf = np.zeros((4, 64, 16), dtype=np.int64)
L = msp.lib()
L.msp_debug_spmv_trace.restype = ctypes.c_int
assert L.msp_debug_spmv_trace(buf.ctypes.data_as(ctypes.c_void_p)) == 0
mhz = 1965.0
names = ["srch", "issue", "land", "rmap", "w0see", "w0gat", "w0walk", "w0fin", "w7see", "w7gat", "w7walk", "w7fin",
         "w0rm", "w7rm", "w0xv", "w7xv"]
for c in range(2):
    print(f"CTA {c} (us)")
    print("  t  " + " ".join(f"{n:>7s}" for n in names))
    for t in range(64):
        row = buf[c, t, :16]
        if not row.any():
            continue
        print(f"{t:3d}  " + " ".join(f"{v / mhz:7.2f}" for v in row))
