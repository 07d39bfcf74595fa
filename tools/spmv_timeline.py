"""Profiling aid: per-tile timestamps of the SpMV kernel roles (MSP_SPMV_DEBUG=16).
Columns: producer iteration start, after split search, after empty wait, row
warp done, worker 0 phase A done, worker NW-1 walk done, worker 0 got the
stage (a_issue), worker 0 got the row map (microseconds)."""
import ctypes, os, sys
import numpy as np
import torch
sys.path.insert(0, os.environ.get("GRAFT_REPO_ROOT", os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import gen
import paper_conf_ipps_daltonbmog15_b200 as msp
from paper_conf_ipps_daltonbmog15_b200 import _lib

A = gen.config("C2", "random")
x = gen.x_vector(A.n, "random", seed=1)
Ad = msp.CsrTensor.from_arrays(A.rp, A.col, A.val, (A.m, A.n), "cuda")
xd = torch.as_tensor(x, device="cuda")
for _ in range(5):
    msp.spmv(Ad, xd)
torch.cuda.synchronize()
h = np.zeros(1024 * 256, dtype=np.int64)
assert _lib.lib().msp_debug_copy_timestamps(h.ctypes.data_as(ctypes.c_void_p), ctypes.c_size_t(h.nbytes)) == 0
ts = h.reshape(1024, 32, 8)[:, :30, :8]
t0 = ts[ts > 0].min()
us = lambda v: round((int(v) - int(t0)) / 1000.0, 2) if v else None  # noqa: E731
ids = [b for b in range(1024) if ts[b, 0, 0] != 0]
for b in ids[:1]:
    print("CTA", b)
    for t in range(30):
        print(t, [us(v) for v in ts[b, t]])
d = ts.astype(np.float64)
ok = (d[ids, 1:, 0] > 0)
srch = (d[ids, :, 1] - d[ids, :, 0])[:, 1:][ok] / 1000
wait = (d[ids, :, 2] - d[ids, :, 1])[:, 1:][ok] / 1000
per = (d[ids, 1:, 0] - d[ids, :-1, 0])[ok] / 1000
tma = (d[ids, :, 3] - d[ids, :, 2])[:, 1:][ok] / 1000
print("producer per-tile period us: median %.2f" % np.median(per))
print("  search us: median %.2f p90 %.2f" % (np.median(srch), np.percentile(srch, 90)))
print("  empty wait us: median %.2f p90 %.2f" % (np.median(wait), np.percentile(wait, 90)))
print("  issue->rows done us: median %.2f p90 %.2f" % (np.median(tma), np.percentile(tma, 90)))
ends = []
for b in ids:
    last = ts[b, :, 5][ts[b, :, 5] > 0]
    ends.append((last.max() - t0) / 1000 if last.size else 0)
ends = np.array(ends)
print("CTA end (first 30 tiles) us: p10 %.1f p50 %.1f p90 %.1f max %.1f" % tuple(np.percentile(ends, [10, 50, 90, 100])))
sb = ids[int(np.argmax(ends))]
print("slowest CTA", sb, "SM?")
for t in range(0, 30, 2):
    print(t, [us(v) for v in ts[sb, t]])
order = np.argsort(ends)[::-1]
print("slowest 16 CTAs:", [(int(ids[i]), round(float(ends[i]), 1)) for i in order[:16]])
idsa = np.array(ids)
print("mean end blockIdx<G/2: %.1f  >=G/2: %.1f" % (ends[idsa < len(ids) // 2].mean(), ends[idsa >= len(ids) // 2].mean()))
nslow = int((ends > np.median(ends) * 1.3).sum())
print("CTAs >1.3x median:", nslow, "of", len(ids))
