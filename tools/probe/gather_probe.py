"""Random-gather probe (measurement aid for C5 SpMV): m outputs,
each the sum of 4 random doubles of x (n doubles); time per gather and, under
ncu, DRAM bytes per gather, per cache operator.

    python tools/probe/gather_probe.py [n_log2 ...]
"""
import ctypes
import json
import os
import subprocess
import sys

import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
so = "/tmp/gather_probe.so"
subprocess.check_call(["/usr/local/cuda/bin/nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-shared",
                       "-Xcompiler", "-fPIC", "-o", so, os.path.join(_HERE, "gather_probe.cu")])
L = ctypes.CDLL(so)
s = torch.cuda.current_stream().cuda_stream
m = 100_000_000
idx = torch.empty(4 * m, dtype=torch.int32, device="cuda")
y = torch.empty(m, dtype=torch.float64, device="cuda")
names = ["ldg", "ldcg", "nc.L1::no_allocate", "nc.L2::64B", "nc.L2::cache_hint(0)"]
reps = int(os.environ.get("REPS", "5"))
if os.environ.get("CSR"):  # the column stream of a BJ config instead of uniform random indices
    sys.path.insert(0, os.path.dirname(os.path.dirname(_HERE)))
    import gen
    A = gen.config(os.environ["CSR"], "int")
    m = A.nnz // 4
    idx = torch.as_tensor(A.col[:4 * m], device="cuda")
    y = torch.empty(m, dtype=torch.float64, device="cuda")
    x = torch.ones(A.n, dtype=torch.float64, device="cuda")
    for mode in range(5):
        for blocks in (148 * 8, 148 * 32):
            f = lambda: L.probe_gather(mode, ctypes.c_void_p(idx.data_ptr()), ctypes.c_void_p(x.data_ptr()),  # noqa
                                       ctypes.c_void_p(y.data_ptr()), ctypes.c_longlong(m), blocks, ctypes.c_void_p(s))
            f()
            torch.cuda.synchronize()
            e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
            e0.record()
            for _ in range(reps):
                f()
            e1.record()
            torch.cuda.synchronize()
            ms = e0.elapsed_time(e1) / reps
            print(json.dumps({"csr": os.environ["CSR"], "nnz": 4 * m, "x_MB": A.n * 8 / 1e6, "mode": names[mode],
                              "blocks": blocks, "us": round(ms * 1e3, 1)}), flush=True)
    sys.exit(0)
for lg in [int(a) for a in sys.argv[1:]] or [20, 23, 26, 27]:
    n = 1 << lg
    x = torch.ones(n, dtype=torch.float64, device="cuda")
    L.probe_fill(ctypes.c_void_p(idx.data_ptr()), ctypes.c_longlong(4 * m), ctypes.c_uint(n), ctypes.c_uint(lg), ctypes.c_void_p(s))
    for mode in range(5):
        for blocks in (148 * 8, 148 * 32):
            f = lambda: L.probe_gather(mode, ctypes.c_void_p(idx.data_ptr()), ctypes.c_void_p(x.data_ptr()),  # noqa
                                       ctypes.c_void_p(y.data_ptr()), ctypes.c_longlong(m), blocks, ctypes.c_void_p(s))
            f()
            torch.cuda.synchronize()
            e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
            e0.record()
            for _ in range(reps):
                f()
            e1.record()
            torch.cuda.synchronize()
            ms = e0.elapsed_time(e1) / reps
            print(json.dumps({"x_MB": n * 8 / 1e6, "mode": names[mode], "blocks": blocks, "ms": round(ms, 3),
                              "ns_per_gather": round(ms * 1e6 / (4 * m), 4),
                              "idx_y_GBs": round((16 * m + 8 * m) / ms / 1e6, 1)}), flush=True)
    del x
