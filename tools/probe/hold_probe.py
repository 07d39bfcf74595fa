"""Bandwidth of a TMA ring vs how long consumers hold each stage (measurement
aid for the SpMV design): 2 GiB read-only stream, CUDA events."""
import ctypes
import os
import subprocess

import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
so = os.path.join(_HERE, "hold_probe.so")
if not os.path.exists(so):
    subprocess.check_call(["/usr/local/cuda/bin/nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-shared",
                           "-Xcompiler", "-fPIC", "-o", so, os.path.join(_HERE, "hold_probe.cu")])
L = ctypes.CDLL(so)
nbytes = 2 << 30
a = torch.ones(nbytes // 4, dtype=torch.int32, device="cuda")
out = torch.zeros(1, dtype=torch.int64, device="cuda")
s = torch.cuda.current_stream().cuda_stream


def bw(blocks, chunk, st, hold, reps=5):
    f = lambda: L.probe_hold(ctypes.c_void_p(a.data_ptr()), ctypes.c_longlong(nbytes), blocks, 64, chunk, st, hold,  # noqa
                             ctypes.c_void_p(out.data_ptr()), ctypes.c_void_p(s))
    for _ in range(2):
        f()
    torch.cuda.synchronize()
    e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        f()
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / reps
    return nbytes / (ms * 1e-3) / 1e9


for per_sm, chunk, st in [(1, 83 * 1024, 2), (1, 41 * 1024, 4), (1, 41 * 1024, 5), (1, 27 * 1024, 7), (2, 41 * 1024, 2),
                          (2, 27 * 1024, 3), (1, 20 * 1024, 10)]:
    row = []
    for hold in (0, 1000, 2000, 3000, 4000, 6000, 8000):
        row.append(f"{bw(148 * per_sm, chunk, st, hold):7.0f}")
    print(f"ctas/sm={per_sm} chunk={chunk // 1024}K st={st}  hold 0/1k/2k/3k/4k/6k/8k cyc: " + " ".join(row), flush=True)
