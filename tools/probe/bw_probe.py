"""Read-bandwidth probe on the GPU (measurement aid): LDG.128 streaming vs a
TMA bulk-copy ring, 2 GiB buffer, CUDA events."""
import ctypes
import json
import os
import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
if not os.path.exists(os.path.join(_HERE, "bw_probe.so")):
    import subprocess
    subprocess.check_call(["/usr/local/cuda/bin/nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-shared",
                           "-Xcompiler", "-fPIC", "-o", os.path.join(_HERE, "bw_probe.so"),
                           os.path.join(_HERE, "bw_probe.cu")])
L = ctypes.CDLL(os.path.join(_HERE, "bw_probe.so"))
nbytes = 2 << 30
a = torch.ones(nbytes // 4, dtype=torch.int32, device="cuda")
out = torch.zeros(1, dtype=torch.int64, device="cuda")
s = torch.cuda.current_stream().cuda_stream


def timeit(fn, reps=10):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / reps
    return nbytes / (ms * 1e-3) / 1e9


res = {}
for blocks, threads in [(148 * 4, 512), (148 * 8, 256), (148 * 16, 256)]:
    res[f"ldg b{blocks} t{threads}"] = timeit(lambda: L.probe_ldg(ctypes.c_void_p(a.data_ptr()), ctypes.c_longlong(nbytes), blocks, threads, ctypes.c_void_p(out.data_ptr()), ctypes.c_void_p(s)))
for per_sm, chunk, st in [(1, 65536, 2), (1, 65536, 3), (1, 32768, 4), (1, 16384, 8), (2, 32768, 2), (2, 16384, 4), (4, 16384, 2), (4, 8192, 4), (1, 98304, 2), (8, 8192, 2)]:
    blocks = 148 * per_sm
    res[f"tma ctas/sm={per_sm} chunk={chunk} st={st}"] = timeit(lambda: L.probe_tma(ctypes.c_void_p(a.data_ptr()), ctypes.c_longlong(nbytes), blocks, 64, chunk, st, ctypes.c_void_p(out.data_ptr()), ctypes.c_void_p(s)))
for k, v in res.items():
    print(f"{k:40s} {v:8.1f} GB/s")
