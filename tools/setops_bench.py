"""Set-operation throughput on B200 (the paper's Fig 2): union of
two sorted lists with the inputs split evenly, keys-32 / keys-64 / pairs-32 /
pairs-64, 10^4 .. 10^8 total inputs; inputs processed per second and the
HBM fraction of the algorithmic bytes (read every input once, write every
output once).  CUDA events around the public call: "sync" = the call that
returns the result size (one host round trip per call), "async" = the
stream-ordered form (size left on the device; calls queued back to back),
"graph" = the async form captured once in a CUDA graph and replayed (the
device-side rate without per-call host work).
Measurement aid, not the bench line."""
import json
import sys
from pathlib import Path

import numpy as np
import torch

ROOT = Path(__file__).resolve().parent.parent
sys.path.insert(0, str(ROOT))
import paper_conf_ipps_daltonbmog15_b200 as msp  # noqa: E402

HBM = json.loads((ROOT / "MEASURED_PEAKS.json").read_text())["hbm_gbs"] if (ROOT / "MEASURED_PEAKS.json").exists() \
    else 6650.0


def main():
    out = []
    g = torch.Generator(device="cuda").manual_seed(1)
    for kind, kdt, vdt in [("keys-32", torch.int32, None), ("keys-64", torch.int64, None),
                           ("pairs-32", torch.int32, torch.int32), ("pairs-64", torch.int64, torch.int64)]:
        for total in [10**4, 10**5, 10**6, 10**7, 10**8]:
            n = total // 2
            hi = 2**30
            a = torch.sort(torch.randint(0, hi, (n,), device="cuda", generator=g, dtype=kdt))[0]
            b = torch.sort(torch.randint(0, hi, (n,), device="cuda", generator=g, dtype=kdt))[0]
            av = bv = None
            if vdt is not None:
                av = torch.arange(n, device="cuda", dtype=vdt)
                bv = torch.arange(n, device="cuda", dtype=vdt)
            for mode in ("sync", "async", "graph"):
                call = (lambda: msp.set_operation("union", a, b, av, bv)) if mode == "sync" else \
                    (lambda: msp.set_operation("union", a, b, av, bv, sync=False))
                for _ in range(3):
                    res = call()
                torch.cuda.synchronize()
                if mode == "graph":  # the async call captured once, replayed: no host work per call
                    graph = torch.cuda.CUDAGraph()
                    with torch.cuda.graph(graph):
                        cres = call()
                    call = graph.replay
                    for _ in range(3):
                        call()
                    torch.cuda.synchronize()
                reps = 20 if total <= 10**7 else 5
                e0 = torch.cuda.Event(enable_timing=True)
                e1 = torch.cuda.Event(enable_timing=True)
                e0.record()
                for _ in range(reps):
                    res = call()
                e1.record()
                torch.cuda.synchronize()
                ms = e0.elapsed_time(e1) / reps
                if mode == "graph":
                    res = cres
                nout = res[0].numel() if mode == "sync" else int(res[2][0].item())
                w = a.element_size() + (av.element_size() if av is not None else 0)
                by = (2 * n + nout) * w
                r = {"kind": kind, "mode": mode, "inputs": 2 * n, "outputs": nout, "ms": ms,
                     "inputs_per_s": 2 * n / (ms * 1e-3), "GB_s": by / (ms * 1e-3) / 1e9,
                     "frac_hbm": by / (ms * 1e-3) / 1e9 / HBM}
                out.append(r)
                print(json.dumps(r), flush=True)
    if len(sys.argv) > 1:
        Path(sys.argv[1]).write_text(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
