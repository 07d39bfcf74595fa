"""SpGEMM per-phase timing (CUDA events) of the shipped path on BJ configs,
with the path taken (info fields).  Env ablations are read once per
process, so compare settings across separate runs:

    python tools/spgemm_phases.py C4 C5 [--reps N]
    MSP_SPGEMM_SMALL=0 python tools/spgemm_phases.py C4 C5"""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(__file__) + "/..")
import gen  # noqa: E402
import oracle  # noqa: E402
import paper_conf_ipps_daltonbmog15_b200 as msp  # noqa: E402


def main():
    argv = sys.argv[1:]
    reps = 3
    if "--reps" in argv:
        reps = int(argv[argv.index("--reps") + 1])
        argv = argv[:argv.index("--reps")] + argv[argv.index("--reps") + 2:]
    for cfg in argv:
        A = gen.config(cfg, "random")
        dA = msp.CsrTensor.from_arrays(A.rp, A.col, A.val, (A.m, A.n), "cuda")
        rec = []
        oc = ov = None  # C preallocated after the first (untimed) call, as bench.py does
        for i in range(reps + 1):
            e = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
            p = msp.SpGemmPlan(dA, dA)
            torch.cuda.synchronize()
            e[0].record()
            p.setup()
            e[1].record()
            p.symbolic()
            e[2].record()
            C = p.numeric(col=oc, val=ov)
            e[3].record()
            if oc is None:
                oc, ov = C.col, C.val
            torch.cuda.synchronize()
            if i >= 1:
                rec.append([e[k].elapsed_time(e[k + 1]) for k in range(3)])
        ph = np.mean(np.array(rec), axis=0)
        info = p.info
        rows = np.unique(np.random.default_rng(0).integers(0, A.m, 400))
        off, wcol, wval, sc = oracle.spgemm_rows(A, A, rows)
        rp, col, val = C.numpy()
        ok = True
        for k, r in enumerate(rows):
            a, b = rp[r], rp[r + 1]
            if b - a != off[k + 1] - off[k] or not np.array_equal(col[a:b], wcol[off[k]:off[k + 1]]):
                ok = False
                break
            good, _ = oracle.check_values(val[a:b], wval[off[k]:off[k + 1]], sc[off[k]:off[k + 1]], A.val.dtype)
            ok = ok and good
        res = {"cfg": cfg, "setup_ms": ph[0], "symbolic_ms": ph[1], "numeric_ms": ph[2], "total_ms": float(ph.sum()),
               "Gprod_s": info.nprods / ph.sum() / 1e6, "nprods": int(info.nprods),
               "small_rows": int(info.small_rows), "bitmap_rows": int(info.bitmap_rows),
               "long_rows": int(info.long_rows), "ntiles": int(info.ntiles), "rowacc": int(info.row_accumulator),
               "sampled_parity": ok,
               "env": {k: v for k, v in os.environ.items() if k.startswith("MSP_")}}
        print(json.dumps(res), flush=True)
        del C, p, dA


if __name__ == "__main__":
    main()
