"""SpGEMM ablation: the shipped pipeline (merge sort by
(row, col), rows kept inside tiles) vs the paper's radix pipeline (radix by
column per tile, 16-bit permutations, global radix sort, re-expansion), per
phase with CUDA events; parity of the radix result on sampled rows.

    python tools/spgemm_compare.py C1 C2 C4 [--json out.json]
Fig 4 knobs (environment, read once per process): MSP_RX_SORT_BITS,
MSP_RX_TWO_PASS."""
import json
import sys

import numpy as np
import torch

sys.path.insert(0, __import__("os").path.dirname(__file__) + "/..")
import gen  # noqa: E402
import oracle  # noqa: E402
import paper_conf_ipps_daltonbmog15_b200 as msp  # noqa: E402


def timed_plan(cls, dA, reps):
    rec = []
    for i in range(reps + 2):
        e = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
        e[0].record()
        p = cls(dA, dA)
        p.setup()
        e[1].record()
        p.symbolic()
        e[2].record()
        C = p.numeric()
        e[3].record()
        if i >= 2:
            rec.append(e)
    torch.cuda.synchronize()
    ph = [float(np.mean([r[k].elapsed_time(r[k + 1]) for r in rec])) for k in range(3)]
    return {"setup_ms": ph[0], "symbolic_ms": ph[1], "numeric_ms": ph[2], "total_ms": sum(ph)}, p, C


def main():
    out = {}
    argv = sys.argv[1:]
    if "--json" in argv:
        argv = argv[:argv.index("--json")] + argv[argv.index("--json") + 2:]
    cfgs = [a for a in argv if not a.startswith("--")]
    for cfg in cfgs:
        scale = 1.0
        if ":" in cfg:
            cfg, sc = cfg.split(":")
            scale = float(sc)
        A = gen.config(cfg, "random", scale=scale)
        dA = msp.CsrTensor.from_arrays(A.rp, A.col, A.val, (A.m, A.n), "cuda")
        reps = 3 if A.nnz > 1e7 else 10
        ship, p1, C1 = timed_plan(msp.SpGemmPlan, dA, reps)
        rad, p2, C2 = timed_plan(msp.SpGemmRadixPlan, dA, reps)
        rows = np.unique(np.random.default_rng(0).integers(0, A.m, 300))
        off, wcol, wval, sc = oracle.spgemm_rows(A, A, rows)
        rp, col, val = C2.numpy()
        ok = True
        for k, r in enumerate(rows):
            a, b = rp[r], rp[r + 1]
            ok &= bool(np.array_equal(col[a:b], wcol[off[k]:off[k + 1]]))
            ok &= oracle.check_values(val[a:b], wval[off[k]:off[k + 1]], sc[off[k]:off[k + 1]], A.val.dtype)[0]
        same = bool(np.array_equal(C1.numpy()[0], rp) and np.array_equal(C1.numpy()[1], col))
        npr = p1.nprods
        out[f"{cfg}@{scale}"] = {"nprods": npr, "nnz_c": C1.nnz, "shipped": ship, "radix": rad,
                                 "radix_over_shipped": rad["total_ms"] / ship["total_ms"],
                                 "shipped_products_per_s": npr / ship["total_ms"] * 1e3,
                                 "radix_products_per_s": npr / rad["total_ms"] * 1e3,
                                 "radix_parity_sampled": ok, "same_structure": same}
        print(cfg, json.dumps(out[f"{cfg}@{scale}"]), flush=True)
        del dA, p1, p2, C1, C2
        torch.cuda.empty_cache()
    if "--json" in sys.argv:
        json.dump(out, open(sys.argv[sys.argv.index("--json") + 1], "w"), indent=1)


if __name__ == "__main__":
    main()
