"""Predictability sweep: SpMV time vs nnz,
SpAdd (A + A^T) time vs nnzA + nnzB and SpGEMM (A * A) time vs Nprods over
>= 20 generated matrices of the BJ families -- 27-point stencils 40^3..200^3,
R-MAT scales 16..22, pathological-skew variants (1e5..1e6-nnz dense rows),
random rows 1e6..1e8 -- mirroring the paper's Figs 6 / 8 / 10 (P:1372-1404,
P:1524-1550).  Fits R^2 and Pearson rho per operation, over all
matrices and per family.  CUDA events, warm-up 3; tool, not the bench line.

    python tools/predict_sweep.py [--quick] [--json out.json]"""
import json
import sys
import time

import numpy as np
import torch

sys.path.insert(0, __import__("os").path.dirname(__file__) + "/..")
import gen  # noqa: E402
import paper_conf_ipps_daltonbmog15_b200 as msp  # noqa: E402


def fit(x, y):
    x, y = np.asarray(x, float), np.asarray(y, float)
    if x.size < 3:
        return None
    A = np.vstack([x, np.ones_like(x)]).T
    c, *_ = np.linalg.lstsq(A, y, rcond=None)
    pred = A @ c
    ss = float(np.sum((y - y.mean()) ** 2))
    return {"r2": 1 - float(np.sum((y - pred) ** 2)) / ss if ss > 0 else 1.0,
            "rho": float(np.corrcoef(x, y)[0, 1]), "n": int(x.size)}


def timed(fn, reps):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    ev = []
    for _ in range(reps):
        a = torch.cuda.Event(enable_timing=True); b = torch.cuda.Event(enable_timing=True)
        a.record(); fn(); b.record()
        ev.append((a, b))
    torch.cuda.synchronize()
    return float(np.median([a.elapsed_time(b) for a, b in ev]))


def matrices(quick):
    for k in ([40, 80, 120] if quick else [40, 60, 80, 100, 120, 160, 200]):
        A = gen.poisson3d_27pt(k)
        yield "stencil27", f"27pt {k}^3", A.with_values(gen.matrices.random_values(A.nnz, k))
    for sc in ([16, 18, 20] if quick else [16, 17, 18, 19, 20, 21, 22]):
        A = gen.rmat(sc, 16, seed=22)
        yield "rmat", f"rmat s{sc}", A.with_values(gen.matrices.random_values(A.nnz, sc, np.float32))
    for s in ([0.05, 0.5] if quick else [0.05, 0.1, 0.25, 0.5, 1.0]):
        A = gen.config("C4", "random", scale=s)
        yield "skew", f"skew {s}", A
    for n in ([10**6, 10**7] if quick else [10**6, 3 * 10**6, 10**7, 3 * 10**7, 10**8]):
        A = gen.random_rows(n)
        yield "randrows", f"randrows {n:.0e}", A.with_values(gen.matrices.random_values(A.nnz, 5))


def main():
    quick = "--quick" in sys.argv
    res = []
    for fam, name, A in matrices(quick):
        t0 = time.time()
        dA = msp.CsrTensor.from_arrays(A.rp, A.col, A.val, (A.m, A.n), "cuda")
        x = torch.as_tensor(gen.x_vector(A.n, "random", seed=1, dtype=A.val.dtype), device="cuda")
        y = torch.empty(A.m, dtype=x.dtype, device="cuda")
        ent = {"family": fam, "name": name, "m": A.m, "nnz": A.nnz}
        ent["spmv_ms"] = timed(lambda: msp.spmv(dA, x, out=y), 20)
        if fam in ("rmat", "stencil27", "skew") and A.nnz < 8e7:
            T = gen.transpose(A)
            dT = msp.CsrTensor.from_arrays(T.rp, T.col, T.val, (T.m, T.n), "cuda")
            ent["spadd_in"] = A.nnz + T.nnz
            ent["spadd_ms"] = timed(lambda: msp.spadd(dA, dT), 5)
            del dT
        if fam in ("stencil27", "skew", "randrows") and A.nnz < 1.1e8:
            p = msp.SpGemmPlan(dA, dA)
            info = p.setup()
            if info.nprods < 8e8:
                def g():
                    q = msp.SpGemmPlan(dA, dA); q.setup(); q.symbolic(); q.numeric()
                ent["nprods"] = int(info.nprods)
                ent["spgemm_ms"] = timed(g, 3)
        ent["wall_s"] = round(time.time() - t0, 1)
        res.append(ent)
        print(json.dumps(ent), flush=True)
        del dA, x, y
        torch.cuda.empty_cache()
    out = {"matrices": res, "fits": {}}
    for op, key in (("spmv", "nnz"), ("spadd", "spadd_in"), ("spgemm", "nprods")):
        pts = [(e[key], e[f"{op}_ms"]) for e in res if f"{op}_ms" in e]
        if pts:
            out["fits"][op] = {"all": fit(*zip(*pts))}
            for fam in sorted({e["family"] for e in res}):
                fp = [(e[key], e[f"{op}_ms"]) for e in res if f"{op}_ms" in e and e["family"] == fam]
                if len(fp) >= 3:
                    out["fits"][op][fam] = fit(*zip(*fp))
    print(json.dumps(out["fits"]))
    if "--json" in sys.argv:
        json.dump(out, open(sys.argv[sys.argv.index("--json") + 1], "w"), indent=1)


if __name__ == "__main__":
    main()
