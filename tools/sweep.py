"""Five-config sweep at 1 GPU (SURVEY §8(d) "Predictability"): times SpMV,
SpAdd (A + A^T) and SpGEMM (A * A) on the BASELINE.json configs C1..C5,
checks sampled rows against the CPU oracle, and fits time ~ work
(nnz for SpMV, nnzA + nnzB for SpAdd, Nprods for SpGEMM): R^2 and Pearson rho.

    python tools/sweep.py [--configs C1,C2,C3,C4,C5] [--ops spmv,spadd,spgemm] [--out gpurun_out/sweep.json]

Timing: CUDA events on the launching stream, 3 warm-ups, mean of 20 (SpMV,
SpAdd) or 5 (SpGEMM) launches; the SpAdd / SpGEMM times cover the whole
public call (symbolic with its nnz(C) read-back, allocation, numeric).
Tuning/evidence tool: not the bench line (bench.py is).
"""
from __future__ import annotations

import argparse
import json
import sys
import time
from pathlib import Path

import numpy as np
import torch

ROOT = Path(__file__).resolve().parent.parent
sys.path.insert(0, str(ROOT))
import gen  # noqa: E402
import oracle  # noqa: E402  (parity samples only)
import paper_conf_ipps_daltonbmog15_b200 as msp  # noqa: E402

HBM = json.loads((ROOT / "MEASURED_PEAKS.json").read_text())["hbm_gbs"] if (ROOT / "MEASURED_PEAKS.json").exists() \
    else 6650.0
OPS = {"C1": "spmv,spadd,spgemm", "C2": "spmv,spgemm", "C3": "spmv,spadd", "C4": "spmv,spgemm",
       "C5": "spmv,spgemm"}


def timed(fn, reps, warm=3):
    for _ in range(warm):
        fn()
    torch.cuda.synchronize()
    evs = []
    for _ in range(reps):
        a = torch.cuda.Event(enable_timing=True)
        b = torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        evs.append((a, b))
    torch.cuda.synchronize()
    return float(np.mean([a.elapsed_time(b) for a, b in evs]))


def fit(xs, ys):
    x = np.asarray(xs, float)
    y = np.asarray(ys, float)
    if x.size < 3:
        return None
    A = np.vstack([x, np.ones_like(x)]).T
    coef, *_ = np.linalg.lstsq(A, y, rcond=None)
    pred = A @ coef
    ss_res = float(np.sum((y - pred) ** 2))
    ss_tot = float(np.sum((y - y.mean()) ** 2))
    return {"r2": 1 - ss_res / ss_tot if ss_tot > 0 else 1.0, "rho": float(np.corrcoef(x, y)[0, 1]),
            "slope_ms_per_unit": float(coef[0]), "intercept_ms": float(coef[1]), "n": int(x.size)}


def sample_rows(m, k=4000, seed=0):
    if m == 0:
        return np.zeros(0, np.int64)
    rng = np.random.default_rng(seed)
    r = np.unique(np.concatenate([rng.integers(0, m, size=k), [0, m - 1]]))
    return r.astype(np.int64)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", default="C1,C2,C3,C4,C5")
    ap.add_argument("--ops", default="spmv,spadd,spgemm")
    ap.add_argument("--out", default=str(ROOT / "gpurun_out" / "sweep.json"))
    args = ap.parse_args()
    want_ops = set(args.ops.split(","))
    res = {"hbm_peak_gbs": HBM, "configs": {}}
    for cfg in args.configs.split(","):
        t0 = time.time()
        A = gen.config(cfg, "random")
        gen_s = time.time() - t0
        vs = A.val.dtype.itemsize
        ent = {"m": A.m, "nnz": A.nnz, "dtype": str(A.val.dtype), "gen_s": gen_s}
        dA = msp.CsrTensor.from_arrays(A.rp, A.col, A.val, (A.m, A.n), "cuda")
        ops = set(OPS[cfg].split(",")) & want_ops
        if "spmv" in ops:
            x = gen.x_vector(A.n, "random", seed=1000 + int(cfg[1]), dtype=A.val.dtype)
            dx = torch.as_tensor(x, device="cuda")
            y = torch.empty(A.m, dtype=dx.dtype, device="cuda")
            ms = timed(lambda: msp.spmv(dA, dx, out=y), 20)
            by = A.nnz * (4 + vs) + A.m * (4 + vs) + 4 + A.n * vs
            rows = sample_rows(A.m)
            want, scale = oracle.spmv(A, x, rows)
            ok, msg = oracle.check_values(y.cpu().numpy()[rows], want, scale, A.val.dtype)
            ent["spmv"] = {"ms": ms, "alg_bytes": by, "GB_s": by / ms / 1e6, "frac_hbm": by / ms / 1e6 / HBM,
                           "GFLOP_s": 2 * A.nnz / ms / 1e6, "parity_rows": int(rows.size), "parity": ok,
                           "msg": msg}
            del dx, y
        if "spadd" in ops:
            T = gen.transpose(A)
            dT = msp.CsrTensor.from_arrays(T.rp, T.col, T.val, (T.m, T.n), "cuda")
            C = msp.spadd(dA, dT)
            ms = timed(lambda: msp.spadd(dA, dT), 10)
            rows = sample_rows(A.m, 2000)
            woff, wcol, wval = oracle.spadd_rows(A, T, rows)
            rp, col, val = C.numpy()
            ok = True
            for k, r in enumerate(rows):
                a, b = rp[r], rp[r + 1]
                wa, wb = woff[k], woff[k + 1]
                ok &= bool(np.array_equal(col[a:b], wcol[wa:wb]) and np.array_equal(val[a:b], wval[wa:wb]))
            ok &= int(rp[-1]) == C.nnz
            by = (A.nnz + T.nnz) * (4 + vs) + C.nnz * (4 + vs) + 3 * 4 * (A.m + 1)
            ent["spadd"] = {"ms": ms, "input_nnz": A.nnz + T.nnz, "nnz_c": C.nnz,
                            "input_nnz_per_s": (A.nnz + T.nnz) / ms * 1e3, "alg_bytes": by,
                            "GB_s": by / ms / 1e6, "parity_rows": int(rows.size), "parity": ok}
            del dT, C
        if "spgemm" in ops:
            try:
                P = msp.SpGemmPlan(dA, dA)
                P.setup()
                P.symbolic()
                C = P.numeric()

                def run():
                    Q = msp.SpGemmPlan(dA, dA)
                    Q.setup()
                    Q.symbolic()
                    Q.numeric()
                ms = timed(run, 5, warm=2)
                rows = sample_rows(A.m, 300)
                woff, wcol, wval, sc = oracle.spgemm_rows(A, A, rows)
                rp, col, val = C.numpy()
                ok, msg = True, ""
                for k, r in enumerate(rows):
                    a, b = rp[r], rp[r + 1]
                    wa, wb = woff[k], woff[k + 1]
                    if not np.array_equal(col[a:b], wcol[wa:wb]):
                        ok, msg = False, f"row {r} structure"
                        break
                    o2, m2 = oracle.check_values(val[a:b], wval[wa:wb], sc[wa:wb], A.val.dtype)
                    if not o2:
                        ok, msg = False, f"row {r}: {m2}"
                        break
                ent["spgemm"] = {"ms": ms, "nprods": int(P.nprods), "nnz_c": int(C.nnz),
                                 "products_per_s": P.nprods / ms * 1e3, "parity_rows": int(rows.size),
                                 "parity": ok, "msg": msg}
                del P, C
            except Exception as e:  # noqa: BLE001  (e.g. workspace larger than HBM)
                ent["spgemm"] = {"error": f"{type(e).__name__}: {e}"[:300]}
        torch.cuda.empty_cache()
        res["configs"][cfg] = ent
        print(cfg, json.dumps(ent), flush=True)
    cf = res["configs"]
    for op, unit in (("spmv", "nnz"), ("spadd", "input_nnz"), ("spgemm", "nprods")):
        pts = [(v[op][unit] if unit != "nnz" else v["nnz"], v[op]["ms"]) for v in cf.values()
               if op in v and "ms" in v[op]]
        if len(pts) >= 3:
            res[f"fit_{op}"] = fit([p[0] for p in pts], [p[1] for p in pts])
    Path(args.out).parent.mkdir(parents=True, exist_ok=True)
    Path(args.out).write_text(json.dumps(res, indent=1))
    print(json.dumps({k: v for k, v in res.items() if k.startswith("fit")}))


if __name__ == "__main__":
    main()
