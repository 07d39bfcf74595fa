"""SpMV tuning sweep (tuning aid, not a bench line): times msp.spmv on a
configuration under several MSP_SPMV_* launch settings, each in its own
process (the library reads the settings once).

    python tools/spmv_tune.py C2 "CFG=0" "K=27,NW=4" "K=27,NW=8" ...
"""
import json
import os
import subprocess
import sys

CHILD = r"""
import sys, json, numpy as np, torch
sys.path.insert(0, '.')
import gen, paper_conf_ipps_daltonbmog15_b200 as msp
import os
cfg = sys.argv[1]
cache = f'/tmp/msp_tune_{cfg}.npz'
if os.path.exists(cache):
    z = np.load(cache)
    A = gen.CSR(int(z['m']), int(z['n']), z['rp'], z['col'], z['val'])
else:
    A = gen.config(cfg, 'random')
    np.savez(cache, m=A.m, n=A.n, rp=A.rp, col=A.col, val=A.val)
if os.environ.get('TUNE_DTYPE'):  # same structure, other value type (tuning aid)
    A = gen.CSR(A.m, A.n, A.rp, A.col, A.val.astype(os.environ['TUNE_DTYPE']))
x = gen.x_vector(A.n, 'random', seed=1000 + int(cfg[1]), dtype=A.val.dtype)
dA = msp.CsrTensor.from_arrays(A.rp, A.col, A.val, (A.m, A.n), 'cuda')
dx = torch.as_tensor(x, device='cuda')
y = torch.empty(A.m, dtype=dx.dtype, device='cuda')
for _ in range(5):
    msp.spmv(dA, dx, out=y)
torch.cuda.synchronize()
ts = []
for _ in range(50):
    a = torch.cuda.Event(enable_timing=True); b = torch.cuda.Event(enable_timing=True)
    a.record(); msp.spmv(dA, dx, out=y); b.record()
    ts.append((a, b))
torch.cuda.synchronize()
ms = [a.elapsed_time(b) for a, b in ts]
vs = A.val.dtype.itemsize
by = A.nnz * (4 + vs) + A.m * (4 + vs) + 4 + A.n * vs
# parity on rows sampled across the matrix (full check is in tests/)
import oracle
rows = np.unique(np.linspace(0, A.m - 1, 20000).astype(np.int64))
want, scale = oracle.spmv(A, x, rows)
ok, msg = oracle.check_values(y.cpu().numpy()[rows], want, scale, A.val.dtype)
print(json.dumps({"mean_us": 1e3 * float(np.mean(ms)), "min_us": 1e3 * float(np.min(ms)),
                  "GBs_mean": by / (np.mean(ms) * 1e-3) / 1e9, "ok": bool(ok), "msg": msg}))
"""


def main():
    cfg = sys.argv[1]
    out = {}
    for spec in sys.argv[2:]:
        env = dict(os.environ)
        for kv in spec.split(","):
            k, v = kv.split("=")
            env[k if k.startswith("MSP_") else "MSP_SPMV_" + k] = v
        env["MSP_VERBOSE"] = "1"
        r = subprocess.run([sys.executable, "-c", CHILD, cfg], env=env, capture_output=True, text=True)
        line = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
        res = json.loads(line[-1]) if line else {"error": r.stderr[-800:]}
        res["launch"] = [ln for ln in r.stderr.splitlines() if ln.startswith("msp spmv")][:1]
        out[spec] = res
        print(cfg, spec, json.dumps(res), flush=True)
    return out


if __name__ == "__main__":
    main()
