"""Time SpAdd A + A^T on a config under the libmsp named by MSP_LIB (experiment aid)."""
import os, sys, json, numpy as np, torch
sys.path.insert(0, '.')
import gen, oracle
import paper_conf_ipps_daltonbmog15_b200 as msp
cfg = sys.argv[1]
cache = f'/tmp/msp_spadd_{cfg}.npz'
if os.path.exists(cache):
    z = np.load(cache); A = gen.CSR(int(z['m']), int(z['n']), z['rp'], z['col'], z['val'])
else:
    A = gen.config(cfg, 'random'); np.savez(cache, m=A.m, n=A.n, rp=A.rp, col=A.col, val=A.val)
T = gen.matrices.transpose(A)
dA = msp.CsrTensor.from_arrays(A.rp, A.col, A.val, (A.m, A.n), 'cuda')
dT = msp.CsrTensor.from_arrays(T.rp, T.col, T.val, (T.m, T.n), 'cuda')
for _ in range(3): C = msp.spadd(dA, dT)
torch.cuda.synchronize()
ev = []
for _ in range(10):
    a = torch.cuda.Event(enable_timing=True); b = torch.cuda.Event(enable_timing=True)
    a.record(); C = msp.spadd(dA, dT); b.record(); ev.append((a, b))
torch.cuda.synchronize()
ms = float(np.mean([a.elapsed_time(b) for a, b in ev]))
rows = np.unique(np.linspace(0, A.m - 1, 2000).astype(np.int64))
Cc = (C.rp.cpu().numpy(), C.col.cpu().numpy(), C.val.cpu().numpy())
ref = oracle.spadd(A, T)
ok = bool(np.array_equal(Cc[0], ref.rp) and np.array_equal(Cc[1], ref.col) and np.array_equal(Cc[2], ref.val))
print(json.dumps({"lib": os.environ.get("MSP_LIB", "default"), "cfg": cfg, "ms": ms, "exact": ok}))
