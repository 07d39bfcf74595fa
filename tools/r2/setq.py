import sys, json, torch, numpy as np
sys.path.insert(0, '.')
import paper_conf_ipps_daltonbmog15_b200 as msp
g = torch.Generator(device="cuda").manual_seed(1)
res = []
for kind, kdt, vdt in [("keys-32", torch.int32, None), ("pairs-64", torch.int64, torch.int64)]:
    n = 10**8 // 2
    a = torch.sort(torch.randint(0, 2**30, (n,), device="cuda", generator=g, dtype=kdt))[0]
    b = torch.sort(torch.randint(0, 2**30, (n,), device="cuda", generator=g, dtype=kdt))[0]
    av = bv = None
    if vdt is not None:
        av = torch.arange(n, device="cuda", dtype=vdt); bv = torch.arange(n, device="cuda", dtype=vdt)
    for _ in range(3): msp.set_operation("union", a, b, av, bv)
    torch.cuda.synchronize()
    ts = []
    for _ in range(10):
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(); msp.set_operation("union", a, b, av, bv); e1.record(); ts.append((e0, e1))
    torch.cuda.synchronize()
    res.append((kind, float(np.mean([x.elapsed_time(y) for x, y in ts]))))
print(json.dumps({"cfg": sys.argv[1] if len(sys.argv) > 1 else "default", "ms": res}))
