"""Runs one set operation a few times (profiling driver for ncu:
`ncu ... python tools/run_setop.py union keys-32 100000000 3`)."""
import sys

import torch

sys.path.insert(0, __import__("os").path.dirname(__file__) + "/..")
import paper_conf_ipps_daltonbmog15_b200 as msp  # noqa: E402

KINDS = {"keys-32": (torch.int32, None), "keys-64": (torch.int64, None),
         "pairs-32": (torch.int32, torch.int32), "pairs-64": (torch.int64, torch.int64)}


def main():
    op = sys.argv[1] if len(sys.argv) > 1 else "union"
    kdt, vdt = KINDS[sys.argv[2] if len(sys.argv) > 2 else "keys-32"]
    total = int(sys.argv[3]) if len(sys.argv) > 3 else 10**8
    reps = int(sys.argv[4]) if len(sys.argv) > 4 else 3
    g = torch.Generator(device="cuda").manual_seed(1)
    n = total // 2
    a = torch.sort(torch.randint(0, 2**30, (n,), device="cuda", generator=g, dtype=kdt))[0]
    b = torch.sort(torch.randint(0, 2**30, (n,), device="cuda", generator=g, dtype=kdt))[0]
    av = torch.arange(n, device="cuda", dtype=vdt) if vdt else None
    bv = torch.arange(n, device="cuda", dtype=vdt) if vdt else None
    for _ in range(reps):
        msp.set_operation(op, a, b, av, bv)
    torch.cuda.synchronize()


if __name__ == "__main__":
    main()
