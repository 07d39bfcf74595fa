"""Runs one libmsp operation on a configuration once (profiling driver for
ncu: `ncu ... python tools/run_op.py spgemm C2`)."""
import sys

import torch

sys.path.insert(0, __import__("os").path.dirname(__file__) + "/..")
import gen  # noqa: E402
import paper_conf_ipps_daltonbmog15_b200 as msp  # noqa: E402


def main():
    op = sys.argv[1] if len(sys.argv) > 1 else "spgemm"
    cfg = sys.argv[2] if len(sys.argv) > 2 else "C2"
    reps = int(sys.argv[3]) if len(sys.argv) > 3 else 1
    A = gen.config(cfg, "random")
    dA = msp.CsrTensor.from_arrays(A.rp, A.col, A.val, (A.m, A.n), "cuda")
    if op == "spmv":
        x = torch.from_numpy(gen.matrices.x_vector(A.n, "random", dtype=A.val.dtype)).cuda()
        for _ in range(reps):
            msp.spmv(dA, x)
    elif op in ("spadd", "spadd_fused"):
        T = gen.matrices.transpose(A)
        dT = msp.CsrTensor.from_arrays(T.rp, T.col, T.val, (T.m, T.n), "cuda")
        for _ in range(reps):
            (msp.spadd_fused if op == "spadd_fused" else msp.spadd)(dA, dT)
    else:
        for _ in range(reps):
            p = msp.SpGemmPlan(dA, dA)
            p.setup()
            p.symbolic()
            p.numeric()
    torch.cuda.synchronize()
    print("done", op, cfg)


if __name__ == "__main__":
    main()
