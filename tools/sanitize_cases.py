"""Small invocations of every libmsp kernel for compute-sanitizer
(memcheck / racecheck / synccheck): SpMV (warp-tile kernel on a 27-point
stencil, CTA-tile transpose walk on irregular rows, empty rows, a long row),
SpAdd (two-phase and one-pass), SpGEMM (short and long rows, 32- and 64-bit
keys, the short-row accumulator), set operations (keys / pairs, all four
ops, the async form), csr_check and the row-offset rebase.
Run: compute-sanitizer --tool memcheck python tools/sanitize_cases.py"""
import sys

import numpy as np
import torch

sys.path.insert(0, __import__("os").path.dirname(__file__) + "/..")
import gen  # noqa: E402
import paper_conf_ipps_daltonbmog15_b200 as msp  # noqa: E402


def dev(A):
    return msp.CsrTensor.from_arrays(A.rp, A.col, A.val, (A.m, A.n), "cuda")


def main():
    A27 = gen.poisson3d_27pt(14)
    A27 = A27.with_values(gen.matrices.random_values(A27.nnz, 1))
    cases = [A27, gen.config("C1", "random"), gen.config("C4", "random", scale=0.002),
             gen.random_csr(700, 700, 3, density=0.02, empty_frac=0.5, dense_rows=2, mode="random"),
             gen.config("C3", "random", scale=1 / 1024)]
    for A in cases:
        dA = dev(A)
        x = torch.as_tensor(gen.x_vector(A.n, "random", dtype=A.val.dtype), device="cuda")
        msp.spmv(dA, x)
        T = gen.transpose(A)
        msp.spadd(dA, dev(T))
        msp.spadd_fused(dA, dev(T))
        if A.m == A.n and A.nnz < 200_000:
            msp.spgemm(dA, dA)
        msp.csr_check(dA)
    # 64-bit SpGEMM keys (row span > 2^(32-22))
    rng = np.random.default_rng(1)
    m, k, n = 3000, 200, 1 << 22
    lens = np.where(np.arange(m) % 7 == 0, rng.integers(1, 3, m), 0)
    rp = np.concatenate([[0], np.cumsum(lens)]).astype(np.int32)
    col = np.concatenate([np.sort(rng.choice(k, size=int(L), replace=False)) for L in lens]).astype(np.int32)
    A = gen.CSR(m, k, rp, col, gen.matrices.random_values(col.size, 2))
    bl = rng.integers(0, 4, k)
    brp = np.concatenate([[0], np.cumsum(bl)]).astype(np.int32)
    bcol = np.concatenate([np.sort(rng.choice(n, size=int(L), replace=False)) for L in bl]).astype(np.int32)
    B = gen.CSR(k, n, brp, bcol, gen.matrices.random_values(bcol.size, 3))
    msp.spgemm(dev(A), dev(B))
    # SpGEMM row accumulator with > 512 output columns per row (several passes), B rows > 32
    bl = np.where(rng.random(300) < 0.1, 0, rng.integers(1, 70, 300))
    brp = np.concatenate([[0], np.cumsum(bl)]).astype(np.int32)
    bcol = np.concatenate([np.sort(rng.choice(60_000, size=int(L), replace=False)) for L in bl]).astype(np.int32)
    B = gen.CSR(300, 60_000, brp, bcol, gen.matrices.random_values(bcol.size, 4))
    al = rng.integers(1, 30, 200)
    arp = np.concatenate([[0], np.cumsum(al)]).astype(np.int32)
    acol = np.concatenate([np.sort(rng.choice(300, size=int(L), replace=False)) for L in al]).astype(np.int32)
    A = gen.CSR(200, 300, arp, acol, gen.matrices.random_values(acol.size, 5))
    msp.spgemm(dev(A), dev(B))
    # set operations
    a = np.sort(rng.integers(0, 500, 20000)).astype(np.int32)
    b = np.sort(rng.integers(0, 500, 15000)).astype(np.int32)
    for op in ("union", "intersection", "difference", "symmetric_difference"):
        msp.set_operation(op, torch.from_numpy(a).cuda(), torch.from_numpy(b).cuda())
        msp.set_operation(op, torch.from_numpy(a.astype(np.int64)).cuda(), torch.from_numpy(b.astype(np.int64)).cuda(),
                          torch.from_numpy(a.astype(np.float64)).cuda(), torch.from_numpy(b.astype(np.float64)).cuda())
        msp.set_operation(op, torch.from_numpy(a).cuda(), torch.from_numpy(b).cuda(), sync=False)
    msp.rebase_offsets(torch.arange(10, dtype=torch.int32, device="cuda"), 5)
    torch.cuda.synchronize()
    print("sanitize cases done", msp.lib().msp_launch_count(), "launches")


if __name__ == "__main__":
    main()
