"""Multi-process (world size 2, gloo, CPU) tests of the row-block exchange
logic of paper_conf_ipps_daltonbmog15_b200.dist: nnz-balanced row split,
all-gather of x slices, replication of CSR row blocks (B) and concatenation of
C row blocks.  The local products are computed with the oracle here (there is
no GPU); on the GPU box the same functions feed libmsp kernels."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, results):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import gen
        import oracle
        from paper_conf_ipps_daltonbmog15_b200 import CsrTensor
        from paper_conf_ipps_daltonbmog15_b200 import dist as mdist

        A = gen.random_csr(301, 301, 7, density=0.03, empty_frac=0.2, dense_rows=1, mode="random")
        x = gen.x_vector(A.n, "random", seed=3)
        starts = mdist.split_rows(A.rp, world)
        assert np.array_equal(starts, oracle.row_split(A.rp, world))
        r0, r1 = int(starts[rank]), int(starts[rank + 1])
        blk = mdist.row_block(A.rp, A.col, A.val, r0, r1, A.n, device="cpu")
        # --- SpMV exchange: x slices -> full x
        xs = mdist.x_slice_of(torch.as_tensor(x), rank, world)
        xf = mdist.allgather_x(xs, A.n)
        assert np.array_equal(xf.numpy(), x)
        Ab = gen.CSR(r1 - r0, A.n, *[t.numpy() for t in (blk.rp, blk.col, blk.val)])
        y_loc, _ = oracle.spmv(Ab, xf.numpy())
        y = mdist.allgather_rows(torch.as_tensor(y_loc), starts).numpy()
        # --- SpGEMM exchange: B row blocks replicated, C row blocks concatenated
        Bf = mdist.gather_csr_blocks(blk)
        assert np.array_equal(Bf.rp.numpy(), A.rp) and np.array_equal(Bf.col.numpy(), A.col)
        assert np.array_equal(Bf.val.numpy(), A.val)
        Bg = gen.CSR(A.m, A.n, Bf.rp.numpy(), Bf.col.numpy(), Bf.val.numpy())
        Cb, _, _ = oracle.spgemm(Ab, Bg)
        Cblk = CsrTensor.from_arrays(Cb.rp, Cb.col, Cb.val, (Cb.m, Cb.n), "cpu")
        Cf = mdist.gather_csr_blocks(Cblk)
        if rank == 0:
            yw, _ = oracle.spmv(A, x)
            W, _, _ = oracle.spgemm(A, A)
            results["spmv"] = bool(np.array_equal(y, yw))
            results["rp"] = bool(np.array_equal(Cf.rp.numpy(), W.rp))
            results["col"] = bool(np.array_equal(Cf.col.numpy(), W.col))
            results["val"] = bool(np.array_equal(Cf.val.numpy(), W.val))
            results["rows"] = [int(s) for s in starts]
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2])
def test_row_blocks_world2(world):
    mgr = mp.Manager()
    results = mgr.dict()
    mp.spawn(_worker, args=(world, _free_port(), results), nprocs=world, join=True)
    assert results["spmv"] and results["rp"] and results["col"] and results["val"], dict(results)
    assert results["rows"][0] == 0 and results["rows"][-1] == 301
