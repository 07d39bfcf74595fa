"""World-size-2 and -3 (gloo, CPU) tests of the halo-exchange SpMV layer
(dist.HaloSpmv): after the one-time plan and one
all_to_all per SpMV, every rank's local x must hold exactly the x entries its
row block references, at the renumbered positions -- checked by computing
the local product with the oracle on the renumbered block and comparing the
concatenated y with the oracle's y on the whole matrix (integer mode: exact).
Also checks that a stencil slab's halo is its neighbour planes only."""
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


def _worker(rank, world, port, which, results):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import gen
        import oracle
        from paper_conf_ipps_daltonbmog15_b200 import dist as mdist
        if which == "random":
            A = gen.random_csr(403, 397, 5, density=0.03, empty_frac=0.2, dense_rows=1, mode="int")
        else:
            A = gen.poisson3d_27pt(12, 12, 12 * world)  # one 12^3 slab per rank
        x = gen.x_vector(A.n, "int")
        starts = mdist.split_rows(A.rp, world)
        r0, r1 = int(starts[rank]), int(starts[rank + 1])
        a0, a1 = int(A.rp[r0]), int(A.rp[r1])
        plan = mdist.HaloSpmv(A.rp[r0:r1 + 1] - a0, A.col[a0:a1], A.val[a0:a1], A.n, device="cpu")
        ns = plan.ns
        plan.x_own.copy_(torch.as_tensor(x[rank * ns: rank * ns + plan.own_len]))
        plan.exchange()
        Ab = gen.CSR(r1 - r0, plan.A.shape[1], *[t.numpy() for t in (plan.A.rp, plan.A.col, plan.A.val)])
        y_loc, _ = oracle.spmv(Ab, plan.x_local.numpy())
        y = mdist.allgather_rows(torch.as_tensor(y_loc), starts).numpy()
        halo = torch.tensor([plan.halo_len], dtype=torch.int64)
        hs = [torch.empty_like(halo) for _ in range(world)]
        dist.all_gather(hs, halo)
        if rank == 0:
            results["ok"] = bool(np.array_equal(y, oracle.spmv(A, x)[0]))
            results["halo"] = [int(h) for h in hs]
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
@pytest.mark.parametrize("which", ["random", "stencil"])
def test_halo_spmv(world, which):
    mgr = mp.Manager()
    results = mgr.dict()
    mp.spawn(_worker, args=(world, _free_port(), which, results), nprocs=world, join=True)
    assert results["ok"], dict(results)
    if which == "stencil":
        # a 12^3 slab's rows reference at most one 12x12 plane from each
        # neighbouring slab (x slices equal the row blocks here)
        assert max(results["halo"]) <= 2 * 12 * 12, results["halo"]
