"""CUDA path of the row-block layer on one GPU (NCCL, world size 1): the x
all-gather, B replication (device offset rebase kernel), local SpMV / SpGEMM
and the concatenation of C, checked against the oracle.  The world-size-2
exchange logic is covered by tests/test_dist_gloo.py on CPU."""
import os
import socket

import numpy as np
import pytest
import torch

import gen
import oracle
from tests.gpu_util import assert_spmv

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def pg():
    import torch.distributed as dist
    if not dist.is_initialized():
        with socket.socket() as s:
            s.bind(("127.0.0.1", 0))
            port = s.getsockname()[1]
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    yield dist
    dist.destroy_process_group()


def test_rebase_kernel():
    from paper_conf_ipps_daltonbmog15_b200 import rebase_offsets
    rp = torch.tensor([7, 9, 9, 20], dtype=torch.int32, device="cuda")
    assert rebase_offsets(rp, 100).cpu().tolist() == [100, 102, 102, 113]


def test_dist_world1(pg):
    from paper_conf_ipps_daltonbmog15_b200 import dist as mdist
    A = gen.config("C4", "random", scale=0.02)
    starts = mdist.split_rows(A.rp, 1)
    blk = mdist.row_block(A.rp, A.col, A.val, int(starts[0]), int(starts[1]), A.n)
    x = gen.x_vector(A.n, "random", seed=5)
    xs = mdist.x_slice_of(torch.as_tensor(x, device="cuda"), 0, 1)
    y = mdist.dist_spmv(blk, xs, A.n).cpu().numpy()
    assert_spmv(A, x, y, label="dist spmv")
    C = mdist.dist_spgemm(blk, blk, gather_c=True)
    W, sc, _ = oracle.spgemm(A, A)
    rp, col, val = C.numpy()
    assert np.array_equal(rp, W.rp) and np.array_equal(col, W.col)
    ok, msg = oracle.check_values(val, W.val, sc, np.float64)
    assert ok, msg


@pytest.mark.parametrize("cfg,scale", [("C4", 0.2), ("C5", 0.005)])
@pytest.mark.parametrize("P", [2, 4, 8])
def test_row_blocks_one_gpu(cfg, scale, P):
    """The multi-GPU decomposition run on one GPU: P nnz-balanced row blocks
    (zero-copy views with rebased offsets), libmsp SpMV and SpGEMM on each
    block against the replicated x / B, blocks concatenated -- y, and C's
    row_offsets / col_idx / values, must equal the oracle's single result bit
    for bit (integer mode, SURVEY §8(e) correctness)."""
    from paper_conf_ipps_daltonbmog15_b200 import SpGemmPlan, spmv
    from paper_conf_ipps_daltonbmog15_b200 import dist as mdist
    from tests.gpu_util import dev
    A = gen.config(cfg, "int", scale=scale)
    x = gen.x_vector(A.n, "int")
    Ad = dev(A)
    xd = torch.as_tensor(x, device="cuda")
    W, _, _ = oracle.spgemm(A, A)
    yw, _ = oracle.spmv(A, x)
    for split in ("nnz", "products"):
        starts = (mdist.split_rows(A.rp, P) if split == "nnz"
                  else mdist.split_rows_by_products(A.rp, A.col, A.rp, P))
        assert starts[0] == 0 and starts[-1] == A.m and np.all(np.diff(starts) >= 0)
        ys, Cs = [], []
        for r in range(P):
            blk = mdist.block_view(Ad, int(starts[r]), int(starts[r + 1]))
            ys.append(spmv(blk, xd))
            p = SpGemmPlan(blk, Ad)
            p.setup()
            p.symbolic()
            Cs.append(p.numeric())
        y = torch.cat(ys).cpu().numpy()
        assert np.array_equal(y, yw), f"{cfg} P={P} {split}: y"
        C = mdist.concat_blocks(Cs)
        rp, col, val = C.numpy()
        assert np.array_equal(rp, W.rp), f"{cfg} P={P} {split}: row_offsets"
        assert np.array_equal(col, W.col), f"{cfg} P={P} {split}: col_idx"
        assert np.array_equal(val, W.val), f"{cfg} P={P} {split}: values"


def test_gather_values():
    from paper_conf_ipps_daltonbmog15_b200 import gather_values
    src = torch.arange(1000, dtype=torch.float64, device="cuda") * 1.5
    idx = torch.as_tensor(np.random.default_rng(1).integers(0, 1000, 777), dtype=torch.int32, device="cuda")
    assert torch.equal(gather_values(src, idx), src[idx.long()])
    s32 = torch.arange(100, dtype=torch.float32, device="cuda")
    i32 = torch.tensor([5, 0, 99], dtype=torch.int32, device="cuda")
    assert gather_values(s32, i32).tolist() == [5.0, 0.0, 99.0]


def test_halo_spmv_world1(pg):
    """The halo-exchange SpMV on one rank (NCCL): no halo, renumbered columns
    equal the originals, result equals the oracle bit for bit (int mode)."""
    from paper_conf_ipps_daltonbmog15_b200 import dist as mdist
    A = gen.config("C4", "int", scale=0.02)
    x = gen.x_vector(A.n, "int")
    plan = mdist.HaloSpmv(A.rp, A.col, A.val, A.n, device=torch.device("cuda", 0))
    assert plan.halo_len == 0 and plan.own_len == A.n
    plan.x_own.copy_(torch.as_tensor(x, device="cuda"))
    y = plan.spmv().cpu().numpy()
    assert np.array_equal(y, oracle.spmv(A, x)[0])
