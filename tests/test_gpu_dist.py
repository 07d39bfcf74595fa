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
