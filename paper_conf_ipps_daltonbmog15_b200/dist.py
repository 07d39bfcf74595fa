"""Multi-GPU row-block layer.

One process per GPU; torch.distributed provides the process group (NCCL over
NVLink/NVSwitch on GPUs; gloo in the CPU tests of the exchange logic).

* Row split: rank r owns rows [R_r, R_{r+1}) with R_r = lower_bound(rp,
  ceil(r*nnz/P)) (`msp_row_split`), i.e. blocks balanced by nonzeros.
* SpMV: x is split in equal padded slices; `allgather_x` rebuilds the full
  x on every rank (the exchange step), then the rank's block of A runs the
  merge-path SpMV locally.  y stays distributed by row blocks.
* SpGEMM: the row blocks of B are replicated with `gather_csr_blocks`
  (sizes all-gathered, then one broadcast per source rank straight into its
  place in the full arrays, offsets rebased on the device); the local
  symbolic / numeric phases run on the rank's rows of A; `gather_csr_blocks`
  also concatenates C's row blocks when a replicated C is wanted.

Compute happens in libmsp kernels (CUDA tensors); only data movement and
offset rebasing are done here.  CPU tensors are accepted so that the exchange
logic can be tested with gloo on a machine without a GPU.
"""
from __future__ import annotations

import numpy as np
import torch
import torch.distributed as dist

from .ops import CsrTensor, rebase_offsets, row_split


def split_rows(rp_host, world: int) -> np.ndarray:
    """[R_0 = 0, R_1, ..., R_P = m] balanced by nonzeros (libmsp host code)."""
    return row_split(rp_host, world)


def row_block(rp, col, val, r0: int, r1: int, ncols: int, device="cuda") -> CsrTensor:
    """Rows [r0, r1) of a CSR matrix given as host arrays -> CsrTensor on
    `device` with offsets rebased to 0."""
    a0, a1 = int(rp[r0]), int(rp[r1])
    rpl = (np.asarray(rp[r0:r1 + 1], dtype=np.int64) - a0).astype(np.int32)
    return CsrTensor.from_arrays(rpl, np.asarray(col[a0:a1]), np.asarray(val[a0:a1]), (r1 - r0, ncols), device)


def _rebase(rp: torch.Tensor, base: int) -> torch.Tensor:
    if rp.is_cuda:
        return rebase_offsets(rp, base)
    return rp - rp[:1] + base  # host-side plumbing for the gloo tests


def allgather_x(x_slice: torch.Tensor, n: int, group=None) -> torch.Tensor:
    """Equal slices (last padded) of x from every rank -> full x[n]."""
    world = dist.get_world_size(group)
    full = torch.empty(x_slice.numel() * world, dtype=x_slice.dtype, device=x_slice.device)
    if x_slice.is_cuda:
        dist.all_gather_into_tensor(full, x_slice.contiguous(), group=group)
    else:
        dist.all_gather(list(full.chunk(world)), x_slice.contiguous(), group=group)
    return full[:n]


def allgather_rows(v_blk: torch.Tensor, starts, group=None) -> torch.Tensor:
    """Row-block pieces of a vector (rank r holds rows [starts[r], starts[r+1]))
    -> the full vector on every rank (pieces padded to the largest block)."""
    world = dist.get_world_size(group)
    sizes = [int(starts[q + 1] - starts[q]) for q in range(world)]
    mx = max(sizes) if sizes else 0
    pad = torch.zeros(mx, dtype=v_blk.dtype, device=v_blk.device)
    pad[:v_blk.numel()] = v_blk
    parts = [torch.empty_like(pad) for _ in range(world)]
    dist.all_gather(parts, pad, group=group)
    return torch.cat([parts[q][:sizes[q]] for q in range(world)])


def x_slice_of(x_full: torch.Tensor, rank: int, world: int) -> torch.Tensor:
    ns = -(-x_full.numel() // world)
    s = torch.zeros(ns, dtype=x_full.dtype, device=x_full.device)
    part = x_full[rank * ns:(rank + 1) * ns]
    s[:part.numel()] = part
    return s


def gather_csr_blocks(blk: CsrTensor, group=None) -> CsrTensor:
    """Row blocks (in rank order) of a matrix -> the full matrix on every rank.
    Sizes are all-gathered first; each rank then broadcasts its block into its
    place in the full arrays; row offsets are rebased by the running nnz."""
    world = dist.get_world_size(group)
    dev = blk.val.device
    meta = torch.tensor([blk.shape[0], blk.nnz], dtype=torch.int64, device=dev)
    metas = [torch.empty_like(meta) for _ in range(world)]
    dist.all_gather(metas, meta, group=group)
    rows = [int(t[0]) for t in metas]
    nnzs = [int(t[1]) for t in metas]
    m, nnz = sum(rows), sum(nnzs)
    rp = torch.empty(m + 1, dtype=torch.int32, device=dev)
    col = torch.empty(nnz, dtype=torch.int32, device=dev)
    val = torch.empty(nnz, dtype=blk.val.dtype, device=dev)
    r_off = np.concatenate([[0], np.cumsum(rows)]).astype(np.int64)
    z_off = np.concatenate([[0], np.cumsum(nnzs)]).astype(np.int64)
    me = dist.get_rank(group)
    for src in range(world):
        rsl = slice(int(r_off[src]), int(r_off[src + 1]) + 1)
        zsl = slice(int(z_off[src]), int(z_off[src + 1]))
        if src == me:
            rp_part = _rebase(blk.rp, int(z_off[src]))
            col[zsl].copy_(blk.col)
            val[zsl].copy_(blk.val)
        else:
            rp_part = torch.empty(rows[src] + 1, dtype=torch.int32, device=dev)
        gsrc = dist.get_global_rank(group, src) if group is not None else src
        dist.broadcast(rp_part, gsrc, group=group)
        if nnzs[src]:
            dist.broadcast(col[zsl], gsrc, group=group)
            dist.broadcast(val[zsl], gsrc, group=group)
        rp[rsl] = rp_part  # already rebased by its source
    return CsrTensor(rp, col, val, (m, blk.shape[1]))


def dist_spmv(A_blk: CsrTensor, x_slice: torch.Tensor, n: int, group=None):
    """y rows of this rank = A_blk @ allgather(x)."""
    from .ops import spmv
    x_full = allgather_x(x_slice, n, group)
    return spmv(A_blk, x_full)


def dist_spgemm(A_blk: CsrTensor, B_blk: CsrTensor, group=None, gather_c: bool = False):
    """Rows of C = A B for this rank (B's row blocks replicated first)."""
    from .ops import SpGemmPlan
    B_full = gather_csr_blocks(B_blk, group)
    plan = SpGemmPlan(A_blk, B_full)
    plan.setup()
    plan.symbolic()
    C_blk = plan.numeric()
    return gather_csr_blocks(C_blk, group) if gather_c else C_blk
