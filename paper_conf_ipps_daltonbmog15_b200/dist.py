"""Multi-GPU row-block layer.

One process per GPU; torch.distributed provides the process group (NCCL over
NVLink/NVSwitch on GPUs; gloo in the CPU tests of the exchange logic).

* Row split: rank r owns rows [R_r, R_{r+1}) with R_r = lower_bound(rp,
  ceil(r*nnz/P)) (`msp_row_split`), i.e. blocks balanced by nonzeros.
* SpMV: x is split in equal padded slices; `allgather_x` rebuilds the full
  x on every rank (the exchange step), then the rank's block of A runs the
  merge-path SpMV locally.  y stays distributed by row blocks.
* SpGEMM: the row blocks of B are replicated with `gather_csr_blocks`
  (sizes all-gathered, then one padded all-gather per CSR array -- three
  collectives at any world size -- and a device-side concatenation with the
  offsets rebased); the local symbolic / numeric phases run on the rank's
  rows of A; `gather_csr_blocks` also concatenates C's row blocks when a
  replicated C is wanted (C may instead stay distributed by row blocks).
* `block_view` / `concat_blocks` are the zero-copy row-block views and the
  concatenation used on one device (the P-block parity tests).

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


def _all_gather_padded(t: torch.Tensor, n_max: int, group=None) -> torch.Tensor:
    """Every rank's `t` padded to n_max entries -> [world * n_max] (one
    collective: all_gather_into_tensor on NCCL, a list all-gather on gloo)."""
    world = dist.get_world_size(group)
    pad = torch.zeros(n_max, dtype=t.dtype, device=t.device)
    pad[:t.numel()] = t
    out = torch.empty(world * n_max, dtype=t.dtype, device=t.device)
    if t.is_cuda:
        dist.all_gather_into_tensor(out, pad, group=group)
    else:
        dist.all_gather(list(out.chunk(world)), pad, group=group)
    return out


def gather_csr_blocks(blk: CsrTensor, group=None) -> CsrTensor:
    """Row blocks (in rank order) of a matrix -> the full matrix on every rank.
    Block sizes are all-gathered first; then ONE padded all-gather per array
    (row offsets, columns, values: three collectives whatever the world
    size) and a device-side concatenation, with each block's offsets rebased
    by the running nnz (msp_rebase_offsets)."""
    world = dist.get_world_size(group)
    dev = blk.val.device
    meta = torch.tensor([blk.shape[0], blk.nnz], dtype=torch.int64, device=dev)
    metas = _all_gather_padded(meta, 2, group).view(world, 2).cpu().numpy()
    rows = [int(r) for r in metas[:, 0]]
    nnzs = [int(z) for z in metas[:, 1]]
    m, nnz = sum(rows), sum(nnzs)
    mr, mz = max(rows) + 1, max(max(nnzs), 1)
    rp_all = _all_gather_padded(blk.rp, mr, group).view(world, mr)
    col_all = _all_gather_padded(blk.col, mz, group).view(world, mz)
    val_all = _all_gather_padded(blk.val, mz, group).view(world, mz)
    return concat_blocks([CsrTensor(rp_all[q, :rows[q] + 1], col_all[q, :nnzs[q]], val_all[q, :nnzs[q]],
                                    (rows[q], blk.shape[1])) for q in range(world)])


def concat_blocks(blocks) -> CsrTensor:
    """Row blocks (each with offsets starting at 0) -> one CSR matrix: columns
    and values concatenated, offsets rebased by the running nnz on the
    device (msp_rebase_offsets).  Used for B replication and for C."""
    dev = blocks[0].val.device
    m = sum(b.shape[0] for b in blocks)
    nnz = sum(b.nnz for b in blocks)
    rp = torch.empty(m + 1, dtype=torch.int32, device=dev)
    col = torch.empty(nnz, dtype=torch.int32, device=dev)
    val = torch.empty(nnz, dtype=blocks[0].val.dtype, device=dev)
    r = z = 0
    for b in blocks:
        rp[r:r + b.shape[0] + 1] = _rebase(b.rp.contiguous(), z)
        col[z:z + b.nnz] = b.col
        val[z:z + b.nnz] = b.val
        r += b.shape[0]
        z += b.nnz
    if not blocks or m == 0:
        rp.zero_()
    return CsrTensor(rp, col, val, (m, blocks[0].shape[1]))


def block_view(A: CsrTensor, r0: int, r1: int) -> CsrTensor:
    """Rows [r0, r1) of a device CSR matrix as a zero-copy block: columns and
    values are views into A's arrays, only the m_r + 1 row offsets are
    rebased to start at 0 (msp_rebase_offsets)."""
    rp_h = A.rp[r0:r1 + 1]
    a0, a1 = int(A.rp[r0]), int(A.rp[r1])
    return CsrTensor(_rebase(rp_h.contiguous(), 0), A.col[a0:a1], A.val[a0:a1], (r1 - r0, A.shape[1]))


def split_rows_by_products(A_rp_host, A_col_host, B_rp_host, world: int) -> np.ndarray:
    """Row blocks balanced by SpGEMM products (sum over a row's nonzeros of
    the referenced B row lengths) instead of by nonzeros: the same
    lower-bound split (msp_row_split) over the per-row product prefix sum."""
    bl = np.diff(np.asarray(B_rp_host, dtype=np.int64))
    w = bl[np.asarray(A_col_host, dtype=np.int64)]
    cs = np.concatenate([[0], np.cumsum(w)])
    rp = np.asarray(A_rp_host, dtype=np.int64)
    prow = cs[rp]  # products before each row
    m = rp.size - 1
    total = int(prow[-1])
    starts = np.empty(world + 1, dtype=np.int32)
    starts[0], starts[world] = 0, m
    for r in range(1, world):
        starts[r] = int(np.searchsorted(prow, -(-r * total // world), side="left"))
        starts[r] = min(max(starts[r], starts[r - 1]), m)
    return starts


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
