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
* `HaloSpmv`: SpMV without replicating x -- a one-time halo plan and one
  all_to_all of the halo values per SpMV.

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


class HaloSpmv:
    """Distributed SpMV WITHOUT replicating x: a halo
    exchange instead of the all-gather.

    x is owned in equal slices of ceil(n/P) entries (as for `allgather_x`).
    Setup (host, once per matrix): the rank's row block lists the columns it
    references; those owned by other ranks form its halo, sorted by global
    index -- hence grouped by owner rank.  The per-owner request lists are
    exchanged once (all_to_all), so every rank knows which of its x entries
    each neighbour needs; the block's column indices are renumbered into a
    local x = [own slice | halo from rank 0 | halo from rank 1 | ...].
    Per SpMV: the rank packs the values its neighbours need
    (`msp_gather_values`), ONE all_to_all_single delivers every halo
    straight into the local x, and the local SpMV (libmsp) runs on the
    renumbered block.  For a banded / stencil matrix the halo is a few planes
    (C2 slabs: 2 x 10^4 entries per neighbour) instead of the whole x; for
    uniformly random columns (C5) it approaches the all-gather.
    """

    def __init__(self, rp_blk, col_blk, val_blk, n: int, group=None, device=None):
        import numpy as np
        self.group = group
        self.world = dist.get_world_size(group)
        self.rank = dist.get_rank(group)
        P, r = self.world, self.rank
        self.n = n
        self.ns = -(-n // P)
        own0 = r * self.ns
        self.own_len = max(0, min(n, own0 + self.ns) - own0)
        cols = np.asarray(col_blk, dtype=np.int64)
        uniq = np.unique(cols)
        owner = uniq // self.ns
        remote = uniq[owner != r]
        rown = remote // self.ns
        need = np.bincount(rown, minlength=P).astype(np.int64)  # entries this rank needs from each owner
        dev = device if device is not None else torch.device("cpu")
        cpu = not (isinstance(dev, torch.device) and dev.type == "cuda") and not (isinstance(dev, str) and
                                                                                   dev.startswith("cuda"))
        coll_dev = torch.device("cpu") if cpu else torch.device(dev)
        # exchange request counts, then the request lists (global indices)
        need_t = torch.as_tensor(need, device=coll_dev)
        give_t = torch.empty_like(need_t)
        dist.all_to_all_single(give_t, need_t, group=group)
        give = give_t.cpu().numpy().astype(np.int64)  # entries each rank needs from this rank
        req = torch.as_tensor(remote.astype(np.int64), device=coll_dev)
        got = torch.empty(int(give.sum()), dtype=torch.int64, device=coll_dev)
        dist.all_to_all_single(got, req, output_split_sizes=give.tolist(), input_split_sizes=need.tolist(),
                               group=group)
        send_idx = (got.cpu().numpy() - own0).astype(np.int32)  # positions in this rank's slice
        assert send_idx.size == 0 or (send_idx.min() >= 0 and send_idx.max() < self.own_len)
        self.send_counts, self.recv_counts = give.tolist(), need.tolist()
        self.halo_len = int(remote.size)
        # renumbered columns: own -> c - own0, remote -> own_len + rank in `remote`
        mine = (cols // self.ns) == r
        local = np.empty(cols.size, dtype=np.int64)
        local[mine] = cols[mine] - own0
        local[~mine] = self.own_len + np.searchsorted(remote, cols[~mine])
        m_blk = len(rp_blk) - 1
        self.A = CsrTensor.from_arrays(np.asarray(rp_blk, dtype=np.int32), local.astype(np.int32), val_blk,
                                       (m_blk, self.own_len + self.halo_len), dev)
        self.send_idx = torch.as_tensor(send_idx, device=dev)
        self.x_local = torch.zeros(self.own_len + self.halo_len, dtype=self.A.val.dtype, device=dev)
        self.send_buf = torch.empty(int(send_idx.size), dtype=self.A.val.dtype, device=dev)

    @property
    def x_own(self) -> torch.Tensor:
        """This rank's slice of x (write the vector here before `spmv`)."""
        return self.x_local[:self.own_len]

    def exchange(self):
        """Halo values of x into x_local (pack + one all_to_all_single)."""
        if self.send_buf.is_cuda:
            from .ops import gather_values
            gather_values(self.x_own, self.send_idx, out=self.send_buf)
        else:  # host plumbing for the gloo tests
            self.send_buf.copy_(self.x_own[self.send_idx.long()])
        dist.all_to_all_single(self.x_local[self.own_len:], self.send_buf, output_split_sizes=self.recv_counts,
                               input_split_sizes=self.send_counts, group=self.group)

    def spmv(self, out: torch.Tensor | None = None) -> torch.Tensor:
        """y rows of this rank = A_blk @ x (halo exchange, then libmsp SpMV)."""
        from .ops import spmv
        self.exchange()
        return spmv(self.A, self.x_local, out=out)
