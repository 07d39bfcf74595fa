"""Seeded CSR generators for the BASELINE.json configs (BJ:7-11) and tiny fuzz.

Every generator returns a :class:`CSR` whose rows are sorted by column and
unique (the input contract of the paper).  Recipes follow
SURVEY.md §8(d) "Synthetic inputs" and are restated in DESIGN.md §3:

* C1 ``poisson2d_5pt(64)``   -- 2-D 5-point Laplacian, diag 4, off-diag -1.
* C2 ``poisson3d_27pt(100)`` -- 3-D 27-point stencil, diag 26, off-diag -1.
* C3 ``rmat(22, 16)``        -- Graph500 R-MAT (0.57, 0.19, 0.19, 0.05), seed 22,
  duplicate edges collapsed, self loops kept.
* C4 ``pathological()``      -- 2M rows, one dense 1M-nnz row at 1,000,003,
  a contiguous block of 500K empty rows at the end plus 500K scattered empty
  rows, every other row 1..16 uniform random columns; seed 4.
* C5 ``random_rows(10**8)``  -- row length uniform in {0..8}, uniform random
  columns, deduplicated within a row; seed 5.

Values: ``mode="int"`` draws {+-1, +-2, +-3} (stencils keep their stencil
values) so every summation order is exact;
``mode="random"`` draws U[-1, 1) with seed 1000 + config number.
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np


@dataclass
class CSR:
    m: int
    n: int
    rp: np.ndarray   # int32 [m+1]
    col: np.ndarray  # int32 [nnz]
    val: np.ndarray  # float64 or float32 [nnz]

    @property
    def nnz(self) -> int:
        return int(self.rp[-1]) if self.m > 0 else 0

    @property
    def dtype(self):
        return self.val.dtype

    def astype(self, dt) -> "CSR":
        return CSR(self.m, self.n, self.rp, self.col, self.val.astype(dt))

    def with_values(self, val: np.ndarray) -> "CSR":
        assert val.shape == self.col.shape
        return CSR(self.m, self.n, self.rp, self.col, val)

    def row_ids(self) -> np.ndarray:
        """COO row index of every nonzero (input-side helper, tests only)."""
        return np.repeat(np.arange(self.m, dtype=np.int64), np.diff(self.rp.astype(np.int64)))

    def dense(self) -> np.ndarray:
        d = np.zeros((self.m, self.n), dtype=np.float64)
        r = self.row_ids()
        # plain scatter; inputs are unique per (row, col)
        d[r, self.col] = self.val
        return d


def _sorted_unique(keys: np.ndarray) -> np.ndarray:
    """np.unique of an int64 key array via an in-place sort and an adjacent
    mask (same result; numpy 2.x's np.unique takes ~100 s on 67M keys)."""
    k = np.sort(keys)
    if k.size == 0:
        return k
    keep = np.empty(k.size, dtype=bool)
    keep[0] = True
    np.not_equal(k[1:], k[:-1], out=keep[1:])
    return k[keep]


def _from_sorted_keys(keys: np.ndarray, m: int, n: int) -> tuple[np.ndarray, np.ndarray]:
    """Sorted unique int64 keys row*n+col -> (rp, col)."""
    rows = keys // n
    cols = (keys - rows * n).astype(np.int32)
    counts = np.bincount(rows, minlength=m).astype(np.int64)
    rp = np.zeros(m + 1, dtype=np.int64)
    np.cumsum(counts, out=rp[1:])
    assert rp[-1] < 2**31
    return rp.astype(np.int32), cols


def int_values(nnz: int, seed: int, dtype=np.float64) -> np.ndarray:
    """Values uniform in {+-1, +-2, +-3} (exactness mode)."""
    rng = np.random.default_rng(seed)
    mag = rng.integers(1, 4, size=nnz, dtype=np.int8)
    sgn = rng.integers(0, 2, size=nnz, dtype=np.int8) * 2 - 1
    return (mag * sgn).astype(dtype)


def random_values(nnz: int, seed: int, dtype=np.float64) -> np.ndarray:
    rng = np.random.default_rng(seed)
    return rng.uniform(-1.0, 1.0, size=nnz).astype(dtype)


def x_vector(n: int, mode: str = "int", seed: int = 1000, dtype=np.float64) -> np.ndarray:
    """Dense x.  int mode: x_j = ((j*7919) mod 7) - 3."""
    if mode == "int":
        j = np.arange(n, dtype=np.int64)
        return (((j * 7919) % 7) - 3).astype(dtype)
    rng = np.random.default_rng(seed)
    return rng.uniform(-1.0, 1.0, size=n).astype(dtype)


# ----------------------------------------------------------------------------
# Stencils (C1, C2)
# ----------------------------------------------------------------------------

def _stencil(dims: tuple[int, ...], offsets: list[tuple[int, ...]], center: float) -> CSR:
    """Grid stencil; `offsets` sorted lexicographically (outermost dim first) so
    that columns come out ascending within each row."""
    dims = tuple(int(d) for d in dims)
    m = int(np.prod(dims))
    coords = np.indices(dims[::-1]).reshape(len(dims), -1)[::-1]  # coords[k] along dims[k], x fastest
    strides = [int(np.prod(dims[:k])) for k in range(len(dims))]   # x stride 1
    row = np.arange(m, dtype=np.int64)
    cols, vals, valid = [], [], []
    for off in offsets:  # off is given outermost-first: (dz, dy, dx)
        off_inner_first = off[::-1]
        ok = np.ones(m, dtype=bool)
        delta = 0
        for k, dk in enumerate(off_inner_first):
            ck = coords[k] + dk
            ok &= (ck >= 0) & (ck < dims[k])
            delta += dk * strides[k]
        cols.append(row + delta)
        valid.append(ok)
        vals.append(center if all(o == 0 for o in off) else -1.0)
    C = np.stack(cols, axis=1)
    V = np.broadcast_to(np.array(vals), C.shape)
    M = np.stack(valid, axis=1)
    counts = M.sum(axis=1)
    rp = np.zeros(m + 1, dtype=np.int64)
    np.cumsum(counts, out=rp[1:])
    return CSR(m, m, rp.astype(np.int32), C[M].astype(np.int32), V[M].astype(np.float64))


def poisson2d_5pt(nx: int, ny: int | None = None) -> CSR:
    """C1: 2-D 5-point Poisson (diag 4, off-diag -1) on an nx*ny grid."""
    ny = nx if ny is None else ny
    offs = [(-1, 0), (0, -1), (0, 0), (0, 1), (1, 0)]  # (dy, dx)
    return _stencil((nx, ny), offs, 4.0)


def poisson3d_27pt(nx: int, ny: int | None = None, nz: int | None = None) -> CSR:
    """C2: 3-D 27-point stencil (diag 26, off-diag -1) on an nx*ny*nz grid."""
    ny = nx if ny is None else ny
    nz = nx if nz is None else nz
    offs = [(dz, dy, dx) for dz in (-1, 0, 1) for dy in (-1, 0, 1) for dx in (-1, 0, 1)]
    return _stencil((nx, ny, nz), offs, 26.0)


# ----------------------------------------------------------------------------
# Power law (C3), pathological (C4), random rows (C5), fuzz
# ----------------------------------------------------------------------------

def rmat(scale: int, edge_factor: int = 16, seed: int = 22,
         probs=(0.57, 0.19, 0.19, 0.05), chunk: int = 1 << 23) -> CSR:
    """C3: R-MAT graph, 2^scale vertices, edge_factor*2^scale edges, no noise,
    no relabel; duplicates collapsed, self loops kept."""
    n = 1 << scale
    ne = edge_factor * n
    a, b, c, _ = probs
    rng = np.random.default_rng(seed)
    keys = np.empty(ne, dtype=np.int64)
    for s in range(0, ne, chunk):
        e = min(ne, s + chunk)
        r = np.zeros(e - s, dtype=np.int64)
        cc = np.zeros(e - s, dtype=np.int64)
        for _ in range(scale):
            u = rng.random(e - s)
            rbit = u >= (a + b)
            cbit = ((u >= a) & (u < a + b)) | (u >= a + b + c)
            r = (r << 1) | rbit
            cc = (cc << 1) | cbit
        keys[s:e] = (r << scale) | cc
    keys = _sorted_unique(keys)
    rows = keys >> scale
    cols = (keys & (n - 1)).astype(np.int32)
    counts = np.bincount(rows, minlength=n)
    rp = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(counts, out=rp[1:])
    return CSR(n, n, rp.astype(np.int32), cols, np.ones(cols.size))


def pathological(n: int = 2_000_000, dense_row: int = 1_000_003, dense_nnz: int = 1_000_000,
                 tail_empty: int = 500_000, scattered_empty: int = 500_000,
                 max_len: int = 16, seed: int = 4) -> CSR:
    """C4: one dense row, 50% empty rows (a contiguous tail block plus scattered
    rows), every other row has 1..max_len uniform random columns."""
    rng = np.random.default_rng(seed)
    lens = rng.integers(1, max_len + 1, size=n).astype(np.int64)
    lens[n - tail_empty:] = 0
    cand = np.setdiff1d(np.arange(n - tail_empty), [dense_row])
    lens[rng.choice(cand, size=scattered_empty, replace=False)] = 0
    lens[dense_row] = 0
    rows = np.repeat(np.arange(n, dtype=np.int64), lens)
    cols = rng.integers(0, n, size=rows.size, dtype=np.int64)
    dcols = np.sort(rng.choice(n, size=dense_nnz, replace=False)).astype(np.int64)
    keys = np.concatenate([rows * n + cols, dense_row * np.int64(n) + dcols])
    keys = _sorted_unique(keys)
    rp, col = _from_sorted_keys(keys, n, n)
    return CSR(n, n, rp, col, np.ones(col.size))


def random_rows(n: int = 100_000_000, max_len: int = 8, seed: int = 5, ncols: int | None = None) -> CSR:
    """C5: row length uniform in {0..max_len}, uniform random columns,
    deduplicated within each row."""
    ncols = n if ncols is None else ncols
    rng = np.random.default_rng(seed)
    lens = rng.integers(0, max_len + 1, size=n).astype(np.int64)
    # Rows in blocks: a padded [rows, max_len] block of draws, slot k >= len
    # masked with a sentinel, sorted along each row, adjacent duplicates
    # dropped (vectorised; a global unique over 4e8 keys takes minutes).
    sent = np.iinfo(np.int64).max
    counts = np.zeros(n, dtype=np.int64)
    parts = []
    blk = 1 << 22
    for s in range(0, n, blk):
        e = min(n, s + blk)
        c = rng.integers(0, ncols, size=(e - s, max_len), dtype=np.int64)
        c[np.arange(max_len)[None, :] >= lens[s:e, None]] = sent
        c.sort(axis=1)
        keep = c != sent
        keep[:, 1:] &= c[:, 1:] != c[:, :-1]
        counts[s:e] = keep.sum(axis=1)
        parts.append(c[keep].astype(np.int32))
    rp = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(counts, out=rp[1:])
    if rp[-1] > np.iinfo(np.int32).max:
        raise ValueError("nnz exceeds int32")
    col = np.concatenate(parts) if parts else np.zeros(0, np.int32)
    return CSR(n, ncols, rp.astype(np.int32), col, np.ones(col.size))


def random_csr(m: int, n: int, seed: int, density: float = 0.1, empty_frac: float = 0.0,
               dense_rows: int = 0, row_len: tuple[int, int] | None = None,
               mode: str = "int", dtype=np.float64) -> CSR:
    """Tiny fuzz matrices: Bernoulli(density) pattern (or uniform row lengths in
    `row_len`), a fraction of forced-empty rows, and `dense_rows` full rows."""
    rng = np.random.default_rng(seed)
    if m == 0 or n == 0:
        return CSR(m, n, np.zeros(m + 1, np.int32), np.zeros(0, np.int32), np.zeros(0, dtype))
    if row_len is None:
        pat = rng.random((m, n)) < density
    else:
        pat = np.zeros((m, n), dtype=bool)
        lens = rng.integers(row_len[0], row_len[1] + 1, size=m)
        for i in range(m):
            k = min(int(lens[i]), n)
            pat[i, rng.choice(n, size=k, replace=False)] = True
    if empty_frac > 0:
        pat[rng.random(m) < empty_frac, :] = False
    if dense_rows > 0:
        pat[rng.choice(m, size=min(dense_rows, m), replace=False), :] = True
    r, c = np.nonzero(pat)
    counts = np.bincount(r, minlength=m)
    rp = np.zeros(m + 1, dtype=np.int64)
    np.cumsum(counts, out=rp[1:])
    if mode == "int":
        val = int_values(c.size, seed + 7, dtype)
    else:
        val = random_values(c.size, seed + 7, dtype)
    return CSR(m, n, rp.astype(np.int32), c.astype(np.int32), val)


def transpose(A: CSR) -> CSR:
    """CSR of A^T (structural re-indexing of the input; used to build the
    A + A^T workload).  Stable, so columns stay sorted within each row."""
    rows = A.row_ids()
    order = np.argsort(A.col, kind="stable")
    counts = np.bincount(A.col, minlength=A.n)
    rp = np.zeros(A.n + 1, dtype=np.int64)
    np.cumsum(counts, out=rp[1:])
    return CSR(A.n, A.m, rp.astype(np.int32), rows[order].astype(np.int32), A.val[order])


def identity(n: int, dtype=np.float64) -> CSR:
    return CSR(n, n, np.arange(n + 1, dtype=np.int32), np.arange(n, dtype=np.int32),
               np.ones(n, dtype=dtype))


# ----------------------------------------------------------------------------
# Named configs (BASELINE.json configs[0..4])
# ----------------------------------------------------------------------------

CONFIGS = {
    "C1": dict(desc="2D Poisson 5-point 64x64 fp64: SpMV, A+A^T, A*A", dtype="f64"),
    "C2": dict(desc="3D Poisson 27-point 100^3 fp64: SpMV, A*A", dtype="f64"),
    "C3": dict(desc="R-MAT scale 22 ef 16 fp32: SpMV, A+A^T", dtype="f32"),
    "C4": dict(desc="pathological skew 2M rows fp64: SpMV, A*A", dtype="f64"),
    "C5": dict(desc="random rows ~400M nnz fp64: SpMV, A*A", dtype="f64"),
}


def config(name: str, mode: str = "int", scale: float = 1.0) -> CSR:
    """Matrix A of config `name` with values in `mode`.  `scale` < 1 shrinks the
    large configs (same recipe, fewer rows) for tests that cannot afford the
    full size."""
    num = int(name[1])
    if name == "C1":
        A = poisson2d_5pt(64)
    elif name == "C2":
        k = max(2, int(round(100 * scale ** (1 / 3))))
        A = poisson3d_27pt(k)
    elif name == "C3":
        sc = 22 if scale >= 1.0 else max(8, 22 + int(np.floor(np.log2(scale))))
        A = rmat(sc, 16, seed=22)
    elif name == "C4":
        n = int(2_000_000 * scale)
        A = pathological(n=n, dense_row=min(n - 1, int(1_000_003 * scale)),
                         dense_nnz=int(1_000_000 * scale), tail_empty=n // 4,
                         scattered_empty=n // 4)
    elif name == "C5":
        A = random_rows(n=int(100_000_000 * scale))
    else:
        raise ValueError(name)
    dt = np.float32 if CONFIGS[name]["dtype"] == "f32" else np.float64
    if name in ("C1", "C2"):
        val = A.val.astype(dt) if mode == "int" else random_values(A.nnz, 1000 + num, dt)
    else:
        val = int_values(A.nnz, 100 + num, dt) if mode == "int" else random_values(A.nnz, 1000 + num, dt)
    return A.with_values(val)
