"""Pure-Python model of the partition rules (TEST INFRASTRUCTURE ONLY).

Used by tests to check GPU tile splits and the multi-GPU row split; never by
the oracle's arithmetic and never by the product path.

* merge_path_split(a, b, d, a_first_on_tie=True): the merge-path diagonal
  search of P:210-224 / Fig 1a: the split (i, d-i) such that the
  first d items of merge(a, b) are a[:i] and b[:d-i].  Ties take `a` first
  (Algorithm 1).
* csr_split(rp, d): the same search on the CSR merge grid of SURVEY §8(a) a1:
  list A = row_end = rp[1:], list B = nonzero indices 0..nnz-1; row end r is
  consumed before nonzero j iff row_end[r] <= j.
* balanced_path_split(a, b, d): merge path followed by the balanced-path
  shift of P:686-790 read as Z23: if a[i-1] == b[j] (matching ranks; always
  rank 0 for unique keys) the split becomes (i, j+1).
"""
from __future__ import annotations

import numpy as np


def merge_path_split(a, b, d: int, a_first_on_tie: bool = True) -> tuple[int, int]:
    lo, hi = max(0, d - len(b)), min(d, len(a))
    while lo < hi:
        mid = (lo + hi) // 2
        # take a[mid] before b[d-mid-1] ?
        if (a[mid] <= b[d - mid - 1]) if a_first_on_tie else (a[mid] < b[d - mid - 1]):
            lo = mid + 1
        else:
            hi = mid
    return lo, d - lo


def merge_order(a, b):
    """Reference merge (A first on ties) -> list of ('a', i) / ('b', j)."""
    i = j = 0
    out = []
    while i < len(a) or j < len(b):
        if j >= len(b) or (i < len(a) and a[i] <= b[j]):
            out.append(("a", i)); i += 1
        else:
            out.append(("b", j)); j += 1
    return out


def csr_split(rp: np.ndarray, d: int) -> tuple[int, int]:
    """Split of the (row_end, nonzero-index) grid at diagonal d -> (rows, nnz)."""
    rp = np.asarray(rp, dtype=np.int64)
    m = rp.size - 1
    nnz = int(rp[-1])
    lo, hi = max(0, d - nnz), min(d, m)
    while lo < hi:
        mid = (lo + hi) // 2
        if rp[mid + 1] <= d - mid - 1:
            lo = mid + 1
        else:
            hi = mid
    return lo, d - lo


def _rank(lst, k: int) -> int:
    """Rank of lst[k] within its run of equal keys."""
    r = 0
    while k - r - 1 >= 0 and lst[k - r - 1] == lst[k]:
        r += 1
    return r


def balanced_path_split(a, b, d: int) -> tuple[int, int]:
    """Merge path, then the starred-diagonal shift (Z23): when a[i-1] and b[j]
    are the same key with the same rank, b[j] joins the left partition."""
    i, j = merge_path_split(a, b, d)
    if 0 < i and j < len(b) and a[i - 1] == b[j] and _rank(a, i - 1) == _rank(b, j):
        j += 1
    return i, j


def row_split(rp: np.ndarray, P: int) -> np.ndarray:
    """Multi-GPU split: R_r = lower_bound(rp, ceil(r nnz / P))."""
    rp = np.asarray(rp, dtype=np.int64)
    nnz = int(rp[-1])
    out = [0]
    for r in range(1, P):
        out.append(int(np.searchsorted(rp, -(-r * nnz // P), side="left")))
    out.append(rp.size - 1)
    return np.array(out, dtype=np.int64)


def balanced_path_split_ranked(a, b, d: int) -> tuple[int, int]:
    """Balanced path for lists WITH duplicate keys (reading R4):
    items are ordered by (key, rank inside the key's run, A before B), so the
    i-th copy of a key in `a` is adjacent to the i-th copy in `b` ("keys with
    matching ranks ... to the same partition").  Returns the split
    (i, j) of diagonal d; i + j == d + 1 when the cut would separate a matched
    pair (the starred diagonal takes the B copy).  For unique keys
    (rank 0 only) this is balanced_path_split (Z23)."""
    import bisect
    a = list(a)
    b = list(b)
    i, j = merge_path_split(a, b, d)
    last = [x for x in (a[i - 1] if i > 0 else None, b[j - 1] if j > 0 else None) if x is not None]
    nxt = [x for x in (a[i] if i < len(a) else None, b[j] if j < len(b) else None) if x is not None]
    if not last or not nxt or max(last) != min(nxt):
        return i, j
    k = max(last)
    a_lo, a_hi = bisect.bisect_left(a, k), bisect.bisect_right(a, k)
    b_lo, b_hi = bisect.bisect_left(b, k), bisect.bisect_right(b, k)
    ca, cb = a_hi - a_lo, b_hi - b_lo
    p = (i - a_lo) + (j - b_lo)          # items of key k before the cut
    m = min(ca, cb)
    if p <= 2 * m:
        ia, ib = (p + 1) // 2, p // 2
        if ia > ib:                      # cut between (k, r) in A and (k, r) in B
            ib += 1
    elif ca > cb:
        ia, ib = p - cb, cb
    else:
        ia, ib = ca, p - ca
    return a_lo + ia, b_lo + ib
