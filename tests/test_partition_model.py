"""Pins of the Python partition model against Fig 1 (re-derived, Z24), the CSR
grid example and brute-force merges."""
import numpy as np

from oracle.partition_model import (balanced_path_split, csr_split, merge_order,
                                    merge_path_split)
from tests.conftest import load_golden


def test_fig1():
    g = load_golden("fig1_partition.json")
    a, b = g["A"], g["B"]
    assert [list(merge_path_split(a, b, d)) for d in g["diagonals"]] == g["merge_path_splits"]
    bal = [balanced_path_split(a, b, d) for d in g["diagonals"]]
    assert [list(x) for x in bal] == g["balanced_path_splits"]
    pts = [(0, 0)] + bal + [(len(a), len(b))]
    sizes = [(pts[t + 1][0] - pts[t][0]) + (pts[t + 1][1] - pts[t][1]) for t in range(4)]
    assert sizes == g["balanced_thread_sizes"]


def test_csr_grid_example():
    g = load_golden("fig1_partition.json")["csr_grid"]
    assert [list(csr_split(g["rp"], d)) for d in g["diagonals"]] == g["splits"]


def test_merge_path_matches_bruteforce():
    rng = np.random.default_rng(0)
    for _ in range(200):
        a = np.sort(rng.integers(0, 12, rng.integers(0, 15)))
        b = np.sort(rng.integers(0, 12, rng.integers(0, 15)))
        order = merge_order(list(a), list(b))
        for d in range(len(a) + len(b) + 1):
            i, j = merge_path_split(a, b, d)
            assert i == sum(1 for s, _ in order[:d] if s == "a") and i + j == d


def test_csr_split_matches_bruteforce():
    rng = np.random.default_rng(1)
    for _ in range(100):
        m = int(rng.integers(0, 12))
        lens = rng.integers(0, 5, m)
        rp = np.concatenate([[0], np.cumsum(lens)])
        nnz = int(rp[-1])
        # merge items: row-end r before nonzero j iff rp[r+1] <= j
        items = []
        r = j = 0
        while r < m or j < nnz:
            if r < m and (j >= nnz or rp[r + 1] <= j):
                items.append("r"); r += 1
            else:
                items.append("n"); j += 1
        for d in range(m + nnz + 1):
            i, jj = csr_split(rp, d)
            assert i == items[:d].count("r") and jj == items[:d].count("n")


def test_balanced_never_splits_pairs():
    rng = np.random.default_rng(2)
    for _ in range(200):
        a = np.unique(rng.integers(0, 30, rng.integers(0, 20)))
        b = np.unique(rng.integers(0, 30, rng.integers(0, 20)))
        for d in range(len(a) + len(b) + 1):
            i, j = balanced_path_split(a, b, d)
            # a matched pair (a[x] == b[y]) lies on one side of the split
            if i > 0 and j < len(b):
                assert a[i - 1] != b[j]
            if j > 0 and i < len(a):
                assert a[i] != b[j - 1]
