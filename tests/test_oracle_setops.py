"""Pins of the set-operation oracle and the ranked balanced-path model
(P:686-810), against definitions independent of both:
Python's multiset arithmetic (collections.Counter: | & - are max / min /
truncated difference of multiplicities), brute-force rank enumeration for the
values, identities, and the paper's Fig 1 lists."""
import bisect
import collections
import json
from pathlib import Path

import numpy as np
import pytest

import oracle
from oracle.partition_model import balanced_path_split_ranked, merge_order

GOLD = json.loads((Path(__file__).parent / "golden" / "fig1_partition.json").read_text())


def expand(cnt: collections.Counter) -> list:
    return sorted(cnt.elements())


def counter_op(op, a, b):
    ca, cb = collections.Counter(a), collections.Counter(b)
    return {"union": ca | cb, "intersection": ca & cb, "difference": ca - cb,
            "symmetric_difference": (ca - cb) + (cb - ca)}[op]


def rand_multiset(rng, n, hi):
    return np.sort(rng.integers(0, hi, size=n)).astype(np.uint32)


@pytest.mark.parametrize("op", list(oracle.SET_OPS))
def test_counter_semantics(op):
    rng = np.random.default_rng(7)
    for _ in range(300):
        a = rand_multiset(rng, int(rng.integers(0, 20)), int(rng.integers(1, 8)))
        b = rand_multiset(rng, int(rng.integers(0, 20)), int(rng.integers(1, 8)))
        got, _ = oracle.set_op(op, a, b)
        assert got.tolist() == expand(counter_op(op, a.tolist(), b.tolist()))


def test_values_follow_key_rank_pairs():
    """Brute force: the r-th copy of key k in A is paired with the r-th copy in
    B; matched pairs keep A's value, the rest keep their own side's value."""
    rng = np.random.default_rng(11)
    for _ in range(200):
        a = rand_multiset(rng, int(rng.integers(0, 16)), 5)
        b = rand_multiset(rng, int(rng.integers(0, 16)), 5)
        av = rng.integers(0, 1000, size=a.size).astype(np.int64)
        bv = rng.integers(1000, 2000, size=b.size).astype(np.int64)
        for op in oracle.SET_OPS:
            exp = []
            for k in sorted(set(a.tolist()) | set(b.tolist())):
                va = [int(v) for kk, v in zip(a, av) if kk == k]
                vb = [int(v) for kk, v in zip(b, bv) if kk == k]
                m = min(len(va), len(vb))
                if op in ("union", "intersection"):
                    exp += [(k, v) for v in va[:m]]
                if op in ("union", "difference", "symmetric_difference"):
                    exp += [(k, v) for v in va[m:]]
                if op in ("union", "symmetric_difference"):
                    exp += [(k, v) for v in vb[m:]]
            keys, vals = oracle.set_op(op, a, b, av, bv)
            assert list(zip(keys.tolist(), vals.tolist())) == exp, op


def test_identities_and_widths():
    rng = np.random.default_rng(3)
    a = rand_multiset(rng, 500, 100)
    e = np.zeros(0, np.uint32)
    assert np.array_equal(oracle.set_op("union", a, e)[0], a)
    assert np.array_equal(oracle.set_op("intersection", a, a)[0], a)
    assert oracle.set_op("difference", a, a)[0].size == 0
    assert oracle.set_op("symmetric_difference", a, a)[0].size == 0
    # 64-bit keys above 2^32 keep unsigned order
    a64 = np.sort(rng.integers(0, 2**63, size=300, dtype=np.int64).astype(np.uint64) * np.uint64(2))
    b64 = np.sort(np.concatenate([a64[::3], a64[1::7] + np.uint64(1)]))
    got = oracle.set_op("union", a64, b64)[0]
    assert got.dtype == np.uint64 and np.all(np.diff(got.astype(object)) >= 0)
    assert got.tolist() == expand(collections.Counter(a64.tolist()) | collections.Counter(b64.tolist()))


def test_fig1_lists_union():
    """Fig 1 lists: A = a b c c c e, B = c c c c d f."""
    a = np.array([ord(c) for c in GOLD["A"]], np.uint32)
    b = np.array([ord(c) for c in GOLD["B"]], np.uint32)
    u = oracle.set_op("union", a, b)[0]
    assert "".join(map(chr, u)) == "abccccdef"
    assert "".join(map(chr, oracle.set_op("intersection", a, b)[0])) == "ccc"


def test_ranked_balanced_path_fig1():
    A, B = GOLD["A"], GOLD["B"]
    splits = [balanced_path_split_ranked(A, B, d) for d in GOLD["diagonals"]]
    assert [list(s) for s in splits] == GOLD["balanced_path_ranked_splits"]
    cuts = [(0, 0)] + splits + [(len(A), len(B))]
    assert [(c1[0] + c1[1]) - (c0[0] + c0[1]) for c0, c1 in zip(cuts, cuts[1:])] == GOLD["balanced_thread_sizes"]


def test_ranked_balanced_path_keeps_pairs():
    """Every cut: i + j in {d, d+1}; for every key the matched copies consumed
    on both sides are equal (no key-rank pair straddles the cut); cuts are
    monotone; unique keys reduce to merge path + the Z23 shift."""
    rng = np.random.default_rng(5)
    for _ in range(200):
        a = sorted(rng.integers(0, 6, size=int(rng.integers(0, 18))).tolist())
        b = sorted(rng.integers(0, 6, size=int(rng.integers(0, 18))).tolist())
        prev = (0, 0)
        for d in range(len(a) + len(b) + 1):
            i, j = balanced_path_split_ranked(a, b, d)
            assert i + j in (d, d + 1) and i >= prev[0] and j >= prev[1]
            prev = (i, j)
            for k in set(a) | set(b):
                ca, cb = a.count(k), b.count(k)
                ua = min(max(i - bisect.bisect_left(a, k), 0), ca)
                ub = min(max(j - bisect.bisect_left(b, k), 0), cb)
                assert min(ua, cb) == min(ub, ca), (a, b, d, k)
    # unique keys: merge order prefix + the rank-0 shift
    a, b = [1, 3, 5, 7], [3, 4, 7, 8]
    for d in range(9):
        i, j = balanced_path_split_ranked(a, b, d)
        mo = merge_order(a, b)[:d]
        i0, j0 = sum(s == "a" for s, _ in mo), sum(s == "b" for s, _ in mo)
        assert (i, j) == ((i0, j0 + 1) if i0 > 0 and j0 < len(b) and a[i0 - 1] == b[j0] else (i0, j0))
