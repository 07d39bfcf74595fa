"""Pins of the comparator every random-mode GPU parity test relies on:
oracle.check_values implements BJ:5's rule (SURVEY §8(c) "Comparison rule";
DESIGN.md §2): per entry |got - want| <= tau * s with tau = 1e-12 (fp64) /
1e-5 (fp32) and s = sum |a||x| (SpMV) or sum |a||b| (SpGEMM, Z18); s == 0
requires an exact zero; NaN positions must match (Z19).

Each case below is built so that the boundary is exact in binary floating
point (want = 0, so err == got exactly), so a wrong tau, a strict/non-strict
mix-up, an inverted s == 0 rule or a NaN-mask bug fails one of them."""
import numpy as np
import pytest

import oracle

TAU = {np.float64: 1e-12, np.float32: 1e-5}


def chk(got, want, scale, dt):
    return oracle.check_values(np.asarray(got, dt), np.asarray(want, dt), np.asarray(scale, np.float64), dt)[0]


def test_tolerances_are_bj5():
    assert oracle.TOL[np.dtype(np.float64)] == 1e-12
    assert oracle.TOL[np.dtype(np.float32)] == 1e-5


def test_boundary_fp64():
    tau = TAU[np.float64]
    # want = 0 and s = 1: err == got exactly, so tau itself is the boundary
    assert chk([tau], [0.0], [1.0], np.float64)                # exactly tau * s passes
    assert not chk([1.01 * tau], [0.0], [1.0], np.float64)     # 1.01 tau * s fails
    assert not chk([-1.01 * tau], [0.0], [1.0], np.float64)    # sign does not matter
    # scale enters linearly: s = 2^10 allows 2^10 tau, not more
    assert chk([tau * 1024.0], [0.0], [1024.0], np.float64)
    assert not chk([tau * 1024.0 * 1.01], [0.0], [1024.0], np.float64)


def test_boundary_fp32():
    # the float32 result is widened to fp64 exactly, so err == f32(got):
    # the largest float32 at or below tau * s passes, the next one fails
    s = 3.0
    lim = 1e-5 * s
    g = np.float32(lim)
    if float(g) > lim:
        g = np.nextafter(g, np.float32(0), dtype=np.float32)
    assert chk([g], [0.0], [s], np.float32)
    assert not chk([np.nextafter(g, np.float32(1), dtype=np.float32)], [0.0], [s], np.float32)
    assert not chk([g], [0.0], [s / 1.01], np.float32)


def test_fp32_one_ulp_passes():
    # both sides round an fp64 accumulator once (Z4): one ulp of |y| <= s is
    # 2^-23 |y| < 1e-5 s
    for y in (1.0, 3.7, -1234.5, 1e-20, 6e4):
        w = np.float32(y)
        g = np.nextafter(w, np.float32(np.inf), dtype=np.float32)
        assert chk([g], [w], [abs(float(w))], np.float32)
        # ... but 200 ulps (>= 2^-24 * 200 |y| > 1e-5 |y|) is not
        g100 = w
        for _ in range(200):
            g100 = np.nextafter(g100, np.float32(np.inf), dtype=np.float32)
        assert not chk([g100], [w], [abs(float(w))], np.float32)


def test_zero_scale_needs_exact_zero():
    assert chk([0.0], [0.0], [0.0], np.float64)
    assert chk([-0.0], [0.0], [0.0], np.float64)               # signed zero is zero
    assert not chk([1e-300], [0.0], [0.0], np.float64)         # any nonzero fails when s == 0
    assert not chk([5e-324], [0.0], [0.0], np.float64)         # even a denormal
    assert not chk([np.float32(1e-45)], [0.0], [0.0], np.float32)


@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_nan_positions(dt):
    nan = np.nan
    assert chk([nan, 1.0], [nan, 1.0], [1.0, 1.0], dt)            # NaN == NaN (Z19)
    assert not chk([nan, 1.0], [0.0, 1.0], [1.0, 1.0], dt)        # NaN only in got
    assert not chk([0.0, 1.0], [nan, 1.0], [1.0, 1.0], dt)        # NaN only in want
    assert not chk([nan, 2.0], [nan, 1.0], [1.0, 1.0], dt)        # other entries still checked


@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_infinities(dt):
    inf = np.inf
    assert chk([inf, -inf], [inf, -inf], [inf, inf], dt)
    assert not chk([inf], [-inf], [inf], dt)
    assert not chk([inf], [1.0], [1.0], dt)


def test_catches_plausible_gpu_mistakes():
    # a dropped term, a shifted row and a sign error are all far outside tau
    rng = np.random.default_rng(0)
    v = rng.uniform(-1, 1, 1000)
    x = rng.uniform(-1, 1, 1000)
    want = np.cumsum(v * x)[::10]
    s = np.cumsum(np.abs(v * x))[::10]
    assert chk(want, want, s, np.float64)
    assert not chk(want - (v * x)[::10], want, s, np.float64)     # dropped term
    assert not chk(np.roll(want, 1), want, s, np.float64)         # off-by-one row
    assert not chk(-want, want, s, np.float64)                    # sign
    # a reassociated sum of the same terms is within tolerance
    alt = np.array([np.sum((v * x)[:k + 1][::-1]) for k in range(0, 1000, 10)])
    assert chk(alt, want, s, np.float64)


def test_reports_first_failure():
    ok, msg = oracle.check_values(np.array([0.0, 1.0, 3.0]), np.array([0.0, 1.0, 2.0]),
                                  np.array([1.0, 1.0, 1.0]), np.float64)
    assert not ok and "1 entries" in msg and "at 2" in msg and "3.0" in msg
