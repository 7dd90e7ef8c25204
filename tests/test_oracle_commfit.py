"""Pins of the communication cost-model fit oracle (reading
R26) against things other than itself: exact recovery of a noiseless line,
numpy's unconstrained least squares and scipy's NNLS on noisy data, the
optimality property on a grid, and the degenerate groups.  CPU only."""
from fractions import Fraction

import numpy as np
import pytest

from oracle import commfit as CF


def sse(a, b, xs, ts):
    return sum((Fraction(t) - a - b * x) ** 2 for x, t in zip(xs, ts))


@pytest.mark.parametrize("seed", range(10))
def test_exact_line_recovered(seed):
    """bytes = k * 10^6, time = alpha + k * beta_fs: a noiseless line in the
    model's own units; the fit returns alpha and beta_fs exactly."""
    rng = np.random.default_rng(seed)
    alpha, beta_fs = int(rng.integers(0, 50_000)), int(rng.integers(0, 80_000))
    ks = rng.integers(0, 5000, int(rng.integers(2, 40)))
    ks[0], ks[1] = 0, 7  # spread
    b = [int(k) * 10**6 for k in ks]
    t = [alpha + int(k) * beta_fs for k in ks]
    a, bb, n = CF.fit_comm(2, [0] * len(b), [1] * len(b), b, t)
    assert (a[0][1], bb[0][1], n[0][1]) == (alpha, beta_fs, len(b))


@pytest.mark.parametrize("seed", range(20))
def test_noisy_matches_numpy_polyfit(seed):
    """Positive intercept and slope: the constraints are inactive, so the fit
    is ordinary least squares -- numpy.polyfit's answer up to its float
    rounding (+-1 after rounding to integers)."""
    rng = np.random.default_rng(100 + seed)
    n = int(rng.integers(5, 300))
    b = rng.integers(1 << 10, 1 << 30, n)
    t = (20_000 + b * 0.04 + rng.normal(0, 2_000, n)).round().astype(np.int64)
    t = np.maximum(t, 0)
    a, bb, _ = CF.fit_comm(2, [1] * n, [0] * n, b.tolist(), t.tolist())
    slope, icpt = np.polyfit(b.astype(np.float64), t.astype(np.float64), 1)
    assert icpt > 0 and slope > 0
    assert abs(a[1][0] - icpt) <= 1.0
    assert abs(bb[1][0] - slope * 1e6) <= 1.0


@pytest.mark.parametrize("seed", range(20))
def test_constrained_matches_scipy_nnls(seed):
    """Data whose unconstrained fit has a negative slope or intercept: the
    result is scipy.optimize.nnls on the design [1, bytes] (float, +-1)."""
    nnls = pytest.importorskip("scipy.optimize").nnls
    rng = np.random.default_rng(200 + seed)
    n = int(rng.integers(4, 200))
    b = rng.integers(0, 1 << 24, n)
    if seed % 2:
        t = (3_000_000 - b * 0.1 + rng.normal(0, 1000, n))  # falling: b = 0 face
    else:
        t = (b * 0.5 - 2_000_000 + rng.normal(0, 1000, n))  # a = 0 face
    t = np.maximum(t.round(), 0).astype(np.int64)
    a, bb, _ = CF.fit_comm(3, [2] * n, [1] * n, b.tolist(), t.tolist())
    scale = 1e6  # bytes in MB for conditioning
    A = np.stack([np.ones(n), b / scale], axis=1)
    x, _ = nnls(A, t.astype(np.float64))
    assert abs(a[2][1] - x[0]) <= 1.0
    assert abs(bb[2][1] - x[1]) <= 1.0  # ns per MB == fs per byte


@pytest.mark.parametrize("seed", range(15))
def test_optimal_on_a_grid(seed):
    """The exact fit (a, b) has an SSE no larger than any feasible point of a
    grid around it (a, b >= 0) -- the definition of a least-squares fit,
    checked in exact arithmetic on small integer data."""
    rng = np.random.default_rng(300 + seed)
    n = int(rng.integers(2, 12))
    xs = [int(v) for v in rng.integers(0, 50, n)]
    ts = [int(v) for v in rng.integers(0, 200, n)]
    a, b = CF.nnls_line(xs, ts)
    assert a >= 0 and b >= 0
    best = sse(a, b, xs, ts)
    for da in np.linspace(-3, 3, 13):
        for db in np.linspace(-0.5, 0.5, 11):
            a2 = a + Fraction(da).limit_denominator(8)
            b2 = b + Fraction(db).limit_denominator(40)
            if a2 >= 0 and b2 >= 0:
                assert sse(a2, b2, xs, ts) >= best


def test_degenerate_groups():
    # no samples -> unknown -> 0; one sample / one size -> mean
    a, b, n = CF.fit_comm(3, [0, 0, 0, 2], [1, 1, 1, 0], [64, 64, 64, 10], [100, 101, 103, 55])
    assert (a[0][1], b[0][1], n[0][1]) == (101, 0, 3)  # mean 101.33 -> 101
    assert (a[2][0], b[2][0], n[2][0]) == (55, 0, 1)
    assert (a[1][2], b[1][2], n[1][2]) == (0, 0, 0)
    assert all(a[d][d] == 0 and b[d][d] == 0 for d in range(3))
    with pytest.raises(ValueError):
        CF.fit_comm(2, [0], [0], [1], [1])
    # rounding is half up: times 1, 2 at one size -> mean 1.5 -> 2
    a, b, _ = CF.fit_comm(2, [0, 0], [1, 1], [5, 5], [1, 2])
    assert a[0][1] == 2
