"""Pins of the Step-1 fit (oracle/calibration.py, reading C12) and parity of the
library's mp_fit_hockney with it.  CPU only."""
from fractions import Fraction as F

import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

from oracle import calibration as OC
from paper_conf_sc_sojoodiasfga25_b200 import mp


def exact_weighted_normal_equations(n, t):
    """The same weighted least squares in exact rationals (normal equations, 2×2)."""
    n = [F(x) for x in n]
    t = [F(x) for x in t]
    w = [1 / (ti * ti) for ti in t]
    s00 = sum(w)
    s01 = sum(wi * ni for wi, ni in zip(w, n))
    s11 = sum(wi * ni * ni for wi, ni in zip(w, n))
    r0 = sum(wi * ti for wi, ti in zip(w, t))
    r1 = sum(wi * ni * ti for wi, ni, ti in zip(w, n, t))
    det = s00 * s11 - s01 * s01
    return (r0 * s11 - r1 * s01) / det, (s00 * r1 - s01 * r0) / det


@settings(max_examples=100, deadline=None)
@given(st.floats(1e-6, 5e-5), st.floats(1e10, 5e12), st.lists(st.integers(20, 31), min_size=2, max_size=8,
                                                              unique=True))
def test_noiseless_recovery(alpha, beta, exps):
    # Eq 1 exactly: T = α + n/β is recovered (to rounding) from any ≥ 2 distinct sizes
    n = [float(1 << e) for e in sorted(exps)]
    t = [alpha + x / beta for x in n]
    a, b = OC.fit_hockney(n, t)
    assert abs(a - alpha) <= 1e-9 * alpha + 1e-15 and abs(b - beta) <= 1e-9 * beta


@settings(max_examples=100, deadline=None)
@given(st.lists(st.tuples(st.integers(1, 2000), st.integers(1, 500)), min_size=3, max_size=8, unique_by=lambda x: x[0]))
def test_matches_exact_rational_normal_equations(pts):
    n = [float(p[0] * 1024 * 1024) for p in pts]
    t = [float(p[1]) * 1e-5 + 1e-6 for p in pts]
    a_ex, g_ex = exact_weighted_normal_equations(n, t)
    a, b = OC.fit_hockney(n, t)
    if g_ex > 0 and a_ex > F(1, 10 ** 7):
        assert abs(a - float(a_ex)) <= 1e-9 * abs(float(a_ex)) + 1e-12
        assert abs(1 / b - float(g_ex)) <= 1e-9 * float(g_ex)


def objective(n, t, a, g):
    return sum(((ti - a - ni * g) / ti) ** 2 for ni, ti in zip(n, t))


def test_clamps():
    # negative intercept → α = 1e-7 with the slope refitted; decreasing times → slope
    # from the last sample
    a, b = OC.fit_hockney([1e6, 2e6, 4e6], [1e-6, 3e-6, 7e-6])
    assert a == 1e-7
    a, b = OC.fit_hockney([1e6, 2e6], [2e-5, 1e-5])
    assert b == 2e6 / 1e-5


@settings(max_examples=100, deadline=None)
@given(st.lists(st.tuples(st.integers(1, 4000), st.integers(1, 500)), min_size=2, max_size=8,
                unique_by=lambda x: x[0]))
def test_clamped_fit_is_the_constrained_optimum(pts):
    # the L2 -> HBM cliff of a size band makes times grow faster than linearly, and
    # the free fit's intercept goes negative; the clamped fit must then be the optimum
    # of the objective on the constraint α = 1e-7: the exact rational 1-D normal
    # equation, and no nearby slope does better (convexity)
    n = [float(p[0] * 65536) for p in pts]
    t = [float(p[1]) * 1e-6 * (1 + p[0] / 400) for p in pts]   # super-linear in n
    a_ex, g_ex = exact_weighted_normal_equations(n, t) if len(n) > 2 or n[0] != n[1] else (None, None)
    a, b = OC.fit_hockney(n, t)
    if a_ex is None or a_ex > F(1, 10 ** 7):
        return
    assert a == 1e-7
    nF = [F(x) for x in n]
    tF = [F(x) for x in t]
    a0 = F(1, 10 ** 7)
    g1 = sum((ti - a0) * ni / ti ** 2 for ni, ti in zip(nF, tF)) / sum(ni * ni / ti ** 2 for ni, ti in zip(nF, tF))
    if g1 <= 0:
        return
    assert abs(1 / b - float(g1)) <= 1e-9 * float(g1)
    g = 1 / b
    f0 = objective(n, t, a, g)
    for d in (1e-4, -1e-4, 1e-2, -1e-2):
        assert objective(n, t, a, g * (1 + d)) >= f0 * (1 - 1e-12)


@settings(max_examples=200, deadline=None)
@given(st.floats(1e-6, 5e-5), st.floats(1e10, 5e12),
       st.lists(st.tuples(st.integers(16, 31), st.floats(-0.2, 0.2)), min_size=2, max_size=10,
                unique_by=lambda x: x[0]))
def test_library_fit_parity(alpha, beta, pts):
    # the fit's domain: calibration schedules (power-of-two sizes) with ±20 % timing noise
    n = [float(1 << e) for e, _ in pts]
    t = [(alpha + x / beta) * (1 + z) for x, (_, z) in zip(n, pts)]
    a_o, b_o = OC.fit_hockney(n, t)
    a_l, b_l = mp.fit_hockney(n, t)
    assert abs(a_l - a_o) <= 1e-7 * abs(a_o) + 1e-13
    assert abs(b_l - b_o) <= 1e-7 * abs(b_o)


def test_library_fit_rejects_bad_input():
    with pytest.raises(mp.MPError):
        mp.fit_hockney([1.0], [1.0])
    with pytest.raises(mp.MPError):
        mp.fit_hockney([1.0, 2.0], [1.0, 0.0])
