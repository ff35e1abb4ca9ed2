"""Pins of the oracle model (oracle/model.py) against things other than itself:
hand-worked golden cases (tests/golden/), exact-rational water-filling, closed-form
identities, brute force and a discrete-event pipeline simulation.  CPU only."""
import json
import math
import os
from fractions import Fraction as F

import pytest
from hypothesis import given, settings, strategies as st

from oracle import model as M
from oracle import optimize as O
from oracle.pipeline import simulate_two_stage, stage_times

US, GBS = 1e-6, 1e9
GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "golden_cases.json")))
CASES = {c["id"]: c for c in GOLD["cases"]}
NOSTAG = M.Options(stagger=False)


def mk(d):
    return M.Path(kind=d["kind"], alpha=d["alpha"] * US, beta=d["beta"] * GBS,
                  alpha2=d.get("alpha2", 0) * US,
                  beta2=d["beta2"] * GBS if "beta2" in d else math.inf,
                  eps=d.get("eps", 0) * US)


def rel(a, b):
    return abs(a - b) / max(abs(b), 1e-300)


# --------------------------------------------------------------------------- goldens

def test_G1_hockney():
    c = CASES["G1"]
    p = mk(c["paths"][0])
    assert rel(M.hockney(c["n"], p.alpha, p.beta), float(F(c["expect"]["T_us"])) * US) < 1e-15
    cfg = M.select(c["n"], [p], M.Options(stagger=False, c_min=0, align=1))
    assert cfg.bytes == [c["n"]] and abs(cfg.theta[0] - 1.0) < 1e-15
    assert rel(cfg.t_pred, 22 * US) < 1e-15


@pytest.mark.parametrize("gid", ["G2", "G3"])
def test_G2_G3_closed_forms(gid):
    c = CASES[gid]
    paths = [mk(d) for d in c["paths"]]
    n = c["n"]
    exp_theta = [float(F(t)) for t in c["expect"]["theta"]]
    om, de = zip(*[M.omega_delta_unpipelined(p) for p in paths])
    th = M.theta_eq24(n, om, de)
    for a, b in zip(th, exp_theta):
        assert abs(a - b) < 1e-12
    assert rel(M.level_eq24(n, om, de), float(F(c["expect"]["T_us"])) * US) < 1e-12
    # Theorem 1: every path finishes at the same time
    ts = [M.path_time_unpipelined(t, n, p) for t, p in zip(th, paths)]
    assert max(ts) - min(ts) < 1e-18
    if gid == "G2":
        th8 = M.theta_eq8(n, [p.alpha for p in paths], [p.beta for p in paths])
        for a, b in zip(th8, exp_theta):
            assert abs(a - b) < 1e-12


def test_G2_G3_exact_rational():
    # Exact rationals in µs and B/µs: Eq 24 and the water-filling optimum agree exactly.
    for gid in ("G2", "G3"):
        c = CASES[gid]
        om, de = [], []
        for d in c["paths"]:
            if d["kind"] == 0:
                om.append(F(1, d["beta"] * 1000))
                de.append(F(d["alpha"]))
            else:
                om.append(F(1, d["beta"] * 1000) + F(1, d["beta2"] * 1000))
                de.append(F(d["alpha"]) + F(d["alpha2"]) + F(d["eps"]))
        n = F(c["n"])
        th = O.theta_eq24_fraction(n, om, de)
        assert th == [F(t) for t in c["expect"]["theta"]]
        T, x = O.water_fill_exact(n, om, de)
        assert T == F(c["expect"]["T_us"])
        assert [xi / n for xi in x] == th


def test_G4_active_set():
    c = CASES["G4"]
    paths = [mk(d) for d in c["paths"]]
    n = c["n"]
    om, de = zip(*[M.omega_delta_unpipelined(p) for p in paths])
    raw = M.theta_eq24(n, om, de)
    for a, b in zip(raw, c["expect"]["raw_theta"]):
        assert abs(a - float(F(b))) < 1e-12
    assert rel(M.level_eq24(n, om, de), 3 * US) < 1e-12
    theta, T, act = M._solve_level_paper(float(n), om, de, paths, [True, True], NOSTAG)
    assert act == [True, False]
    assert abs(theta[0] - 1.0) < 1e-15 and theta[1] == 0.0
    assert rel(T, 2.5 * US) < 1e-12
    assert de[1] >= T       # the excluded path's Δ is above the level (C1)


@pytest.mark.parametrize("gid", ["G5", "G7"])
def test_G5_G7_pipeline(gid):
    c = CASES[gid]
    p = mk(c["path"])
    x = c["x"]
    e = c["expect"]
    assert M.bottleneck_case(p) == e["case"]
    ks = M.k_opt(x, p)
    assert rel(ks * ks, float(F(e["k_star_sq"]))) < 1e-12
    assert rel(M.t_at_k_opt(x, p), e["T_kstar_us"] * US) < 1e-12
    for k, t in e["T_k_us"].items():
        assert rel(M.pipelined_time(float(x), int(k), p), float(F(t)) * US) < 1e-12
    assert M.k_integer(ks) == e["k_int"]


def test_G6_two_pass_phi():
    c = CASES["G6"]
    p = mk(c["path"])
    x = c["x"]
    e = c["expect"]
    phi = M.phi_two_pass(x, p)
    assert rel(phi, e["phi"]) < 1e-12
    assert rel(M.k_eq19(x, phi, p), e["k19"]) < 1e-12
    om, de = M.omega_delta_eq22(phi, p)
    assert rel(om, e["Omega_s_per_B"]) < 1e-12
    assert rel(de, e["Delta_us"] * US) < 1e-12
    assert rel(x * om + de, e["T21_us"] * US) < 1e-12


# --------------------------------------------------------------------------- identities

staged = st.builds(
    lambda a, b, a2, b2, e: M.Path(M.GPU_STAGED, a * US, b * GBS, a2 * US, b2 * GBS, e * US),
    st.floats(0.2, 20), st.floats(10, 900), st.floats(0.2, 20), st.floats(10, 900), st.floats(0.1, 20))


@settings(max_examples=200, deadline=None)
@given(staged, st.floats(1e4, 4e9))
def test_eq17_18_is_eq13_at_real_kstar(p, x):
    # Eq 17/18 equal the Eq 13 case expression evaluated at the real k* of Eq 14/15.
    ks = M.k_opt(x, p)
    m = x / ks
    if M.bottleneck_case(p) == 1:
        t13 = ks * (p.alpha + m / p.beta) + p.eps + p.alpha2 + m / p.beta2
    else:
        t13 = p.alpha + m / p.beta + ks * (p.eps + p.alpha2 + m / p.beta2)
    assert rel(M.t_at_k_opt(x, p), t13) < 1e-12


@settings(max_examples=200, deadline=None)
@given(staged, st.floats(1e4, 4e9), st.floats(0.05, 20))
def test_eq19_20_22_identities(p, x, phi):
    # Eq 19 substituted into Eq 13 gives Eq 20, which is Eq 21 with Eq 22's Ω, Δ.
    k = M.k_eq19(x, phi, p)
    m = x / k
    if M.bottleneck_case(p) == 1:
        t13 = k * (p.alpha + m / p.beta) + p.eps + p.alpha2 + m / p.beta2
    else:
        t13 = p.alpha + m / p.beta + k * (p.eps + p.alpha2 + m / p.beta2)
    assert rel(M.t_eq20(x, phi, p), t13) < 1e-10
    om, de = M.omega_delta_eq22(phi, p)
    assert rel(x * om + de, t13) < 1e-10


@settings(max_examples=200, deadline=None)
@given(staged, st.floats(1e4, 4e9))
def test_two_pass_phi_reproduces_eq14_15(p, x):
    # Reading C4: with c = 1, Eq 19 at θ⁽⁰⁾ is Eq 14/15 and Eq 21 is Eq 17/18.
    phi = M.phi_two_pass(x, p)
    assert rel(M.k_eq19(x, phi, p), M.k_opt(x, p)) < 1e-12
    om, de = M.omega_delta_eq22(phi, p)
    assert rel(x * om + de, M.t_at_k_opt(x, p)) < 1e-12


@settings(max_examples=300, deadline=None)
@given(st.floats(0.01, 400))
def test_k_integer_is_exact_argmin(ks):
    # C5: for f(k) = A k + B/k with B/A = ks², the rule returns the smallest integer argmin;
    # and that argmin lies in {floor(k*), ceil(k*)} (Eq 14/15's derivative).
    A = 1.0
    B = ks * ks
    vals = {k: A * k + B / k for k in range(1, 500)}
    best = min(vals.values())
    argmins = [k for k, v in vals.items() if v <= best * (1 + 1e-13)]
    k = M.k_integer(ks)
    assert k == min(argmins) or abs(vals[k] - best) <= best * 1e-13
    assert k in (max(1, math.floor(ks)), math.ceil(ks)) or ks < 1


def test_eq11_reduces_to_eq8():
    # Ω = 1/β, Δ = α in Eq 11 gives Eq 8 exactly (rationals).
    al = [F(1), F(3), F(7, 2)]
    be = [F(100000), F(50000), F(70000)]
    n = F(5 * 10 ** 6)
    om = [1 / b for b in be]
    th11 = O.theta_eq24_fraction(n, om, al)
    sb = sum(be)
    sab = sum(a * b for a, b in zip(al, be))
    th8 = [b / sb * (1 - a / n * sb + sab / n) for a, b in zip(al, be)]
    assert th11 == th8
    assert sum(th11) == 1


@settings(max_examples=150, deadline=None)
@given(st.lists(st.tuples(st.integers(1, 40), st.integers(1, 900)), min_size=2, max_size=6),
       st.integers(10 ** 5, 10 ** 9))
def test_eq24_active_set_equals_water_filling(ps, n):
    # The C2 active-set loop over Eq 24 reaches the exact water-filling optimum
    # (an independent breakpoint-scan algorithm in exact rationals).
    paths = [M.Path(M.DIRECT, a * US, b * GBS) for a, b in ps]
    om, de = zip(*[M.omega_delta_unpipelined(p) for p in paths])
    theta, T, act = M._solve_level_paper(float(n), om, de, paths, [True] * len(paths), NOSTAG)
    omF = [F(1, b * 1000) for _, b in ps]
    deF = [F(a) for a, _ in ps]
    Tx, x = O.water_fill_exact(F(n), omF, deF)
    assert rel(T, float(Tx) * US) < 1e-9
    for t, xi in zip(theta, x):
        assert abs(t - float(xi / n)) < 1e-9
    assert abs(sum(theta) - 1) < 1e-12
    # Theorem 1 on the active set; inactive paths have Δ >= T (C1)
    for i, p in enumerate(paths):
        if act[i]:
            assert rel(M.path_time_unpipelined(theta[i], n, p), T) < 1e-9
        else:
            assert de[i] >= T * (1 - 1e-12)


@settings(max_examples=100, deadline=None)
@given(st.lists(st.tuples(st.integers(1, 40), st.integers(10, 900)), min_size=2, max_size=5),
       st.integers(10 ** 6, 10 ** 9), st.integers(0, 4), st.floats(1.05, 3.0))
def test_monotonicity_P184(ps, n, i, factor):
    # a larger β_i gives a larger θ_i; a larger α_i a smaller θ_i (on the active set).
    i = i % len(ps)
    paths = [M.Path(M.DIRECT, a * US, b * GBS) for a, b in ps]

    def th(paths):
        om, de = zip(*[M.omega_delta_unpipelined(p) for p in paths])
        return M._solve_level_paper(float(n), om, de, paths, [True] * len(paths), NOSTAG)[0]

    base = th(paths)
    up_b = list(paths)
    up_b[i] = M.Path(M.DIRECT, paths[i].alpha, paths[i].beta * factor)
    up_a = list(paths)
    up_a[i] = M.Path(M.DIRECT, paths[i].alpha * factor, paths[i].beta)
    assert th(up_b)[i] >= base[i] - 1e-12
    assert th(up_a)[i] <= base[i] + 1e-12


def test_eq8_grid_brute_force():
    # The Eq 8 optimum is below every grid point and within one grid step of the best.
    paths = [M.Path(M.DIRECT, 1 * US, 100 * GBS), M.Path(M.DIRECT, 3 * US, 50 * GBS),
             M.Path(M.DIRECT, 2 * US, 70 * GBS)]
    n = 4_000_000
    om, de = zip(*[M.omega_delta_unpipelined(p) for p in paths])
    T = M.level_eq24(n, om, de)
    steps = 256
    best = min(M.total_time_unpipelined([g / steps for g in gr], n, paths)
               for gr in O.simplex_grid(3, steps))
    assert T <= best * (1 + 1e-12)
    assert best <= T + n * max(om) / steps


# --------------------------------------------------------------------------- Eq 13 vs DES

@settings(max_examples=200, deadline=None)
@given(staged, st.floats(1e5, 2e9), st.integers(1, 64))
def test_eq13_matches_pipeline_simulation(p, x, k):
    s1, s2 = stage_times(x, k, p.alpha, p.beta, p.eps, p.alpha2, p.beta2)
    sim = simulate_two_stage(k, s1, s2)
    # B200 mode is the exact pipeline for every case (C3) …
    assert rel(M.pipelined_time(x, k, p, M.B200), sim) < 1e-12
    # … and Eq 13 (paper) agrees whenever its case names the true bottleneck stage.
    case = M.bottleneck_case(p)
    if (case == 1 and s1 >= s2) or (case == 2 and s2 >= s1):
        assert rel(M.pipelined_time(x, k, p, M.PAPER), sim) < 1e-12
    else:
        assert M.pipelined_time(x, k, p, M.PAPER) <= sim * (1 + 1e-12)


def test_des_finite_ring_never_faster():
    for k in (1, 3, 8, 20):
        for s1, s2 in ((1.0, 2.0), (2.0, 1.0), (1.0, 1.0)):
            inf = simulate_two_stage(k, s1, s2)
            assert simulate_two_stage(k, s1, s2, slots=2) >= inf - 1e-15
            assert simulate_two_stage(k, s1, s2, slots=k) == inf


# ------------------------------------------------- reading C28: stage-2 availability (wake)

@settings(max_examples=200, deadline=None)
@given(staged, st.floats(1e5, 2e9), st.integers(1, 64), st.floats(0, 500))
def test_c28_wake_matches_pipeline_simulation(p, x, k, wake_us):
    # B200 mode with a relay that starts A after the message: the closed form
    # max(s1 + s2 + (k−1)·max(s1, s2), A + k·s2) against the event simulation whose
    # second link is busy until A (oracle/pipeline.py, chunk by chunk)
    import dataclasses
    q = dataclasses.replace(p, wake=wake_us * US)
    s1, s2 = stage_times(x, k, q.alpha, q.beta, q.eps, q.alpha2, q.beta2)
    assert rel(M.pipelined_time(x, k, q, M.B200), simulate_two_stage(k, s1, s2, start2=q.wake)) < 1e-12
    # the wake only ever delays, and A = 0 is C3 exactly
    assert M.pipelined_time(x, k, q, M.B200) >= M.pipelined_time(x, k, p, M.B200)
    assert simulate_two_stage(k, s1, s2, start2=0.0) == simulate_two_stage(k, s1, s2)


def test_c28_wake_special_cases():
    # A huge wake: the second link alone after A, k·s2; k = 1 store-and-forward: s1 + s2
    # unless the relay is not up yet (max(s1, A) + s2)
    p = M.Path(M.GPU_STAGED, 2 * US, 400 * GBS, 3 * US, 500 * GBS, 1 * US, wake=10e-3)
    x = 64 * 2 ** 20
    for k in (1, 4, 32):
        s2 = p.eps + p.alpha2 + x / k / p.beta2
        assert M.pipelined_time(x, k, p, M.B200) == pytest.approx(p.wake + k * s2, rel=1e-15)
    p = M.Path(M.GPU_STAGED, 2 * US, 400 * GBS, 3 * US, 500 * GBS, 1 * US, wake=5 * US)
    s1 = p.alpha + x / p.beta
    s2 = p.eps + p.alpha2 + x / p.beta2
    assert M.pipelined_time(x, 1, p, M.B200) == pytest.approx(max(s1, p.wake) + s2, rel=1e-15)
