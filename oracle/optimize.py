"""ORACLE (test infrastructure only; see oracle/__init__.py).  Exact optimisers.

These are *not* the paper's method; they solve the paper's optimisation problem
(Eq 5) exactly, by means independent of Eq 24 / Algorithm 1, so that the
selector in oracle/model.py can be pinned against them.

* water_fill_exact   — Eq 5 for affine path times T_i = Ω_i x_i + Δ_i, exact rationals,
                       by a breakpoint scan over Δ-sorted paths (textbook water-filling).
* level_continuous_k — Eq 5 with every staged path at its real optimal k (Eq 17/18),
                       by inverting the quadratic in sqrt(x) and bisecting on the level.
* level_integer_k    — Eq 5 with integer k (Eq 13 is affine in x for fixed k), by
                       bisecting the level on cap_i(T) = max_k (T − c_ik)/s_ik.
* lp_port_exact      — B200 mode (C14): min T over every active subset with scipy's
                       LP solver (a library primitive).
* brute_force        — enumerate θ on a simplex grid × k in 1..K and evaluate O2.
"""
from __future__ import annotations

import itertools
import math
from fractions import Fraction
from typing import List, Sequence

from . import model as M


def water_fill_exact(n, omegas: Sequence, deltas: Sequence):
    """Exact solution of min_x max_{i: x_i>0} (Ω_i x_i + Δ_i), Σ x_i = n, x >= 0.

    Inputs may be Fractions (exact) or floats.  Sort by Δ; for m = 1..p take the m
    smallest-Δ paths as the active set, the level is T_m = (n + Σ Δ/Ω)/Σ 1/Ω; it is
    the optimum when Δ_(m) < T_m <= Δ_(m+1).  Returns (T*, x[])."""
    p = len(omegas)
    order = sorted(range(p), key=lambda i: deltas[i])
    for m in range(1, p + 1):
        act = order[:m]
        inv = sum(1 / omegas[i] for i in act)
        dsum = sum(deltas[i] / omegas[i] for i in act)
        T = (n + dsum) / inv
        nxt = deltas[order[m]] if m < p else None
        if deltas[order[m - 1]] < T and (nxt is None or T <= nxt):
            x = [0] * p
            for i in act:
                x[i] = (T - deltas[i]) / omegas[i]
            return T, x
    raise AssertionError("no consistent active set")


def _inv_quadratic(T, a, b, c):
    """Largest y >= 0 with a y² + b y + c <= T (a > 0, b >= 0); 0 if T <= c."""
    if T <= c:
        return 0.0
    disc = b * b + 4.0 * a * (T - c)
    return (-b + math.sqrt(disc)) / (2.0 * a)


def level_continuous_k(n: float, paths: Sequence[M.Path], mode=M.PAPER, iters=300):
    """Exact optimum of Eq 5 when each staged path runs at its real optimal k*.

    With y = sqrt(x): Eq 17 is T = y²/β + 2 sqrt(α/β') y + ε + α'; Eq 18 is
    T = y²/β' + 2 sqrt((ε+α')/β) y + α; direct T = x/β + α (Eq 6).
    Each inverse x_i(T) is increasing, so bisect on Σ x_i(T) = n."""
    def x_of(T, p):
        if p.kind == M.DIRECT:
            return max(0.0, (T - p.alpha) * p.beta)
        if M.bottleneck_case(p, mode) == 1:
            y = _inv_quadratic(T, 1.0 / p.beta, 2.0 * math.sqrt(p.alpha / p.beta2), p.eps + p.alpha2)
        else:
            y = _inv_quadratic(T, 1.0 / p.beta2, 2.0 * math.sqrt((p.eps + p.alpha2) / p.beta), p.alpha)
        return y * y

    lo, hi = 0.0, 1e-9
    while sum(x_of(hi, p) for p in paths) < n:
        hi *= 2.0
    for _ in range(iters):
        mid = 0.5 * (lo + hi)
        if sum(x_of(mid, p) for p in paths) >= n:
            hi = mid
        else:
            lo = mid
    return hi, [x_of(hi, p) for p in paths]


def level_integer_k(n: float, paths: Sequence[M.Path], k_max=64, mode=M.PAPER, iters=300):
    """Exact optimum of Eq 5 over real x and integer k in 1..k_max, Eq 13 model.

    For fixed k, Eq 13 (paper) is affine in x: case 1 T = kα + ε + α' + x(1/β + 1/(kβ'));
    case 2 T = α + k(ε + α') + x(1/(kβ) + 1/β').  So the capacity of path i at level
    T is max_k (T − c_ik)/s_ik (or 0), increasing in T; bisect on Σ cap_i = n.
    (No issue stagger.)"""
    def affine(p):
        if p.kind == M.DIRECT:
            return [(1.0 / p.beta, p.alpha)]
        out = []
        for k in range(1, k_max + 1):
            if M.bottleneck_case(p, mode) == 1:
                out.append((1.0 / p.beta + 1.0 / (k * p.beta2), k * p.alpha + p.eps + p.alpha2))
            else:
                out.append((1.0 / (k * p.beta) + 1.0 / p.beta2, p.alpha + k * (p.eps + p.alpha2)))
        return out

    lines = [affine(p) for p in paths]

    def cap(T, ls):
        return max(0.0, max((T - c) / s for s, c in ls))

    lo, hi = 0.0, 1e-9
    while sum(cap(hi, ls) for ls in lines) < n:
        hi *= 2.0
    for _ in range(iters):
        mid = 0.5 * (lo + hi)
        if sum(cap(mid, ls) for ls in lines) >= n:
            hi = mid
        else:
            lo = mid
    return hi


def level_integer_k_b200(n: float, paths: Sequence[M.Path], k_max=256, iters=300):
    """Exact optimum of Eq 5 over real x and integer k in 1..k_max with the B200-mode
    exact pipeline time (C3): T = max(T1, T2), T1 = kα + ε + α' + x(1/β + 1/(kβ')),
    T2 = α + k(ε + α') + x(1/(kβ) + 1/β').  At level T path i carries
    max_k min((T − c1)/s1, (T − c2)/s2) bytes (or 0), increasing in T; bisect on
    Σ cap_i = n.  (No issue stagger, no shared port.)  Reading C28: a path with a
    stage-2 availability time A adds T3 = A + k(ε + α') + x/β' to the max."""
    def pieces(p):
        if p.kind == M.DIRECT:
            return [((1.0 / p.beta, p.alpha),)]
        out = []
        for k in range(1, k_max + 1):
            pc = ((1.0 / p.beta + 1.0 / (k * p.beta2), k * p.alpha + p.eps + p.alpha2),
                  (1.0 / (k * p.beta) + 1.0 / p.beta2, p.alpha + k * (p.eps + p.alpha2)))
            if p.wake > 0:  # reading C28: T3 = A + k(ε + α') + x/β'
                pc += ((1.0 / p.beta2, p.wake + k * (p.eps + p.alpha2)),)
            out.append(pc)
        return out

    lines = [pieces(p) for p in paths]

    def cap(T, ls):
        return max(0.0, max(min((T - c) / s for s, c in pc) for pc in ls))

    lo, hi = 0.0, 1e-9
    while sum(cap(hi, ls) for ls in lines) < n:
        hi *= 2.0
    for _ in range(iters):
        mid = 0.5 * (lo + hi)
        if sum(cap(mid, ls) for ls in lines) >= n:
            hi = mid
        else:
            lo = mid
    return hi


def lp_port_exact(n: float, omegas, deltas, weights, port_alpha, port_beta):
    """B200 mode (C14): min T s.t. Ω_i x_i + Δ_i <= T (i in A), Σ w_i x_i <= (T − α_S) β_S,
    Σ x_i = n, x >= 0, minimised over every non-empty active subset A (scipy HiGHS).

    Solved in well-scaled units (θ_i = x_i / n, T in µs) and returned in seconds/bytes."""
    from scipy.optimize import linprog
    us = 1e-6
    p = len(omegas)
    best = (math.inf, None)
    for r in range(1, p + 1):
        for A in itertools.combinations(range(p), r):
            nv = len(A) + 1                       # θ_A..., T[µs]; minimise T
            cost = [0.0] * len(A) + [1.0]
            A_ub, b_ub = [], []
            for j, i in enumerate(A):
                row = [0.0] * nv
                row[j] = omegas[i] * n / us
                row[-1] = -1.0
                A_ub.append(row)
                b_ub.append(-deltas[i] / us)
            if any(weights[i] > 0 for i in A) and port_beta != math.inf:
                A_ub.append([weights[i] * n / port_beta / us for i in A] + [-1.0])
                b_ub.append(-port_alpha / us)
            A_eq = [[1.0] * len(A) + [0.0]]
            res = linprog(cost, A_ub=A_ub, b_ub=b_ub, A_eq=A_eq, b_eq=[1.0],
                          bounds=[(0, None)] * nv, method="highs")
            if res.status == 0 and res.fun * us < best[0]:
                x = [0.0] * p
                for j, i in enumerate(A):
                    x[i] = res.x[j] * n
                best = (res.fun * us, x)
    return best


def simplex_grid(p: int, steps: int):
    """All θ in the p-simplex with coordinates in {0, 1/steps, ..., 1}, θ_0 = remainder."""
    for rest in itertools.product(range(steps + 1), repeat=p - 1):
        if sum(rest) <= steps:
            yield (steps - sum(rest),) + rest


def brute_force(n: int, paths: Sequence[M.Path], opts: M.Options, port=None,
                steps=64, k_values=range(1, 65)):
    """Enumerate every config on the grid (θ step 1/steps; one k per staged path from
    k_values) and evaluate it with O2.  Returns (T_min, bytes, chunks)."""
    p = len(paths)
    best = (math.inf, None, None)
    staged = [i for i in range(p) if paths[i].kind != M.DIRECT]
    for g in simplex_grid(p, steps):
        nbytes = [n * gi // steps for gi in g]
        nbytes[0] += n - sum(nbytes)
        live = [i for i in staged if nbytes[i] > 0]
        for ks in itertools.product(k_values, repeat=len(live)):
            chunks = [1] * p
            for i, k in zip(live, ks):
                chunks[i] = k
            t = M.evaluate(n, nbytes, chunks, paths, opts, port)
            if t < best[0]:
                best = (t, nbytes, chunks)
    return best


def to_fraction_paths(paths: Sequence[M.Path]):
    """Ω_i, Δ_i of the unpipelined model in exact rationals."""
    om, de = [], []
    for p in paths:
        if p.kind == M.DIRECT:
            om.append(1 / Fraction(p.beta))
            de.append(Fraction(p.alpha))
        else:
            om.append(1 / Fraction(p.beta) + 1 / Fraction(p.beta2))
            de.append(Fraction(p.alpha) + Fraction(p.alpha2) + Fraction(p.eps))
    return om, de


def theta_eq24_fraction(n, omegas, deltas) -> List[Fraction]:
    """Eq 24 evaluated in exact rationals (Fractions in, Fractions out)."""
    inv_sum = sum(1 / o for o in omegas)
    delta_sum = sum(d / o for d, o in zip(deltas, omegas))
    return [1 / (o * inv_sum) * (1 - d / n * inv_sum + delta_sum / n) for o, d in zip(omegas, deltas)]
