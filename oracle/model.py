"""ORACLE (test infrastructure only; see oracle/__init__.py).  Model + selector.

Plain fp64 restatement of the extended-Hockney multi-path model of
PAPER.md §3 (Eq 1-24) and of Algorithm 1 (§4), with the readings
of the garbled / silent passages listed in DESIGN.md §3 ("Readings", C1-C17).

Units (C11): bytes, seconds, bytes/second.

Every function cites the passage it follows.  No blocking, fusion or reordering
beyond the paper's own formula order.

Parity status
-------------
* ``hockney``, ``path_time_unpipelined``, ``total_time_unpipelined``, ``theta_eq8``,
  ``theta_eq24``, ``pipelined_time``, ``k_opt``, ``t_at_k_opt``, ``phi_two_pass``,
  ``omega_delta_eq22``, ``k_integer``, ``evaluate``: pinned by tests/test_oracle_model.py
  (golden hand-worked cases G1-G7 in tests/golden/, exact-rational water-filling,
  brute force, a discrete-event pipeline simulation, closed-form identities).
* ``select``: pinned against brute-force grids and the exact optimisers in
  oracle/optimize.py (selector quality, Theorem 1 invariant, Σ shares = n).
* Calibrated α/β/ε/φ values on B200 hardware: parity unpinned (the paper prints
  no values).
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field, replace
from typing import List, Optional, Sequence

# Path kinds, P:107-111 (§3.1): (1) Direct, (2) GPU-staged, (3) Host-staged.
DIRECT, GPU_STAGED, HOST_STAGED = 0, 1, 2
# Model modes (C3/C8/C14): the paper verbatim, or the B200 extension
# (exact two-stage pipeline, calibrated issue stagger, one shared port).
PAPER, B200 = 0, 1

INF = math.inf


@dataclass
class Path:
    """Per-path model parameters, Table 1."""
    kind: int
    alpha: float            # α_i   startup latency of the first link [s]
    beta: float             # β_i   bandwidth of the first link [B/s]
    alpha2: float = 0.0     # α'_i  second link (staged paths only) [s]
    beta2: float = INF      # β'_i  [B/s]; INF for a direct path (1/β' = 0)
    eps: float = 0.0        # ε_i   synchronisation overhead at the staging device [s]
    c: float = 1.0          # multiplier of the topology constant φ (C4)
    sigma: float = 0.0      # issue latency counted by the stagger in B200 mode (C8)
    w: float = 0.0          # bytes of shared-port traffic per payload byte (C14)
    via: int = -1           # relay device (GPU-staged) or -1
    wake: float = 0.0       # B200 mode (C28): earliest start of stage 2 after the message starts [s]


@dataclass
class Port:
    """One shared port (B200 mode, C14): T >= alpha + sum_i w_i b_i / beta."""
    alpha: float = 0.0
    beta: float = INF


@dataclass
class Options:
    mode: int = PAPER
    stagger: bool = True        # Alg 1 line 17 / P:318 ("add previous α to Δ_i")
    align: int = 256            # share alignment A (C7)
    c_min: int = 64 * 1024      # smallest staged share / chunk (C5, C7)
    k_max: int = 1024           # chunk-count cap (C5)
    slot_bytes: int = 0         # largest chunk the staging ring holds (0 = no limit)
    refine: Optional[bool] = None   # pass 3 (C18); None = on in B200 mode only


@dataclass
class Config:
    """Alg 1 output: configs[] (chunks) and shares[] (bytes)."""
    bytes: List[int]
    chunks: List[int]
    theta: List[float] = field(default_factory=list)
    t_pred: float = 0.0         # O2 evaluation of this config
    t_level: float = 0.0        # linearised common finish time (Eq 21 level)
    theta_level: List[float] = field(default_factory=list)  # θ of the last level solve (Σ = 1)


# ----------------------------------------------------------------------------- §3.1

def hockney(n: float, alpha: float, beta: float) -> float:
    """Eq 1: T = α + n/β."""
    return alpha + n / beta


def path_time_unpipelined(theta: float, n: float, p: Path) -> float:
    """Eq 2: T_i = α_i + θ_i n/β_i + ε_i + α'_i + θ_i n/β'_i.

    A direct path is Eq 2 with α' = ε = 0 and 1/β' = 0 (Eq 6)."""
    if p.kind == DIRECT:
        return p.alpha + theta * n / p.beta
    return p.alpha + theta * n / p.beta + p.eps + p.alpha2 + theta * n / p.beta2


def total_time_unpipelined(thetas: Sequence[float], n: float, paths: Sequence[Path]) -> float:
    """Eq 4: T = max_i T_i over the paths that carry data (θ_i > 0)."""
    return max(path_time_unpipelined(t, n, p) for t, p in zip(thetas, paths) if t > 0)


# ----------------------------------------------------------------------------- §3.2-3.3

def omega_delta_unpipelined(p: Path):
    """Definitions after Eq 9: Ω_i = 1/β_i + 1/β'_i, Δ_i = α_i + α'_i + ε_i.
    Direct path: Ω_i = 1/β_i, Δ_i = α_i."""
    if p.kind == DIRECT:
        return 1.0 / p.beta, p.alpha
    return 1.0 / p.beta + 1.0 / p.beta2, p.alpha + p.alpha2 + p.eps


def theta_eq8(n: float, alphas: Sequence[float], betas: Sequence[float]) -> List[float]:
    """Eq 8: θ_i = β_i/Σβ_j · (1 − α_i Σβ_j / n + Σ α_j β_j / n)."""
    sum_b = sum(betas)
    sum_ab = sum(a * b for a, b in zip(alphas, betas))
    return [b / sum_b * (1.0 - a / n * sum_b + sum_ab / n) for a, b in zip(alphas, betas)]


def theta_eq24(n: float, omegas: Sequence[float], deltas: Sequence[float]) -> List[float]:
    """Eq 11 / Eq 24:
    θ_i = 1/(Ω_i Σ_j 1/Ω_j) · (1 − Δ_i/n · Σ_j 1/Ω_j + 1/n · Σ_j Δ_j/Ω_j)."""
    inv_sum = sum(1.0 / o for o in omegas)                       # Alg 1 line 22 inv_sum
    delta_sum = sum(d / o for d, o in zip(deltas, omegas))       # Alg 1 line 22 delta_sum
    return [1.0 / (o * inv_sum) * (1.0 - d / n * inv_sum + delta_sum / n)
            for o, d in zip(omegas, deltas)]


def level_eq24(n: float, omegas: Sequence[float], deltas: Sequence[float]) -> float:
    """The common finish time implied by Eq 24 (every T_i = θ_i n Ω_i + Δ_i equal,
    Theorem 1):  T* = (n + Σ Δ_j/Ω_j) / Σ 1/Ω_j."""
    inv_sum = sum(1.0 / o for o in omegas)
    delta_sum = sum(d / o for d, o in zip(deltas, omegas))
    return (n + delta_sum) / inv_sum


# ----------------------------------------------------------------------------- §3.4

def bottleneck_case(p: Path, mode: int = PAPER) -> int:
    """Eq 13 case: case 1 iff β_i < β'_i, else case 2.

    B200 mode (C3) breaks the β = β' tie by the per-chunk latency terms:
    case 1 iff α_i > ε_i + α'_i."""
    if p.beta < p.beta2:
        return 1
    if mode == B200 and p.beta == p.beta2 and p.alpha > p.eps + p.alpha2:
        return 1
    return 2


def pipelined_time(x: float, k: int, p: Path, mode: int = PAPER) -> float:
    """Staged path carrying x = θ_i n bytes in k chunks.

    Per chunk m = x/k (Eq 12); stage 1 s1 = α + m/β, stage 2 s2 = ε + α' + m/β'.
    PAPER mode, Eq 13:  case 1: k·s1 + s2;  case 2: s1 + k·s2.
    B200 mode (C3): the exact two-stage pipeline, s1 + s2 + (k−1)·max(s1, s2); with a
    stage-2 availability time A = p.wake (C28: the relay kernel starts A after the
    message), max(s1 + s2 + (k−1)·max(s1, s2), A + k·s2)."""
    m = x / k
    s1 = p.alpha + m / p.beta
    s2 = p.eps + p.alpha2 + m / p.beta2
    if mode == B200:
        return max(s1 + s2 + (k - 1) * max(s1, s2), p.wake + k * s2)
    if bottleneck_case(p, PAPER) == 1:
        return k * (p.alpha + m / p.beta) + p.eps + p.alpha2 + m / p.beta2
    return p.alpha + m / p.beta + k * (p.eps + p.alpha2 + m / p.beta2)


def k_opt(x: float, p: Path, mode: int = PAPER) -> float:
    """Eq 14, case 1: k = sqrt(θn / (α β'));
    Eq 15, case 2: k = sqrt(θn / (β (ε + α')))."""
    if bottleneck_case(p, mode) == 1:
        return math.sqrt(x / (p.alpha * p.beta2))
    return math.sqrt(x / (p.beta * (p.eps + p.alpha2)))


def t_at_k_opt(x: float, p: Path, mode: int = PAPER) -> float:
    """Eq 17, case 1: 2 sqrt(θnα/β') + θn/β + ε + α';
    Eq 18, case 2: 2 sqrt(θn(ε+α')/β) + θn/β' + α."""
    if bottleneck_case(p, mode) == 1:
        return 2.0 * math.sqrt(x * p.alpha / p.beta2) + x / p.beta + p.eps + p.alpha2
    return 2.0 * math.sqrt(x * (p.eps + p.alpha2) / p.beta) + x / p.beta2 + p.alpha


def phi_two_pass(x0: float, p: Path, mode: int = PAPER) -> float:
    """Topology constant φ_i (Eq 19), reading C4: φ is computed from the
    first-pass (unpipelined) share x0 = θ⁽⁰⁾_i n so that Eq 19 reproduces Eq 14/15
    at θ⁽⁰⁾ (times the calibrated multiplier c_i):
      case 1: φ¹ = c·sqrt(α β' / x0);   case 2: φ² = c·sqrt((ε + α') β / x0)."""
    if bottleneck_case(p, mode) == 1:
        return p.c * math.sqrt(p.alpha * p.beta2 / x0)
    return p.c * math.sqrt((p.eps + p.alpha2) * p.beta / x0)


def k_eq19(x: float, phi: float, p: Path, mode: int = PAPER) -> float:
    """Eq 19: case 1: k = φ¹ θn/(α β');  case 2: k = φ² θn/((ε + α') β)."""
    if bottleneck_case(p, mode) == 1:
        return phi * x / (p.alpha * p.beta2)
    return phi * x / ((p.eps + p.alpha2) * p.beta)


def t_eq20(x: float, phi: float, p: Path, mode: int = PAPER) -> float:
    """Eq 20: case 1: θn(1/β + φ¹/β') + ε + α' + α/φ¹;
    case 2: θn(φ²/β + 1/β') + α + (ε + α')/φ²."""
    if bottleneck_case(p, mode) == 1:
        return x * (1.0 / p.beta + phi / p.beta2) + p.eps + p.alpha2 + p.alpha / phi
    return x * (phi / p.beta + 1.0 / p.beta2) + p.alpha + (p.eps + p.alpha2) / phi


def omega_delta_eq22(phi: float, p: Path, mode: int = PAPER):
    """Eq 22: case 1: Ω = 1/β + φ¹/β', Δ = ε + α' + α/φ¹;
    case 2: Ω = φ²/β + 1/β', Δ = α + (ε + α')/φ².  Direct: Ω = 1/β, Δ = α."""
    if p.kind == DIRECT:
        return 1.0 / p.beta, p.alpha
    if bottleneck_case(p, mode) == 1:
        return 1.0 / p.beta + phi / p.beta2, p.eps + p.alpha2 + p.alpha / phi
    return phi / p.beta + 1.0 / p.beta2, p.alpha + (p.eps + p.alpha2) / phi


def k_integer(k_real: float) -> int:
    """Reading C5: the smallest integer k >= 1 with k(k+1) >= k_real².

    For f(k) = A k + B/k (the Eq 13 case expressions as functions of k, with
    k_real = sqrt(B/A) from Eq 14/15), f(k) <= f(k+1) iff k(k+1) >= B/A, so this is
    the exact integer minimiser, ties going to the lower k.  A relative slack of
    1e-12 makes exact ties (k_real² = k(k+1), e.g. golden G5/G7) robust to the
    rounding of a square root that is squared again."""
    target = k_real * k_real * (1.0 - 1e-12)
    k = 1
    while k * (k + 1) < target:
        k += 1
    return k


# ----------------------------------------------------------------------------- O2

def issue_stagger(paths: Sequence[Path], active: Sequence[bool], mode: int, enabled: bool) -> List[float]:
    """Alg 1 line 17 / P:318: the issue latency of every earlier *active* path is
    accumulated into Δ_i.  PAPER: σ_j = α_j; B200: σ_j = calibrated p.sigma (C8)."""
    out = []
    acc = 0.0
    for p, a in zip(paths, active):
        out.append(acc if enabled else 0.0)
        if a:
            acc += p.alpha if mode == PAPER else p.sigma
    return out


def evaluate(n: int, nbytes: Sequence[int], chunks: Sequence[int], paths: Sequence[Path],
             opts: Options, port: Optional[Port] = None) -> float:
    """O2 (the mp_predict contract): predicted time of a config.

    Per path with b_i > 0: direct Eq 6; staged Eq 13 with k_i chunks
    (B200 mode: exact two-stage pipeline, C3); plus the issue stagger; then
    T = max_i T_i (Eq 4).  B200 mode adds the shared-port bound (C14)."""
    assert sum(nbytes) == n
    if n == 0:
        return 0.0
    active = [b > 0 for b in nbytes]
    stag = issue_stagger(paths, active, opts.mode, opts.stagger)
    t = 0.0
    for p, b, k, s, a in zip(paths, nbytes, chunks, stag, active):
        if not a:
            continue
        if p.kind == DIRECT:
            ti = p.alpha + b / p.beta
        else:
            ti = pipelined_time(float(b), int(k), p, opts.mode)
        t = max(t, ti + s)
    if opts.mode == B200 and port is not None and port.beta != INF:
        load = sum(p.w * b for p, b in zip(paths, nbytes))
        if load > 0:
            t = max(t, port.alpha + load / port.beta)
    return t


# ----------------------------------------------------------------------------- O3

def _solve_level_paper(n: float, omegas, deltas, paths, active, opts):
    """Eq 24 with the active-set rule C2: compute θ over the active set,
    drop every path with θ_i < 0, repeat (at most p rounds).  The stagger is
    recomputed over the current active set every round (C8)."""
    active = list(active)
    while True:
        stag = issue_stagger(paths, active, opts.mode, opts.stagger)
        idx = [i for i in range(len(paths)) if active[i]]
        om = [omegas[i] for i in idx]
        de = [deltas[i] + stag[i] for i in idx]
        th = theta_eq24(n, om, de)
        neg = [i for i, t in zip(idx, th) if t < 0]
        if not neg:
            theta = [0.0] * len(paths)
            for i, t in zip(idx, th):
                theta[i] = t
            return theta, level_eq24(n, om, de), active
        for i in neg:
            active[i] = False


def port_fill(T: float, omegas, deltas, paths, active, port: Port):
    """B200 mode (C14): the most bytes the active paths can deliver by time T.

    Each active path can carry at most u_i(T) = max(0, (T − Δ_i)/Ω_i) (the linear
    path time T_i = Ω_i x + Δ_i inverted); the shared port admits
    Σ w_i x_i <= max(0, T − α_port)·β_port.  This is a fractional knapsack: fill the
    paths in ascending w (ties: path order)."""
    order = sorted([i for i in range(len(paths)) if active[i]], key=lambda i: (paths[i].w, i))
    room = INF if port.beta == INF else max(0.0, T - port.alpha) * port.beta
    x = [0.0] * len(paths)
    for i in order:
        u = max(0.0, (T - deltas[i]) / omegas[i])
        if paths[i].w > 0 and room != INF:
            u = min(u, room / paths[i].w)
            room -= paths[i].w * u
        x[i] = u
    return x


def _solve_level_port(n: float, omegas, deltas, paths, active, opts, port: Port):
    """B200 mode level solve: the smallest T with port_fill(T) >= n, by bisection
    (200 halvings), inside the same active-set loop as C2 (drop paths that carry
    nothing, recompute the stagger, repeat)."""
    active = list(active)
    while True:
        stag = issue_stagger(paths, active, opts.mode, opts.stagger)
        de = [d + s for d, s in zip(deltas, stag)]

        def cap(T):
            return sum(port_fill(T, omegas, de, paths, active, port))

        lo, hi = 0.0, 1e-9
        while cap(hi) < n:
            hi *= 2.0
        for _ in range(200):
            mid = 0.5 * (lo + hi)
            if cap(mid) >= n:
                hi = mid
            else:
                lo = mid
        x = port_fill(hi, omegas, de, paths, active, port)
        new_active = [a and xi > 0 for a, xi in zip(active, x)]
        if new_active == active:
            return [xi / n for xi in x], hi, active
        active = new_active


def select(n: int, paths: Sequence[Path], opts: Options, port: Optional[Port] = None,
           path_mask: Optional[Sequence[bool]] = None,
           dshift: Optional[Sequence[float]] = None) -> Config:
    """O3 — canonical reading of Algorithm 1 `populate_path_config`.

    paths[0] is the direct path (A1 order: direct, GPU-staged by device, host).
      1. θ⁽⁰⁾: unpipelined Ω, Δ solved with Eq 11 + active set (C2)
         [B200 mode: the shared-port level solve, C14].
      2. φ_i from θ⁽⁰⁾ (Eq 19 two-pass reading, C4); Ω_i, Δ_i from Eq 22.
      3. θ from Eq 24 + active set (C2) [B200: port level solve].
      4. k_i from Eq 19 rounded by C5, clamped to [⌈b/slot⌉, min(K_max, ⌊b/C_min⌋)].
      5. shares: non-direct b_i = ⌊θ_i n / A⌋ A, dropped if < C_min; the direct path
         takes n − Σ (Alg 1 lines 24-28 "give leftover to direct", C7).
      6. [reading C18, B200 mode by default] pass 3: Eq 24 again with the affine
         integer-k coefficients of Eq 13 (``omega_delta_fixed_k``); new shares.
      7. t_pred = O2 of the config; t_level = the last level solve's finish time.

    dshift (NEXT f2, reading C24, oracle/window.py): every level solve uses
    max(0, Δ_i − dshift_i) in place of Δ_i (the per-message coefficients of a window)."""
    p = len(paths)
    assert paths[0].kind == DIRECT
    mask = list(path_mask) if path_mask is not None else [True] * p
    mask[0] = True                          # the direct path is never excluded
    if n == 0:
        return Config([0] * p, [0] * p, [0.0] * p, 0.0, 0.0)
    if port is None:
        port = Port()

    def level(om, de, act):
        if dshift is not None:
            de = [max(0.0, d - s) for d, s in zip(de, dshift)]
        if opts.mode == B200:
            return _solve_level_port(float(n), om, de, paths, act, opts, port)
        return _solve_level_paper(float(n), om, de, paths, act, opts)

    # Pass 1 — unpipelined (Alg 1 lines 15-16).
    od0 = [omega_delta_unpipelined(q) for q in paths]
    theta0, _, act0 = level([o for o, _ in od0], [d for _, d in od0], mask)

    # Pass 2 — pipelined linearisation (Alg 1 lines 18-19, Eq 19-22).
    omegas, deltas, phis = [], [], []
    act1 = list(act0)
    for i, q in enumerate(paths):
        if q.kind == DIRECT or not act0[i]:
            om, de = omega_delta_unpipelined(q)
            phis.append(0.0)
        else:
            phi = phi_two_pass(theta0[i] * n, q, opts.mode)
            om, de = omega_delta_eq22(phi, q, opts.mode)
            phis.append(phi)
        omegas.append(om)
        deltas.append(de)
    act1[0] = True
    theta, t_level, act2 = level(omegas, deltas, act1)

    # Shares (Alg 1 lines 23-28) and chunk counts (Alg 1 line 19, C5).
    nbytes = _shares(n, theta, act2, opts)
    chunks = [0] * p
    chunks[0] = 1
    for i in range(1, p):
        if nbytes[i]:
            k = k_integer(k_eq19(theta[i] * n, phis[i], paths[i], opts.mode))
            chunks[i] = _clamp_k(k, nbytes[i], opts)

    # Optional pass 3 (reading C18, default in B200 mode): with every k_i now an
    # integer, Eq 13 is affine in θ_i — case 1 Ω = 1/β + 1/(kβ'),
    # Δ = kα + ε + α'; case 2 Ω = 1/(kβ) + 1/β', Δ = α + k(ε + α') — so Eq 24 is
    # solved once more with those coefficients, equalising the integer-k finish times.
    refine = opts.refine if opts.refine is not None else (opts.mode == B200)
    if refine and opts.mode == B200:
        # Reading C26 (B200 mode): the exact pipeline T(x, k) = max(T1, T2) (C3)
        # picks its bottleneck stage per chunk size, so k_i is the exact integer
        # argmin of T at the path's share (``k_exact``) and the affine piece of Eq 13
        # used for Eq 24 is the one that is binding there (``piece_exact``); two
        # rounds of (k, piece, Eq 24, shares), then k once more for the final shares.
        for _round in range(2):
            om3, de3 = [], []
            for i, q in enumerate(paths):
                if q.kind == DIRECT or nbytes[i] == 0:
                    om, de = omega_delta_unpipelined(q) if q.kind == DIRECT else (1.0, 0.0)
                else:
                    chunks[i] = k_exact(float(nbytes[i]), q, nbytes[i], opts)
                    om, de = piece_exact(float(nbytes[i]), chunks[i], q)
                om3.append(om)
                de3.append(de)
            act3 = [i == 0 or nbytes[i] > 0 for i in range(p)]
            theta, t_level, act3 = level(om3, de3, act3)
            nbytes = _shares(n, theta, act3, opts)
        chunks = [1] + [k_exact(float(nbytes[i]), paths[i], nbytes[i], opts) if nbytes[i] else 0
                        for i in range(1, p)]
        cfg = Config(nbytes, chunks, [theta[i] if nbytes[i] > 0 or i == 0 else 0.0 for i in range(p)])
        cfg.t_pred = evaluate(n, nbytes, chunks, paths, opts, port)
        cfg.t_level = t_level
        cfg.theta_level = list(theta)
        # Reading C26, last step: the model's own prediction decides between this
        # split and the direct path alone (any path but the direct one may be
        # excluded), for plain messages (not a window's shifted coefficients).
        if dshift is None:
            direct = [n] + [0] * (p - 1)
            t_direct = evaluate(n, direct, [1] + [0] * (p - 1), paths, opts, port)
            if t_direct < cfg.t_pred:
                return Config(direct, [1] + [0] * (p - 1), [1.0] + [0.0] * (p - 1), t_direct, t_direct,
                              [1.0] + [0.0] * (p - 1))
        return cfg
    if refine:
        om3, de3 = [], []
        for i, q in enumerate(paths):
            om, de = omega_delta_fixed_k(q, max(1, chunks[i]), opts.mode)
            om3.append(om)
            de3.append(de)
        act3 = [i == 0 or nbytes[i] > 0 for i in range(p)]
        theta, t_level, act3 = level(om3, de3, act3)
        nbytes = _shares(n, theta, act3, opts)
        chunks = [1] + [_clamp_k(chunks[i], nbytes[i], opts) if nbytes[i] else 0
                        for i in range(1, p)]

    cfg = Config(nbytes, chunks, [theta[i] if nbytes[i] > 0 or i == 0 else 0.0 for i in range(p)])
    cfg.t_pred = evaluate(n, nbytes, chunks, paths, opts, port)
    cfg.t_level = t_level
    cfg.theta_level = list(theta)
    return cfg


def k_exact(x: float, p: Path, b: int, opts: Options) -> int:
    """Reading C26 (B200 mode): the integer k in C5's clamp range minimising the exact
    two-stage pipeline time of x bytes (C3).  With s1 = α + x/(kβ) and
    s2 = ε + α' + x/(kβ'), T(k) = s1 + s2 + (k−1)·max(s1, s2) = max(T1, T2) where
    T1 = k·s1 + s2 (Eq 13 case 1) and T2 = s1 + k·s2 (case 2), both convex in k, so
    T is convex and its real minimiser is the minimiser of T1 (Eq 14), of T2 (Eq 15)
    or the stage crossover s1 = s2; the integer argmin is the floor or ceiling of one
    of them (or a bound of the range).  Ties go to the smaller k (C5)."""
    lo = _clamp_k(1, b, opts)
    hi = max(lo, _clamp_k(10 ** 9, b, opts))
    e = p.eps + p.alpha2
    cands = {lo, hi}
    reals = [math.sqrt(x / (p.alpha * p.beta2)), math.sqrt(x / (p.beta * e))]
    if p.alpha != e:
        kc = x * (1.0 / p.beta2 - 1.0 / p.beta) / (p.alpha - e)
        if kc > 0:
            reals.append(kc)
    A = p.wake
    if A > 0:
        # C28: T3 = A + k·e + x/β' (increasing in k) joins the max; the new crossovers:
        # T3 = T2 at A − α = x/(kβ); T3 = T1 at (e − α)k² + (A − e + x/β' − x/β)k − x/β' = 0
        if A > p.alpha:
            reals.append(x / (p.beta * (A - p.alpha)))
        qa, qb, qc = e - p.alpha, A - e + x / p.beta2 - x / p.beta, -x / p.beta2
        if qa == 0.0:
            if qb != 0.0:
                reals.append(-qc / qb)
        else:
            disc = qb * qb - 4.0 * qa * qc
            if disc >= 0.0:
                for sgn in (1.0, -1.0):
                    reals.append((-qb + sgn * math.sqrt(disc)) / (2.0 * qa))
    for r in reals:
        if not (r > 0.0) or r > 1e12:
            continue
        for k in (math.floor(r), math.ceil(r)):
            cands.add(min(hi, max(lo, int(k))))
    best = None
    for k in sorted(cands):
        t = pipelined_time(x, k, p, B200)
        if best is None or t < best[0]:
            best = (t, k)
    return best[1]


def piece_exact(x: float, k: int, p: Path):
    """Reading C26: the affine piece (Ω, Δ) of the exact pipeline time at k chunks
    that binds at x bytes — case 1 (Ω = 1/β + 1/(kβ'), Δ = kα + ε + α') when
    T1 >= T2, else case 2 (Ω = 1/(kβ) + 1/β', Δ = α + k(ε + α')); C28: the
    availability piece (Ω = 1/β', Δ = A + k(ε + α')) when it is the largest."""
    m = x / k
    s1 = p.alpha + m / p.beta
    s2 = p.eps + p.alpha2 + m / p.beta2
    t12 = s1 + s2 + (k - 1) * max(s1, s2)
    if p.wake > 0 and p.wake + k * s2 > t12:
        return 1.0 / p.beta2, p.wake + k * (p.eps + p.alpha2)
    if s1 >= s2:
        return 1.0 / p.beta + 1.0 / (k * p.beta2), k * p.alpha + p.eps + p.alpha2
    return 1.0 / (k * p.beta) + 1.0 / p.beta2, p.alpha + k * (p.eps + p.alpha2)


def omega_delta_fixed_k(p: Path, k: int, mode: int = PAPER):
    """Eq 13 at a fixed integer k, written as T = Ω x + Δ (x = θ n):
    case 1: Ω = 1/β + 1/(kβ'), Δ = kα + ε + α';  case 2: Ω = 1/(kβ) + 1/β',
    Δ = α + k(ε + α').  Direct: Ω = 1/β, Δ = α."""
    if p.kind == DIRECT:
        return 1.0 / p.beta, p.alpha
    if bottleneck_case(p, mode) == 1:
        return 1.0 / p.beta + 1.0 / (k * p.beta2), k * p.alpha + p.eps + p.alpha2
    return 1.0 / (k * p.beta) + 1.0 / p.beta2, p.alpha + k * (p.eps + p.alpha2)


def _shares(n: int, theta, active, opts: Options) -> List[int]:
    """Alg 1 lines 23-28 (reading C7): non-direct b_i = ⌊θ_i n / A⌋·A, dropped below
    C_min; the direct path takes the leftover n − Σ b_i."""
    p = len(theta)
    nbytes = [0] * p
    for i in range(1, p):
        if active[i] and theta[i] > 0:
            b = int(math.floor(theta[i] * n / opts.align)) * opts.align
            nbytes[i] = b if b >= opts.c_min else 0
    nbytes[0] = n - sum(nbytes[1:])
    return nbytes


def _clamp_k(k: int, b: int, opts: Options) -> int:
    """Reading C5: clamp k to [⌈b / slot_bytes⌉, min(K_max, ⌊b / C_min⌋)] (the slot
    bound wins), k >= 1."""
    k = min(k, min(opts.k_max, max(1, b // opts.c_min)))
    if opts.slot_bytes > 0:
        k = max(k, -(-b // opts.slot_bytes))
    return max(1, k)


def masked(paths: Sequence[Path], mask: Sequence[bool]) -> List[Path]:
    """Helper for tests: the sub-list of paths selected by a mask (direct kept)."""
    return [q for i, q in enumerate(paths) if i == 0 or mask[i]]


def with_defaults(p: Path, **kw) -> Path:
    return replace(p, **kw)
