"""ORACLE (test infrastructure only; see oracle/__init__.py).  NEXT f2: windows and BIBW.

SURVEY §8(f) f2 / PAPER.md Observation 2 ("larger window sizes allow for more
concurrent transfers, reducing the impact of latency") and Observation 5 (P:379-385:
"contention between the bidirectional transfers along the host-staged path … the
model should be extended to account for host-staged contention, PCIe
configuration").  The paper's model is per message (reading C15); these are the
readings C24 (window) and C25 (bidirectional host contention) of DESIGN.md §3.

C24 — a window of w back-to-back messages of n bytes with one config
--------------------------------------------------------------------
Every message on path i is split into an *issue* phase of length a_i (the part of its
startup α_i that may overlap the previous message on that path, a_i = min(h_i, α_i),
h_i >= 0 a calibrated per-path parameter) and a *serve* phase of length T_i − a_i
(T_i = the O2 path time of one message, Eq 6 / Eq 13, with the stagger).  Issue j+1
may run while message j serves; serve j+1 starts after issue j+1 and serve j.  That
is a two-stage pipeline over the w messages (the same shape as P:224-228), so

    T_i^w = a_i + (T_i − a_i) + (w − 1)·max(a_i, T_i − a_i)
          = T_i + (w − 1)·max(a_i, T_i − a_i).

The shared port (B200 mode, C14) is one more such pipeline: T_port = α_S +
Σ_i w_i b_i / β_S per message, overlappable part a_S = min(α_S, min a_i over the
active paths with w_i > 0).  A window also pays a fixed completion cost τ
(OMB's wait-all + ack; a calibrated pair parameter, 0 by default):

    T^w = τ + max(max_i T_i^w, T_port^w).                              (W1)

w = 1 gives O2 (+ τ); h = 0 gives w·T (+ τ), the paper's per-message model.

C27 — host submission (NEXT f4's small-message regime): the messages of a
window are enqueued by the host one call at a time, h_sub seconds apart (the caller's
cost per mp_send / mp_xfer call, calibrated), so message j cannot start before
(j − 1)·h_sub.  For the two-stage pipeline with those release times the finish of the
last message is (a flow-shop argument on the release-time grid; pinned against the
event simulation of oracle/pipeline.py)

    T_i^w = T_i + (w − 1)·max(a_i, T_i − a_i, h_sub),

the same for the port; h_sub = 0 is C24.  Small messages, whose GPU time is below the
host's cost per call, are submission-bound: T^w ≈ τ + T_1 + (w − 1)·h_sub.

Selection for a window (``select_window``): while serve >= issue on every path,
T_i^w / w = T_i − (1 − 1/w)·a_i, i.e. each path's per-message Δ_i drops by
(1 − 1/w)·a_i and the port's α_S by (1 − 1/w)·a_S (a_S over the paths the mask
allows) — so Alg 1 (O3) runs unchanged on those shifted coefficients in every pass (``M.select(..., dshift=, port=)``);
t_pred is (W1) of the selected config.

C25 — bidirectional host contention for known concurrent flows
--------------------------------------------------------------
A GPU's PCIe link is full duplex nominally, but when its up and down directions both
carry host legs the measured rate of each falls (SM copies on B200: 52.5 GB/s one way,
39.1 GB/s each way in duplex, profiles/r01/diag_host2.jsonl).  On top of the fair
share of C19: for a flow s → d with s != d, its host up leg at s is scaled by κ_s if
any flow's host *down* leg enters s, and its down leg at d by κ_d if any flow's host
up leg leaves d (κ_g in (0, 1], calibrated, 1 by default).  A loopback flow (s = d)
is calibrated with both of its legs running at once (duplex already) and is not
scaled.
"""
from __future__ import annotations

from dataclasses import replace
from typing import Optional, Sequence

from . import flows as F
from . import model as M


def issue_part(p: M.Path, h: float) -> float:
    """C24: the overlappable issue phase a_i = min(h_i, α_i)."""
    return min(max(h, 0.0), p.alpha)


def port_issue_part(port: M.Port, paths, h, active) -> float:
    """C24: the port's overlappable startup, a_S = min(α_S, min a_i over the active
    paths that load it) — the port overlaps no more than the paths through it."""
    a = [issue_part(p, hi) for p, hi, act in zip(paths, h, active) if act and p.w > 0]
    return min([port.alpha] + a) if a else 0.0


def path_window_time(t1: float, a: float, w: int, h_sub: float = 0.0) -> float:
    """C24: two-stage pipeline (issue a, serve t1 − a) over w messages:
    T^w = t1 + (w − 1)·max(a, t1 − a); C27: messages released h_sub apart,
    T^w = t1 + (w − 1)·max(a, t1 − a, h_sub)."""
    return t1 + (w - 1) * max(a, t1 - a, h_sub)


def evaluate_window(n: int, w: int, nbytes, chunks, paths: Sequence[M.Path], h: Sequence[float],
                    opts: M.Options, port: Optional[M.Port] = None, tau: float = 0.0,
                    h_sub: float = 0.0) -> float:
    """(W1): time of w back-to-back messages of n bytes with the config (nbytes, chunks);
    h_sub = the host's submission time per message (C27); a relay's start A (C28) delays
    the window once."""
    assert w >= 1 and sum(nbytes) == n
    if n == 0:
        return 0.0
    active = [b > 0 for b in nbytes]
    stag = M.issue_stagger(paths, active, opts.mode, opts.stagger)
    t = 0.0
    for p, b, k, s, a, hi in zip(paths, nbytes, chunks, stag, active, h):
        if not a:
            continue
        if p.kind == M.DIRECT:
            ti = p.alpha + b / p.beta                          # Eq 6
            t = max(t, path_window_time(ti + s, issue_part(p, hi), w, h_sub))
        elif opts.mode == M.B200 and p.wake > 0:
            # C28: the relay starts A late once and then lingers through the window:
            # the wake-free message's window plus the first message's delay
            t0 = M.pipelined_time(float(b), int(k), replace(p, wake=0.0), opts.mode)
            t1 = M.pipelined_time(float(b), int(k), p, opts.mode)
            t = max(t, path_window_time(t0 + s, issue_part(p, hi), w, h_sub) + (t1 - t0))
        else:
            ti = M.pipelined_time(float(b), int(k), p, opts.mode)  # Eq 13
            t = max(t, path_window_time(ti + s, issue_part(p, hi), w, h_sub))
    if opts.mode == M.B200 and port is not None and port.beta != M.INF:
        load = sum(p.w * b for p, b in zip(paths, nbytes))
        if load > 0:
            a_s = port_issue_part(port, paths, h, active)
            t = max(t, path_window_time(port.alpha + load / port.beta, a_s, w, h_sub))
    return tau + t


def select_window(n: int, w: int, paths: Sequence[M.Path], h: Sequence[float], opts: M.Options,
                  port: Optional[M.Port] = None, path_mask=None, tau: float = 0.0,
                  h_sub: float = 0.0) -> M.Config:
    """C24 selection: O3 on the per-message coefficients of a window (Δ_i − (1 − 1/w)·a_i,
    port α_S − (1 − 1/w)·a_S over the mask's paths); t_pred = (W1) of the result (with
    C27's h_sub), t_level = w·(per-message level) + τ.  (A submission-bound window's
    time does not depend on the split; the split is chosen for the serve-bound case.)"""
    assert w >= 1
    shift = [(1.0 - 1.0 / w) * issue_part(p, hi) for p, hi in zip(paths, h)]
    wport = None
    if port is not None:
        allowed = [True] * len(paths) if path_mask is None else [i == 0 or bool(m) for i, m in enumerate(path_mask)]
        a_s = port_issue_part(port, paths, h, allowed)
        wport = M.Port(alpha=port.alpha - (1.0 - 1.0 / w) * a_s, beta=port.beta)
    # C28: one relay start per window, spread over its w messages in the selection
    wpaths = [replace(p, wake=p.wake / w) for p in paths]
    cfg = M.select(n, wpaths, opts, wport, path_mask, dshift=shift)
    if n == 0:
        return cfg
    cfg.t_pred = evaluate_window(n, w, cfg.bytes, cfg.chunks, paths, h, opts, port, tau, h_sub)
    cfg.t_level = w * cfg.t_level + tau
    return cfg


# ----------------------------------------------------------------------------- C25

def duplex_flags(flows, paths_of):
    """Per flow: (scale the up leg at src?, scale the down leg at dst?) under C25."""
    up_users, down_users = {}, {}
    for f, (s, d, _, mask) in enumerate(flows):
        for i, p in enumerate(paths_of(f)):
            if mask[i] and p.kind == M.HOST_STAGED:
                up_users[s] = up_users.get(s, 0) + 1
                down_users[d] = down_users.get(d, 0) + 1
    out = []
    for s, d, _, _ in flows:
        if s == d:
            out.append((False, False))
        else:
            out.append((down_users.get(s, 0) > 0, up_users.get(d, 0) > 0))
    return out


def select_flows_duplex(flows, pair_paths, pair_port, opts: M.Options, kappa, window: int = 1,
                        window_of=None) -> list:
    """C19 fair share, then C25's duplex factor κ_g on the host legs, then O3 per flow.
    kappa(g) -> κ_g.  window > 1 (C24): every flow sends a window of that many messages,
    so each is selected with select_window and its pair's window model,
    window_of(s, d) -> (h, τ)."""
    facs = F.share_factors(flows, lambda f: pair_paths(flows[f][0], flows[f][1]))
    dup = duplex_flags(flows, lambda f: pair_paths(flows[f][0], flows[f][1]))
    out = []
    for (s, d, n, mask), fac, (up, down) in zip(flows, facs, dup):
        paths, port, m = F.shared_model(pair_paths(s, d), pair_port(s, d), fac, mask)
        paths = [replace(p, beta=p.beta * (kappa(s) if up else 1.0),
                         beta2=p.beta2 * (kappa(d) if down else 1.0)) if p.kind == M.HOST_STAGED else p
                 for p in paths]
        if window > 1 and window_of is not None:
            h, tau = window_of(s, d)
            out.append(select_window(n, window, paths, h, opts, port, m, tau))
        else:
            out.append(M.select(n, paths, opts, port, m))
    return out


# ----------------------------------------------------------------------------- C24 fit

def fit_window(samples, window: int, npaths: int, h_sub: float = 0.0):
    """The C24 estimator of Step 1 (mp_calibrate_window): samples = [(path, T1, TW, pred)]
    with T1 one message on an idle stream, TW `window` back-to-back messages, pred the
    model's one-message time.  τ = max(0, median(T1 − pred) over the direct path's
    samples); h_i = median over path i's samples of max(0, T1 − τ − (TW − T1)/(W − 1))
    (the serve-bound branch of W1: TW − T1 = (W − 1)·(T_i − a_i)).  C27: a sample whose
    steady per-message time (TW − T1)/(W − 1) does not exceed the host's submission time
    h_sub·(1 + 1e-6) is submission-bound and says nothing about a_i — it is skipped.
    Medians of an even count take the upper middle value."""
    from statistics import median_high
    d = [t1 - pred for p, t1, _, pred in samples if p == 0]
    tau = max(0.0, median_high(d)) if d else 0.0
    h = []
    for i in range(npaths):
        a = [max(0.0, t1 - tau - (tw - t1) / (window - 1)) for p, t1, tw, _ in samples
             if p == i and (tw - t1) / (window - 1) > h_sub * (1 + 1e-6)]
        h.append(median_high(a) if a else 0.0)
    return h, tau
