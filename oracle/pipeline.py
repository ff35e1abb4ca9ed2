"""ORACLE (test infrastructure only; see oracle/__init__.py).  Pipeline simulation.

Discrete-event simulation of the staged transfer of PAPER.md §3.4:
every chunk goes (1) source → staging, (2) a synchronisation point, (3) staging →
destination.  Stage 1 is serial on the first link, stage 2 serial on the second;
chunk c may start stage 2 only after its own stage 1 is done.  With a
finite ring of S staging slots, chunk c may only start stage 1 once chunk c − S has
left its slot.

Used to pin Eq 13: with unlimited slots the finish time is
s1 + s2 + (k−1)·max(s1, s2), which equals Eq 13's case expression whenever the
case names the true bottleneck stage.
"""
from __future__ import annotations

import math


def simulate_two_stage(k: int, s1: float, s2: float, slots: int = 0, start2: float = 0.0) -> float:
    """Finish time of k chunks through a two-stage pipeline with per-chunk stage
    times s1 (first link incl. its α) and s2 (ε + α' + second link).  slots = 0
    means unlimited staging buffers.  start2: the second stage is not available before
    this time (reading C28: the relay kernel's start)."""
    f1 = [0.0] * k      # stage-1 finish of each chunk
    f2 = [0.0] * k      # stage-2 finish of each chunk
    link1_free = 0.0
    link2_free = start2
    for c in range(k):
        start1 = link1_free
        if slots and c >= slots:
            start1 = max(start1, f2[c - slots])      # wait for the slot to drain
        f1[c] = start1 + s1
        link1_free = f1[c]
        start2 = max(link2_free, f1[c])              # sync point: chunk has landed
        f2[c] = start2 + s2
        link2_free = f2[c]
    return f2[-1] if k else 0.0


def stage_times(x: float, k: int, alpha: float, beta: float, eps: float, alpha2: float,
                beta2: float):
    """Per-chunk stage times of Eq 12, m = x/k."""
    m = x / k
    return alpha + m / beta, eps + alpha2 + (m / beta2 if beta2 != math.inf else 0.0)


def simulate_window(w: int, a: float, b: float, h_sub: float = 0.0) -> float:
    """Finish time of w messages through a two-stage pipeline (reading C24: an issue
    phase a that may overlap the previous message, then a serve phase b), message j
    released by the host at (j − 1)·h_sub (reading C27)."""
    f1 = f2 = 0.0
    for j in range(w):
        f1 = max(f1, j * h_sub) + a       # issue: after the previous issue and the release
        f2 = max(f2, f1) + b              # serve: after its issue and the previous serve
    return f2
