"""ORACLE (test infrastructure only; see oracle/__init__.py).  Step-1 fit.

PAPER.md §4 Step 1: "the performance model parameters are extracted once per
system topology" — how is not given; reading C12: per link, a least
squares fit of the Hockney line T(n) = α + n/β (Eq 1) over the measured sizes,
each residual weighted by 1/T² (relative error), subject to α >= 1e-7 s (Eq 14 needs
α > 0: when the free optimum violates it, α = 1e-7 and the slope is refitted for that α
— the constrained optimum of the convex objective), a non-positive slope replaced by
the last sample's n/t.

The fit is solved with numpy's least-squares routine (a library primitive) on the
row-scaled system; tests/test_oracle_calibration.py pins it to exact rational normal
equations and to noiseless recovery.
"""
from __future__ import annotations

from typing import Sequence, Tuple

import numpy as np


def fit_hockney(n: Sequence[float], t: Sequence[float]) -> Tuple[float, float]:
    """Weighted least squares of t ≈ α + n·g with weights 1/t² (minimise
    Σ ((t_i − α − n_i g) / t_i)²); returns (α, β = 1/g) with the C12 clamps."""
    n = np.asarray(n, dtype=np.float64)
    t = np.asarray(t, dtype=np.float64)
    A = np.stack([np.ones_like(n), n], axis=1) / t[:, None]   # rows scaled by 1/t_i
    b = t / t                                                  # t_i / t_i
    (alpha, g), *_ = np.linalg.lstsq(A, b, rcond=None)
    if not alpha > 1e-7:
        # the clamp is a constraint of the fit (α >= 1e-7): the objective is a convex
        # quadratic, so when the free optimum has α below the bound the constrained
        # optimum lies on it — α = 1e-7 and the best slope for that α (1-column lstsq)
        alpha = 1e-7
        (g,), *_ = np.linalg.lstsq(n[:, None] / t[:, None], (t - alpha) / t, rcond=None)
    if not g > 0:
        g = t[-1] / n[-1]
    return float(alpha), float(1.0 / g)
