"""ORACLE (test infrastructure only; see oracle/__init__.py).  NEXT f4: size bands.

PAPER.md §5.2 Observation 4: "The model-driven predictions are less accurate
for smaller message sizes ... due to the linear nature of the Hockney's model and the
way the asymptotic bandwidth is calculated"; "piecewise α/β".
Reading C20: every pair carries one or more *size bands*; band j holds
a complete parameter set (every path's α, β, α', β', ε, c, σ, w and the shared port)
and applies to messages of n bytes with n_min_j <= n < n_min_{j+1} (n_min_0 = 0).  A
message is modelled and selected (Eq 1-24, Alg 1) entirely with its band's parameters
— the paper's model unchanged, only its inputs depend on n.

Band fit (Step 1, reading C12 per band): band j is fitted (oracle.calibration
.fit_hockney) on the measured sizes s with e_j <= s <= e_{j+1} (both edges inclusive,
e_0 = 0, e_{B} = ∞); a band with fewer than two such sizes takes the fit of the
nearest band above it that has two, else of the nearest below.
"""
from __future__ import annotations

from typing import List, Sequence, Tuple

from . import calibration as OC
from . import model as M


def band_index(edges: Sequence[int], n: int) -> int:
    """Index j of the band holding n: the last j with edges[j] <= n (edges[0] == 0,
    strictly increasing)."""
    j = 0
    for i, e in enumerate(edges):
        if e <= n:
            j = i
    return j


def select_banded(n: int, bands: Sequence[Tuple[int, Sequence[M.Path], M.Port]], opts: M.Options,
                  mask=None) -> M.Config:
    """Alg 1 with the parameters of n's band.  bands: [(n_min, paths, port)], n_min
    ascending, the first 0."""
    j = band_index([b[0] for b in bands], n)
    _, paths, port = bands[j]
    if mask is not None:
        paths = [p for p, m in zip(paths, mask) if m]
    return M.select(n, list(paths), opts, port)


def fit_bands(n: Sequence[float], t: Sequence[float], edges: Sequence[float]) -> List[Tuple[float, float]]:
    """Per-band (α, β) by the C12 fit over the sizes inside each band (edges
    inclusive); bands without two sizes borrow as stated in the module docstring."""
    B = len(edges)
    fits: List = [None] * B
    for j in range(B):
        lo = edges[j]
        hi = edges[j + 1] if j + 1 < B else float("inf")
        pts = [(x, y) for x, y in zip(n, t) if lo <= x <= hi]
        if len(pts) >= 2:
            fits[j] = OC.fit_hockney([p[0] for p in pts], [p[1] for p in pts])
    own = list(fits)                      # bands fitted on their own sizes
    for j in range(B):
        if own[j] is None:
            above = [own[i] for i in range(j + 1, B) if own[i] is not None]
            below = [own[i] for i in range(j - 1, -1, -1) if own[i] is not None]
            if not above and not below:
                raise ValueError("no band has two sizes")
            fits[j] = above[0] if above else below[0]
    return fits
