"""Seeded synthetic inputs shared by the oracle-side tests and the CUDA-side tests.

Holds none of the method's arithmetic: only random-number recipes.

* ``payload(n, size_index, src_rank)`` — uniformly random bytes, seed
  20251116 + 8·size_index + src_rank.  numpy PCG64.
* ``topology(seed, n_relays, host)`` — a random but physically plausible parameter
  table (α, β, α', β', ε, c, σ, w) for one (src, dst) pair, as plain dicts.
"""
from __future__ import annotations

import numpy as np

BASE_SEED = 20251116

# Path kinds (mirrors the C ABI enum and the paper's taxonomy P:107-111).
DIRECT, GPU_STAGED, HOST_STAGED = 0, 1, 2


def payload_seed(size_index: int, src_rank: int = 0) -> int:
    return BASE_SEED + 8 * size_index + src_rank


def payload(n: int, size_index: int = 0, src_rank: int = 0) -> np.ndarray:
    """n uniformly random bytes (uint8)."""
    rng = np.random.Generator(np.random.PCG64(payload_seed(size_index, src_rank)))
    return rng.integers(0, 256, size=n, dtype=np.uint8)


def debug_payload(n: int, seed: int = BASE_SEED) -> np.ndarray:
    """Each little-endian 8-byte word = (word offset) XOR seed, so a misplaced chunk
    can be located by reading the bytes it landed on."""
    words = (np.arange((n + 7) // 8, dtype=np.uint64) ^ np.uint64(seed))
    return words.view(np.uint8)[:n].copy()


def topology(seed: int, n_relays: int = 2, host: bool = True, us=1e-6, gbs=1e9):
    """A random parameter table: direct + n_relays GPU-staged + optional host-staged.

    Ranges are B200-like (NVLink 5 / PCIe Gen5; not from the paper):
    α ∈ [1, 8] µs, NVLink β ∈ [300, 800] GB/s, PCIe β ∈ [20, 60] GB/s,
    ε ∈ [0.5, 5] µs; c = 1; σ ∈ [0, 2] µs; port weight 1 on NVLink paths."""
    rng = np.random.Generator(np.random.PCG64(seed))
    u = lambda lo, hi: float(rng.uniform(lo, hi))
    paths = [dict(kind=DIRECT, alpha=u(1, 8) * us, beta=u(300, 800) * gbs, alpha2=0.0,
                  beta2=float("inf"), eps=0.0, c=1.0, sigma=u(0, 2) * us, w=1.0, via=-1)]
    for r in range(n_relays):
        paths.append(dict(kind=GPU_STAGED, alpha=u(1, 8) * us, beta=u(300, 800) * gbs,
                          alpha2=u(1, 8) * us, beta2=u(300, 800) * gbs, eps=u(0.5, 5) * us,
                          c=1.0, sigma=u(0, 2) * us, w=1.0, via=2 + r))
    if host:
        paths.append(dict(kind=HOST_STAGED, alpha=u(2, 10) * us, beta=u(20, 60) * gbs,
                          alpha2=u(2, 10) * us, beta2=u(20, 60) * gbs, eps=u(1, 8) * us,
                          c=1.0, sigma=u(0, 2) * us, w=0.0, via=-1))
    return paths
