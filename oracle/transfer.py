"""ORACLE (test infrastructure only; see oracle/__init__.py).  Reference transfer (O1).

The method moves bytes; its result has a plain definition: after the transfer,
dst[0:n] == src[0:n] byte for byte and nothing outside [0, n) of dst is touched.
This module replays that definition *through the chosen split* (SURVEY §8c O1):
every path takes a contiguous byte range in path order (direct first, reading C6),
every staged range is cut into k chunks, and each chunk is copied
source → staging buffer → destination.  The chunks are asserted to cover
[0, n) exactly once.
"""
from __future__ import annotations

from typing import List, Sequence, Tuple

import numpy as np

DIRECT = 0


def path_ranges(nbytes: Sequence[int]) -> List[Tuple[int, int]]:
    """Reading C6: path i owns [Σ_{j<i} b_j, Σ_{j<=i} b_j) (path order, direct first)."""
    out, off = [], 0
    for b in nbytes:
        out.append((off, b))
        off += b
    return out


def chunk_ranges(off: int, b: int, k: int, align: int) -> List[Tuple[int, int]]:
    """Reading C6: a staged share of b bytes in k chunks.  With U = b // A units of A
    bytes (and rem = b − U·A), chunk j covers units [⌊jU/k⌋, ⌊(j+1)U/k⌋); the last
    chunk also takes the rem tail bytes.  Valid when 1 <= k <= max(1, U)."""
    if b == 0:
        return []
    U, rem = divmod(b, align)
    assert 1 <= k <= max(1, U), (b, k, align)
    out = []
    for j in range(k):
        s = align * (j * U // k)
        e = align * ((j + 1) * U // k)
        if j == k - 1:
            e += rem
        out.append((off + s, e - s))
    return out


def layout(nbytes: Sequence[int], chunks: Sequence[int], kinds: Sequence[int], align: int):
    """Every (path, chunk, offset, length) the transfer performs, in path order."""
    out = []
    for i, (off, b) in enumerate(path_ranges(nbytes)):
        if b == 0:
            continue
        if kinds[i] == DIRECT:
            out.append((i, 0, off, b))
        else:
            for j, (o, ln) in enumerate(chunk_ranges(off, b, chunks[i], align)):
                out.append((i, j, o, ln))
    return out


def replay(src: np.ndarray, nbytes: Sequence[int], chunks: Sequence[int], kinds: Sequence[int],
           align: int, dst: np.ndarray) -> np.ndarray:
    """Copy src[0:n] into dst[0:n] through the split: direct chunks straight, staged
    chunks via a staging buffer.  Asserts exact single coverage."""
    n = int(sum(nbytes))
    assert src.dtype == np.uint8 and dst.dtype == np.uint8 and len(src) >= n and len(dst) >= n
    covered = np.zeros(n, dtype=np.int32)
    for i, _j, off, ln in layout(nbytes, chunks, kinds, align):
        if kinds[i] == DIRECT:
            dst[off:off + ln] = src[off:off + ln]
        else:
            stage = src[off:off + ln].copy()          # step (1): source → staging
            dst[off:off + ln] = stage                 # step (3): staging → destination
        covered[off:off + ln] += 1
    assert n == 0 or (covered.min() == 1 and covered.max() == 1), "chunks must cover [0,n) once"
    return dst


def reference_transfer(src: np.ndarray, n: int) -> np.ndarray:
    """The plain definition (O1): the first n bytes of src."""
    return src[:n].copy()
