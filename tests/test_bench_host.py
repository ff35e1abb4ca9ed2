"""Host logic of bench.py that needs no GPU: the compact exhaustive sweep behind the
bench line's `e_sel` (the metric's "model-vs-sweep optimum error %")."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402

MiB = 1 << 20


def test_esel_grid_covers_the_path_kinds_and_splits_exactly():
    n, npaths = 1 << 30, 8          # config 3: direct + 6 relays + host
    g = bench.esel_grid(n, npaths, npaths - 1)
    assert len(g) == len({(tuple(b), tuple(c)) for b, c in g}) >= 20
    assert ([n] + [0] * 7, [1] + [0] * 7) in g                       # direct alone
    for nb, ch in g:
        assert sum(nb) == n and nb[0] > 0 and ch[0] == 1              # Eq 3: shares sum to n
        for i in range(1, npaths):
            assert (nb[i] == 0) == (ch[i] == 0)                       # unused paths have k = 0
            if nb[i]:
                assert nb[i] % 256 == 0 and nb[i] // ch[i] <= 30 * MiB  # A-aligned, chunks fit a slot
    kinds = {tuple(i for i in range(1, npaths) if nb[i]) for nb, _ in g}
    assert (7,) in kinds and (1,) in kinds and tuple(range(1, 7)) in kinds and tuple(range(1, 8)) in kinds
