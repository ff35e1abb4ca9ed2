"""Pins of the reference transfer (O1): the replay through any split reproduces the
plain definition dst[0:n] == src[0:n], covers every byte once and leaves the canaries."""
import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

import synth
from oracle import transfer as X

CANARY = 4096


@settings(max_examples=100, deadline=None)
@given(st.integers(0, 300_000), st.lists(st.integers(0, 5), min_size=1, max_size=7),
       st.sampled_from([1, 16, 256]), st.integers(0, 99))
def test_replay_equals_definition(n, weights, align, seed):
    kinds = [0] + [1] * (len(weights) - 1)
    tot = sum(weights) or 1
    nbytes = [n * w // tot // align * align for w in weights]
    nbytes[0] += n - sum(nbytes)
    chunks = [1] + [max(1, min(1 + (seed + i) % 7, max(1, b // align))) if b else 0
                    for i, b in enumerate(nbytes[1:])]
    src = synth.payload(n + 64, seed % 20)
    dst = np.full(n + 2 * CANARY, 0xA5, dtype=np.uint8)
    X.replay(src, nbytes, chunks, kinds, align, dst[CANARY:CANARY + n])
    assert np.array_equal(dst[CANARY:CANARY + n], X.reference_transfer(src, n))
    assert (dst[:CANARY] == 0xA5).all() and (dst[CANARY + n:] == 0xA5).all()


def test_chunk_ranges_balanced():
    r = X.chunk_ranges(1000, 10 * 256 + 17, 4, 256)
    assert [ln for _, ln in r] == [512, 768, 512, 768 + 17]
    assert r[0][0] == 1000 and sum(ln for _, ln in r) == 10 * 256 + 17
    with pytest.raises(AssertionError):
        X.chunk_ranges(0, 3 * 256, 4, 256)


def test_debug_payload_locates_words():
    p = synth.debug_payload(64, seed=5)
    w = p.view(np.uint64)
    assert list(w) == [i ^ 5 for i in range(8)]
