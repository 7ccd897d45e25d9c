"""Pins for the oracle's random-number primitives (R4, R6, R23).

Philox4x32-10 is pinned by the published Random123 known-answer vectors
(Salmon et al., SC'11, kat_vectors); uniform_below and the A-Res key by closed
forms and distribution properties -- not by re-typing their formulas.
"""
import math
from collections import Counter

import numpy as np
import pytest

from tests._stats import chi_square_p

# Random123 kat_vectors, philox4x32 R=10: (ctr, key, expected output)
KAT = [
    ([0, 0, 0, 0], [0, 0], [0x6627E8D5, 0xE169C58D, 0xBC57AC4C, 0x9B00DBD8]),
    ([0xFFFFFFFF] * 4, [0xFFFFFFFF] * 2, [0x408F276D, 0x41C83B0E, 0xA20BC7C6, 0x6D5451FD]),
    ([0x243F6A88, 0x85A308D3, 0x13198A2E, 0x03707344], [0xA4093822, 0x299F31D0],
     [0xD16CFE09, 0x94FDCCEB, 0x5001E420, 0x24126EA1]),
]


@pytest.mark.parametrize("ctr,key,want", KAT)
def test_philox_kat(oracle_lib, ctr, key, want):
    assert oracle_lib.philox4x32_10(ctr, key) == want


def test_uniform_below_edges(oracle_lib):
    ub = oracle_lib.uniform_below
    M = 0xFFFFFFFF
    for n in [1, 2, 3, 7, 1000, 2**31, 2**40 + 3]:
        assert ub(n, 0, 0) == 0                      # r = 0 -> 0
        assert ub(n, M, M) == n - 1                  # r = 2^64-1 -> n-1
    assert ub(1, 0x12345678, 0x9ABCDEF0) == 0        # n = 1 -> always 0
    # n = 2^j: the draw is the top j bits of r = r1:r0 (closed form)
    r0, r1 = 0xDEADBEEF, 0xC0FFEE11
    r = (r1 << 32) | r0
    for j in [1, 5, 17, 32, 40]:
        assert ub(2**j, r0, r1) == r >> (64 - j)
    # r = 2^63 (one half) -> floor(n / 2)
    for n in [3, 7, 10, 999]:
        assert ub(n, 0, 0x80000000) == n // 2


def test_uniform_below_monotone_and_uniform(oracle_lib):
    ub = oracle_lib.uniform_below
    rng = np.random.default_rng(1)
    words = rng.integers(0, 2**32, size=(60000, 2), dtype=np.uint64)
    for n in [3, 7, 1000]:
        vals = [ub(n, int(a), int(b)) for a, b in words]
        assert min(vals) >= 0 and max(vals) < n
        c = Counter(vals)
        assert chi_square_p(c, {i: 1.0 / n for i in range(n)}, len(vals)) > 1e-3
    # monotone non-decreasing in r
    prev = -1
    for hi in range(0, 2**32, 2**28):
        v = ub(1000, 0, hi)
        assert v >= prev
        prev = v


def test_ares_key_closed_forms(oracle_lib):
    key = oracle_lib.ares_key
    # E = -ln((r + 0.5) 2^-32) is Exp(1) over a uniform r: mean 1, P(E > 1) = e^-1.
    M = 1 << 16
    rs = [int((i + 0.5) * (2**32 / M)) for i in range(M)]
    es = np.array([key(r, 1.0) for r in rs])
    assert abs(es.mean() - 1.0) < 2e-3
    assert abs((es > 1.0).mean() - math.exp(-1)) < 1e-3
    # strictly decreasing in r, scales exactly as 1/bias
    assert np.all(np.diff(es) < 0)
    for r in [0, 1, 2**31, 2**32 - 1]:
        assert key(r, 4.0) == key(r, 1.0) / 4.0
    # r = 2^32 - 1: u = 1 - 2^-33 exactly, E = -ln(1-x) ~= x (x = 2^-33)
    assert key(2**32 - 1, 1.0) == pytest.approx(2.0**-33, rel=1e-9)
    # r = 0: u = 2^-33, E = 33 ln 2
    assert key(0, 1.0) == pytest.approx(33 * math.log(2.0), rel=1e-15)
