"""Pins for the oracle's random draws (SURVEY 8(c) "Pins": Philox, uniform mapping).

The paper generates the initial swarm and the per-iteration random weight
matrices L, G with Thrust (Sec 3.1; Eq. 1: components ~ U(0,1)).
Reading 6 fixes Philox4x32-10 keyed on (seed, t, i, j); reading 5 fixes the
24-bit uniform mapping.  Pins: published KAT vectors, exact mapping edge
cases, and distribution tests.
"""
import os

import numpy as np
import pytest
from scipy import stats

import oracle as orc


def _kat_rows(golden_dir):
    rows = []
    with open(os.path.join(golden_dir, "philox4x32_10_kat.txt")) as fh:
        for line in fh:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            parts = line.split()
            assert parts[0] == "10"
            vals = [int(p, 16) for p in parts[1:]]
            rows.append((vals[0:4], vals[4:6], vals[6:10]))
    return rows


def test_philox_kat(golden_dir):
    rows = _kat_rows(golden_dir)
    assert len(rows) == 3
    for ctr, key, out in rows:
        got = orc.philox4x32_10(ctr, key)
        assert [int(v) for v in got] == out, (ctr, key, [hex(v) for v in got])


def test_stream_layout_uses_counter_and_key():
    # word(tag, t, i, j) = Philox(ctr={j>>2, i, t, tag}, key={seed lo, seed hi})[j & 3]
    seed = 0x0123456789ABCDEF
    key = [seed & 0xFFFFFFFF, seed >> 32]
    for tag, t, i in [(0, 1, 0), (1, 7, 12345), (2, 0, 99), (3, 0, 2**32 - 1)]:
        for j in range(0, 11):
            blk = orc.philox4x32_10([j >> 2, i, t, tag], key)
            assert orc.word(seed, tag, t, i, j) == int(blk[j & 3])
    # bulk helper agrees with the scalar one
    w = orc.words(seed, 1, 3, 17, 5, 9)
    assert [int(v) for v in w] == [orc.word(seed, 1, 3, 17, 5 + k) for k in range(9)]


def test_uniform_mapping_exact():
    # U(w) = (w >> 8) * 2^-24: exact in fp32, range [0, 1 - 2^-24]
    assert orc.uniform(0) == 0.0
    assert orc.uniform(0xFF) == 0.0
    assert orc.uniform(0x100) == 2.0 ** -24
    assert orc.uniform(0xFFFFFFFF) == 1.0 - 2.0 ** -24
    assert orc.uniform(0x80000000) == 0.5
    for w in [1, 0x1234_5678, 0xDEAD_BEEF, 0x7FFF_FFFF]:
        assert orc.uniform(w) == (w >> 8) / 2.0 ** 24


def test_uniform_distribution():
    # 2^17 draws of one stream: KS against U(0,1), mean within 4 sigma.
    u = np.array([orc.uniform(w) for w in orc.words(2021, 0, 1, 3, 0, 1 << 17)])
    assert u.min() >= 0.0 and u.max() < 1.0
    sigma = np.sqrt(1.0 / 12.0 / u.size)
    assert abs(u.mean() - 0.5) < 4 * sigma
    assert stats.kstest(u, "uniform").pvalue > 1e-4


def test_streams_are_distinct_and_uncorrelated():
    n = 1 << 14
    a = orc.words(7, 0, 1, 0, 0, n).astype(np.float64)
    b = orc.words(7, 1, 1, 0, 0, n).astype(np.float64)  # other tag
    c = orc.words(7, 0, 2, 0, 0, n).astype(np.float64)  # other iteration
    e = orc.words(8, 0, 1, 0, 0, n).astype(np.float64)  # other seed
    for other in (b, c, e):
        assert not np.array_equal(a, other)
        assert abs(np.corrcoef(a, other)[0, 1]) < 4.0 / np.sqrt(n)


@pytest.mark.parametrize("seed", [0, 1, 2**64 - 1])
def test_seed_halves_both_matter(seed):
    lo_flip = seed ^ 1
    hi_flip = seed ^ (1 << 40)
    w = orc.word(seed, 0, 1, 0, 0)
    assert orc.word(lo_flip, 0, 1, 0, 0) != w
    assert orc.word(hi_flip, 0, 1, 0, 0) != w
