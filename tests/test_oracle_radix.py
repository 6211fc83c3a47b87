"""Pins for oracle/radix.py (no GPU).

  * histogram rows sum to n and equal a pure-Python count;
  * each counting pass equals Python's stable `sorted(..., key=digit)` (Timsort,
    a different primitive) - stability is what LSD correctness needs;
  * after all P passes the codes equal the library sort (LSD radix theorem).
"""
import numpy as np
import pytest

import msort_inputs as mi
from oracle import codec, radix


@pytest.mark.parametrize("kt", mi.KEY_TYPES)
def test_histogram_counts(kt):
    a = mi.np_generate(3000, kt, "uniform", seed=4)
    h = radix.histograms(a, kt)
    assert h.shape == (radix.num_passes(kt), 256)
    assert np.all(h.sum(axis=1) == len(a))
    t = [int(x) for x in codec.encode(a, kt)]
    for k in range(radix.num_passes(kt)):
        ref = [0] * 256
        for v in t:
            ref[(v >> (8 * k)) & 255] += 1
        assert list(h[k]) == ref


def test_exclusive_bases():
    row = np.array([3, 0, 5] + [0] * 252 + [2], dtype=np.uint64)
    b = radix.exclusive_bases(row)
    assert b[0] == 0 and b[1] == 3 and b[2] == 3 and b[3] == 8 and b[255] == 8


@pytest.mark.parametrize("kt", mi.KEY_TYPES)
def test_counting_pass_is_stable_digit_sort(kt):
    a = mi.np_generate(2000, kt, "uniform", seed=6)
    t = codec.encode(a, kt)
    # force duplicate digits so stability is visible
    t = t & np.array(0x0F0F0F0F0F0F0F0F if codec.BITS[kt] == 64 else 0x0F0F0F0F, dtype=t.dtype)
    cur = t
    for k in range(radix.num_passes(kt)):
        nxt = radix.counting_pass(cur, k)
        ref = sorted(range(len(cur)), key=lambda i: (int(cur[i]) >> (8 * k)) & 255)
        assert np.array_equal(nxt, cur[ref])
        cur = nxt
    assert np.array_equal(cur, np.sort(t))


@pytest.mark.parametrize("dist", mi.DISTRIBUTIONS)
def test_lsd_equals_sort_u32(dist):
    a = mi.np_generate(20000, "u32", dist, seed=1)
    t = codec.encode(a, "u32")
    assert np.array_equal(radix.lsd_radix_sort_codes(t, "u32")[-1], np.sort(t))
