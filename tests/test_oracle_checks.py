"""Pins for oracle/checks.py (no GPU): the any-size properties agree with the
definition on small inputs and reject plausible corruptions."""
import numpy as np
import pytest

import msort_inputs as mi
from oracle import checks, codec, sort


@pytest.mark.parametrize("kt", mi.KEY_TYPES)
def test_properties_accept_sorted_reject_corrupt(kt):
    a = mi.np_generate(20000, kt, "uniform", seed=8)
    out = sort.oracle_sort(a, kt)
    assert checks.is_sorted_codes(codec.encode(out, kt))
    assert checks.fingerprint(a, kt) == checks.fingerprint(out, kt)
    ranks = np.array([0, 1, 17, 9999, 19999])
    assert checks.order_statistic_ok(a, out, kt, ranks).all()
    # corruptions: swap two distinct neighbours / replace a key by a duplicate of its neighbour
    bad = out.copy()
    bits = codec.bits_of(bad, kt)
    i = int(np.nonzero(bits[1:] != bits[:-1])[0][100])
    bits[i], bits[i + 1] = bits[i + 1].copy(), bits[i].copy()
    assert not checks.is_sorted_codes(codec.encode(bad, kt))
    assert not checks.order_statistic_ok(a, bad, kt, np.array([i, i + 1])).any()
    dup = out.copy()
    db = codec.bits_of(dup, kt)
    db[i + 1] = db[i]
    assert checks.is_sorted_codes(codec.encode(dup, kt))          # still sorted ...
    assert checks.fingerprint(a, kt) != checks.fingerprint(dup, kt)  # ... but not a permutation


def test_order_statistic_with_duplicates():
    a = np.array([5, 1, 5, 5, 2, 9, 1], dtype=np.uint32)
    out = np.sort(a)
    assert checks.order_statistic_ok(a, out, "u32", np.arange(7)).all()
    wrong = out.copy()
    wrong[3] = 2
    assert not checks.order_statistic_ok(a, wrong, "u32", np.array([3]))[0]
