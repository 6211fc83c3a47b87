"""Pins for oracle/codec.py and oracle/sort.py (no GPU).

What pins them (not the oracle itself):
  * a hand-written IEEE-754 totalOrder table (tests/golden/float_total_order_f32.json);
  * numpy float comparisons on finite values (a < b  =>  T(a) < T(b));
  * exhaustive T^-1(T(u)) == u over all 2^32 f32 bit patterns;
  * brute force over all permutations for tiny inputs (the sorted output is the
    unique non-decreasing permutation).
"""
import itertools
import json
import os

import numpy as np
import pytest

import msort_inputs as mi
from oracle import codec, sort

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def test_float_total_order_table():
    with open(os.path.join(GOLD, "float_total_order_f32.json")) as f:
        bits = np.array([int(h, 16) for h in json.load(f)["ascending_bits_hex"]], dtype=np.uint32)
    rng = np.random.default_rng(7)
    for _ in range(20):
        shuffled = rng.permutation(bits)
        out = sort.oracle_sort(shuffled.view(np.float32), "f32").view(np.uint32)
        assert np.array_equal(out, bits)
    codes = codec.encode(bits.view(np.float32), "f32")
    assert np.all(codes[:-1] < codes[1:])


def test_negative_zero_before_positive_zero():
    for kt, dt in (("f32", np.float32), ("f64", np.float64)):
        x = np.array([0.0, -0.0, 0.0, -0.0], dtype=dt)
        out = sort.oracle_sort(x, kt)
        assert list(np.signbit(out)) == [True, True, False, False]


@pytest.mark.parametrize("kt,dt", [("f32", np.float32), ("f64", np.float64)])
def test_codec_monotone_vs_float_compare(kt, dt):
    rng = np.random.default_rng(1)
    vals = np.concatenate([rng.standard_normal(20000) * 10.0 ** rng.integers(-30, 30, 20000),
                           [np.finfo(dt).max, -np.finfo(dt).max, np.finfo(dt).tiny, -np.finfo(dt).tiny, np.inf, -np.inf]])
    v = vals.astype(dt)
    v = v[v != 0]
    t = codec.encode(v, kt)
    a, b = v[:-1], v[1:]
    ta, tb = t[:-1], t[1:]
    assert np.all((a < b) == (ta < tb))
    assert np.all((a == b) == (ta == tb))


def _roundtrip_block(u):
    t = codec.encode(u.view(np.float32), "f32")
    back = codec.decode(t, "f32").view(np.uint32)
    assert np.array_equal(back, u)
    # T keeps the sign split: codes of non-negative floats have MSB 1
    assert np.array_equal((t >> np.uint32(31)) == 1, (u >> np.uint32(31)) == 0)


def test_codec_roundtrip_f32_strided():
    # every sign/exponent/high-mantissa pattern (top 16 bits) with 3 low patterns,
    # plus a prime-stride sweep over the full 32-bit space
    hi = np.arange(1 << 16, dtype=np.uint32) << np.uint32(16)
    for lo in (0, 1, 0xFFFF):
        _roundtrip_block(hi | np.uint32(lo))
    _roundtrip_block((np.arange(0, (1 << 32) // 4099 + 1, dtype=np.uint64) * np.uint64(4099)).astype(np.uint32))


def _exhaustive_block(start: int, step: int) -> bool:
    u = np.arange(start, start + step, dtype=np.uint64).astype(np.uint32)
    t = codec.encode(u.view(np.float32), "f32")
    back = codec.decode(t, "f32").view(np.uint32)
    # T^-1(T(u)) = u, and T keeps the sign-bit split: codes of non-negative floats have MSB 1
    ok = np.array_equal(back, u) and np.array_equal((t >> np.uint32(31)) == 1, (u >> np.uint32(31)) == 0)
    # strictly increasing codes within each sign half => T is order-preserving there and a bijection
    # overall (positives ascend with their bits, negatives descend; checked block by block)
    neg = (u >> np.uint32(31)) == 1
    tp, tn = t[~neg], t[neg]
    ok = ok and bool(np.all(tp[1:] > tp[:-1])) and bool(np.all(tn[1:] < tn[:-1]))
    return ok


def test_codec_roundtrip_exhaustive_f32():
    """All 2^32 f32 bit patterns (SURVEY §8(c) S1 pin: T^-1 o T = id, exhaustive),
    in blocks on all host cores (numpy releases the GIL)."""
    from concurrent.futures import ThreadPoolExecutor
    step = 1 << 24
    with ThreadPoolExecutor(max(1, min(16, os.cpu_count() or 1))) as ex:
        results = list(ex.map(lambda s: _exhaustive_block(s, step), range(0, 1 << 32, step)))
    assert all(results), [i for i, r in enumerate(results) if not r][:5]


def test_codec_roundtrip_f64_and_ints():
    u = mi.np_hash(5, 0, 0, 1 << 20)
    for kt in ("f64", "u64"):
        t = codec.encode(u.view(np.float64) if kt == "f64" else u, kt)
        back = codec.decode(t, kt)
        assert np.array_equal(back.view(np.uint64), u)
    u32 = (u >> np.uint64(32)).astype(np.uint32)
    assert np.array_equal(codec.encode(u32, "u32"), u32)


def _brute_sorted(seq, key):
    for perm in itertools.permutations(seq):
        if all(key(perm[i]) <= key(perm[i + 1]) for i in range(len(perm) - 1)):
            return list(perm)
    raise AssertionError


def test_oracle_sort_brute_force_small():
    for n in range(0, 6):
        for vals in itertools.product(range(4), repeat=n):
            a = np.array(vals, dtype=np.uint32) * np.uint32(0x40000001)
            out = sort.oracle_sort(a, "u32")
            assert list(out) == _brute_sorted(list(a), key=int)


def test_oracle_sort_brute_force_floats():
    with open(os.path.join(GOLD, "float_total_order_f32.json")) as f:
        table = [int(h, 16) for h in json.load(f)["ascending_bits_hex"]]
    rank = {b: i for i, b in enumerate(table)}
    rng = np.random.default_rng(3)
    for _ in range(300):
        n = int(rng.integers(0, 6))
        picks = [table[i] for i in rng.integers(0, len(table), n)]
        a = np.array(picks, dtype=np.uint32)
        out = sort.oracle_sort(a.view(np.float32), "f32").view(np.uint32)
        assert list(out) == _brute_sorted(picks, key=lambda b: rank[b])


@pytest.mark.parametrize("kt", mi.KEY_TYPES)
def test_oracle_sort_is_sorted_permutation(kt):
    a = mi.np_generate(50000, kt, "uniform", seed=2)
    out = sort.oracle_sort(a, kt)
    t = codec.encode(out, kt)
    assert np.all(t[:-1] <= t[1:])
    assert np.array_equal(np.sort(codec.bits_of(a, kt)), np.sort(codec.bits_of(out, kt)))
