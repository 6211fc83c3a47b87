"""Properties of the sorted output that hold at any size (oracle side).

Used for full-size parity (BASELINE.json configs at 4e9 keys) where a full
oracle copy is too slow or too large: SURVEY.md §8(c) "What pins each part" -
non-decreasing under the T order AND a permutation of the input together imply
equality with the unique sorted result; sampled outputs are checked one by
one as order statistics of the input.
"""
from __future__ import annotations

import numpy as np

from . import codec

_MIX_A = np.uint64(0xD6E8FEB86659FD93)


def is_sorted_codes(codes: np.ndarray) -> bool:
    """codes[i] <= codes[i+1] for all i (non-decreasing under T; reading Q1)."""
    if len(codes) < 2:
        return True
    return bool(np.all(codes[:-1] <= codes[1:]))


def fingerprint(keys: np.ndarray, key_type: str, block: int = 1 << 24) -> tuple[int, int, int]:
    """Order-independent multiset fingerprint (count, sum mix1, xor mix2) mod 2^64
    of the key codes.  Equal multisets give equal fingerprints; a permutation
    check at sizes where a full histogram is too large."""
    n = len(keys)
    s = np.uint64(0)
    x = np.uint64(0)
    with np.errstate(over="ignore"):
        for off in range(0, n, block):
            t = codec.encode(keys[off:off + block], key_type).astype(np.uint64)
            h = (t ^ (t >> np.uint64(29))) * _MIX_A
            h ^= h >> np.uint64(32)
            s = s + np.sum(h, dtype=np.uint64)
            h2 = (t + np.uint64(0x9E3779B97F4A7C15)) * np.uint64(0xBF58476D1CE4E5B9)
            h2 ^= h2 >> np.uint64(31)
            x ^= np.bitwise_xor.reduce(h2) if len(h2) else np.uint64(0)
    return n, int(s), int(x)


def order_statistic_ok(input_keys: np.ndarray, output_keys: np.ndarray, key_type: str,
                       ranks: np.ndarray, block: int = 1 << 24) -> np.ndarray:
    """For each sampled rank k: out[k] is the k-th smallest input key, i.e.
    #{input < out[k]} <= k < #{input <= out[k]} (under T).  Returns a bool per rank."""
    ranks = np.asarray(ranks, dtype=np.int64)
    vals = codec.encode(output_keys[ranks], key_type)
    lt = np.zeros(len(ranks), dtype=np.int64)
    le = np.zeros(len(ranks), dtype=np.int64)
    order = np.argsort(vals, kind="stable")
    sv = vals[order]
    m = len(sv)
    lt_s = np.zeros(m + 1, dtype=np.int64)
    le_s = np.zeros(m + 1, dtype=np.int64)
    for off in range(0, len(input_keys), block):
        t = codec.encode(input_keys[off:off + block], key_type)
        # input t < sv[j]  <=>  j >= #{sv <= t};   input t <= sv[j]  <=>  j >= #{sv < t}
        lt_s += np.bincount(np.searchsorted(sv, t, side="right"), minlength=m + 1)
        le_s += np.bincount(np.searchsorted(sv, t, side="left"), minlength=m + 1)
    lt[order] = np.cumsum(lt_s)[:m]
    le[order] = np.cumsum(le_s)[:m]
    return (lt <= ranks) & (ranks < le)
