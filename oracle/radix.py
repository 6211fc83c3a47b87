"""LSD radix sort, step by step (oracle side).

PAPER.md §5.1: the single-GPU chunk sort is an LSB radix sort
(Thrust/CUB) that computes "the histogram once" and decouples the
prefix sum, so each pass reads and writes the keys once (2n instead of 3n,
P:1551-1561).  The digit width is internal to Thrust; reading Q10
fixes r = 8 bits, so a K-byte key takes P = K passes, least significant digit
first.  Digits are taken from T(key) (reading Q1).

Oracle steps:
  histograms(codes)       one count array of 2^r bins per digit position (S2)
  exclusive_bases(hist)   global bucket base per digit value (prefix sum, S2)
  counting_pass(codes, k) stable distribution of all keys by digit k (S3):
                          out[base[d] + #{j < i : digit_k(j) == d}] = key i
"""
from __future__ import annotations

import numpy as np

from . import codec

RADIX_BITS = 8
RADIX = 1 << RADIX_BITS


def num_passes(key_type: str) -> int:
    return codec.BITS[key_type] // RADIX_BITS


def digit(codes: np.ndarray, k: int) -> np.ndarray:
    """Digit k (k = 0 is least significant) of unsigned codes."""
    return ((codes >> np.array(RADIX_BITS * k, dtype=codes.dtype)) & np.array(RADIX - 1, dtype=codes.dtype)).astype(np.int64)


def histograms(keys: np.ndarray, key_type: str) -> np.ndarray:
    """[P, 256] digit counts of T(keys) for every pass (P:1559 'histogram once')."""
    t = codec.encode(keys, key_type)
    return np.stack([np.bincount(digit(t, k), minlength=RADIX) for k in range(num_passes(key_type))]).astype(np.uint64)


def exclusive_bases(hist_row: np.ndarray) -> np.ndarray:
    """Exclusive prefix sum of one histogram row: first output slot of each digit value."""
    out = np.zeros(RADIX, dtype=np.uint64)
    run = 0
    for d in range(RADIX):
        out[d] = run
        run += int(hist_row[d])
    return out


def counting_pass(codes: np.ndarray, k: int) -> np.ndarray:
    """One stable LSD pass over unsigned codes on digit k (textbook counting sort).

    out[base[d] + rank] = codes[i], rank = number of earlier keys with the same digit.
    Vectorised form of the textbook loop: a stable argsort of the digit gives, for
    every output slot in order, the input index that lands there.
    """
    d = digit(codes, k)
    order = np.argsort(d, kind="stable")
    return codes[order]


def lsd_radix_sort_codes(codes: np.ndarray, key_type: str) -> list[np.ndarray]:
    """All intermediate results of the P passes (index p = after pass p)."""
    out = []
    cur = codes
    for k in range(num_passes(key_type)):
        cur = counting_pass(cur, k)
        out.append(cur)
    return out
