"""Key codec T and its inverse (oracle side).

The paper sorts "integers, floats, longs and doubles" (PAPER.md P:3232-3236,
§6.3) with Thrust's LSB radix sort and merges by comparison
(P:1596-1598).  It is silent on the order of -0.0/+0.0 and NaN.
reading Q1: the order is the unsigned order of T(key), where
  u32/u64: T = identity
  f32/f64: T(u) = u ^ (sign(u) ? all-ones : sign-bit)
which is IEEE-754 totalOrder on bit patterns (-NaN < -inf < ... < -0.0 < +0.0 <
... < +inf < +NaN).  Keys never change bits: T^-1(T(u)) == u.
"""
from __future__ import annotations

import numpy as np

UINT = {"u32": np.uint32, "u64": np.uint64, "f32": np.uint32, "f64": np.uint64}
BITS = {"u32": 32, "u64": 64, "f32": 32, "f64": 64}
FLOAT = {"f32", "f64"}


def bits_of(keys: np.ndarray, key_type: str) -> np.ndarray:
    """Raw key bits as unsigned integers of the key width (a view, no copy)."""
    return np.ascontiguousarray(keys).view(UINT[key_type])


def encode(keys: np.ndarray, key_type: str) -> np.ndarray:
    """T(keys) as unsigned integers (new array). DESIGN.md reading Q1."""
    u = bits_of(keys, key_type).copy()
    if key_type not in FLOAT:
        return u
    w = UINT[key_type]
    sign = np.array(1 << (BITS[key_type] - 1), dtype=w)
    ones = np.array((1 << BITS[key_type]) - 1, dtype=w)
    neg = (u & sign) != 0
    # negative: flip all bits; non-negative: flip the sign bit
    return u ^ np.where(neg, ones, sign)


def decode(codes: np.ndarray, key_type: str) -> np.ndarray:
    """T^-1(codes) -> keys of key_type (new array)."""
    w = UINT[key_type]
    u = np.ascontiguousarray(codes).astype(w, copy=True)
    if key_type in FLOAT:
        sign = np.array(1 << (BITS[key_type] - 1), dtype=w)
        ones = np.array((1 << BITS[key_type]) - 1, dtype=w)
        was_nonneg = (u & sign) != 0
        u = u ^ np.where(was_nonneg, sign, ones)
    dt = {"u32": np.uint32, "u64": np.uint64, "f32": np.float32, "f64": np.float64}[key_type]
    return u.view(dt)

