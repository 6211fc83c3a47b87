"""The plain definition of what the hot path computes (oracle side).

Problem statement: n keys in host memory end up sorted ascending (PAPER.md
P:2244-2248, §6); the P2P sort reaches exactly this result, only faster
(§5.2).  Under the total order of DESIGN.md reading Q1 the
keys-only sort is unique, so the oracle is exact and byte-comparable.

Steps: copy -> T -> library sort -> T^-1.
"""
from __future__ import annotations

import numpy as np

from . import codec


def oracle_sort(keys: np.ndarray, key_type: str) -> np.ndarray:
    """Sorted copy of `keys` under the T order (reading Q1)."""
    t = codec.encode(keys, key_type)
    t.sort(kind="stable")   # library sort primitive on unsigned codes
    return codec.decode(t, key_type)
