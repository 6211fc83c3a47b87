"""Seeded synthetic key generators shared by the oracle side and the CUDA side.

This module holds NO arithmetic of the sorting method (no codec, no radix, no
pivot, no merge).  It only turns (seed, index) into keys, so that the oracle
(`oracle/`) and the CUDA path (`paper_conf_sigmod_maltenbergeritr22_b200`) can
be fed the same bytes.  Both a numpy (host) and a torch (any device) version of
every generator exist; they are integer-exact and produce identical bytes
(checked by tests/test_inputs.py).

Workload recipe:
  * counter-based splitmix64: h(seed, stream, i) = mix64(salt(seed, stream) +
    (i + 1) * GOLDEN), so generation is parallel and thread-count independent;
  * distributions follow the paper's Fig.16 set (uniform, normal, sorted,
    reverse-sorted, nearly-sorted) plus
    zipf from BASELINE.json; key types u32/u64/f32/f64.
"""
from __future__ import annotations

import numpy as np

GOLDEN = 0x9E3779B97F4A7C15
M1 = 0xBF58476D1CE4E5B9
M2 = 0x94D049BB133111EB
MASK64 = (1 << 64) - 1

KEY_TYPES = ("u32", "u64", "f32", "f64")
DISTRIBUTIONS = ("uniform", "normal", "sorted", "reverse", "nearly", "zipf", "zipf_rank")

NP_DTYPE = {"u32": np.uint32, "u64": np.uint64, "f32": np.float32, "f64": np.float64}
KEY_BYTES = {"u32": 4, "u64": 8, "f32": 4, "f64": 8}

ZIPF_S = 1.1
ZIPF_RANKS = 1 << 20

# IEEE special values placed at 1% of positions of the float workloads
# (SURVEY §8(c) Q1 table): +-0, +-denorm_min, +-1, +-max, +-inf, +-qNaN, +-sNaN
# with payloads.  Given as bit patterns.
F32_SPECIALS = np.array([
    0x00000000, 0x80000000, 0x00000001, 0x80000001, 0x3F800000, 0xBF800000,
    0x7F7FFFFF, 0xFF7FFFFF, 0x7F800000, 0xFF800000, 0x7FC00000, 0xFFC00000,
    0x7FC00123, 0x7F800001, 0xFF800001, 0x7FA00005], dtype=np.uint32)
F64_SPECIALS = np.array([
    0x0000000000000000, 0x8000000000000000, 0x0000000000000001, 0x8000000000000001,
    0x3FF0000000000000, 0xBFF0000000000000, 0x7FEFFFFFFFFFFFFF, 0xFFEFFFFFFFFFFFFF,
    0x7FF0000000000000, 0xFFF0000000000000, 0x7FF8000000000000, 0xFFF8000000000000,
    0x7FF8000000000123, 0x7FF0000000000001, 0xFFF0000000000001, 0x7FF4000000000005],
    dtype=np.uint64)


def _salt(seed: int, stream: int) -> int:
    z = (seed * GOLDEN + (stream + 1) * M1) & MASK64
    z = ((z ^ (z >> 30)) * M1) & MASK64
    z = ((z ^ (z >> 27)) * M2) & MASK64
    return z ^ (z >> 31)


def _zipf_cdf() -> np.ndarray:
    k = np.arange(1, ZIPF_RANKS + 1, dtype=np.float64)
    w = k ** (-ZIPF_S)
    cdf = np.cumsum(w)
    return cdf / cdf[-1]


_ZIPF_CDF = None


def zipf_cdf() -> np.ndarray:
    global _ZIPF_CDF
    if _ZIPF_CDF is None:
        _ZIPF_CDF = _zipf_cdf()
    return _ZIPF_CDF


# ----------------------------------------------------------------------------
# numpy (host) version
# ----------------------------------------------------------------------------

def np_hash(seed: int, stream: int, start: int, count: int) -> np.ndarray:
    """uint64 splitmix64 outputs for indices [start, start+count)."""
    i = np.arange(start, start + count, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = np.uint64(_salt(seed, stream)) + (i + np.uint64(1)) * np.uint64(GOLDEN)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(M1)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(M2)
        z = z ^ (z >> np.uint64(31))
    return z


def _np_fmix32(x: np.ndarray) -> np.ndarray:
    x = x.astype(np.uint64) & np.uint64(0xFFFFFFFF)
    with np.errstate(over="ignore"):
        x ^= x >> np.uint64(16)
        x = (x * np.uint64(0x85EBCA6B)) & np.uint64(0xFFFFFFFF)
        x ^= x >> np.uint64(13)
        x = (x * np.uint64(0xC2B2AE35)) & np.uint64(0xFFFFFFFF)
        x ^= x >> np.uint64(16)
    return x


def _np_sorted_u32(n: int, start: int, count: int) -> np.ndarray:
    i = np.arange(start, start + count, dtype=np.uint64)
    nn = np.uint64(max(n, 1))
    a = (i << np.uint64(16)) // nn
    ra = (i << np.uint64(16)) % nn
    return (a << np.uint64(16)) + ((ra << np.uint64(16)) // nn)


def np_generate(n: int, key_type: str = "u32", dist: str = "uniform", seed: int = 1,
                start: int = 0, count: int | None = None) -> np.ndarray:
    """Keys [start, start+count) of the length-n workload (dist, key_type, seed)."""
    if count is None:
        count = n - start
    if key_type not in KEY_TYPES:
        raise ValueError(key_type)
    if key_type in ("u64",):
        if dist != "uniform":
            raise ValueError("u64 workloads are uniform (SURVEY §8(d) C5)")
        return np_hash(seed, 0, start, count)
    if key_type in ("f32", "f64"):
        if dist != "uniform":
            raise ValueError("float workloads are uniform + 1% specials (SURVEY §8(d) C5)")
        h = np_hash(seed, 0, start, count)
        x = -1000.0 + 2000.0 * ((h >> np.uint64(11)).astype(np.float64) * (2.0 ** -53))
        pick = ((np_hash(seed, 1, start, count) >> np.uint64(1)) % np.uint64(100)) == 0
        which = (np_hash(seed, 2, start, count) >> np.uint64(1)) % np.uint64(16)
        if key_type == "f32":
            bits = x.astype(np.float32).view(np.uint32).copy()
            bits[pick] = F32_SPECIALS[which[pick].astype(np.int64)]
            return bits.view(np.float32)
        bits = x.view(np.uint64).copy()
        bits[pick] = F64_SPECIALS[which[pick].astype(np.int64)]
        return bits.view(np.float64)
    # u32
    if dist == "uniform":
        out = np_hash(seed, 0, start, count) >> np.uint64(32)
    elif dist == "sorted":
        out = _np_sorted_u32(n, start, count)
    elif dist == "reverse":
        out = np.uint64(0xFFFFFFFF) - _np_sorted_u32(n, start, count)
    elif dist == "nearly":
        out = _np_sorted_u32(n, start, count)
        pick = ((np_hash(seed, 2, start, count) >> np.uint64(1)) % np.uint64(100)) == 0
        out[pick] = (np_hash(seed, 3, start, count) >> np.uint64(32))[pick]
    elif dist == "normal":
        acc = np.zeros(count, dtype=np.int64)
        for j in range(12):
            acc += (np_hash(seed, 10 + j, start, count) >> np.uint64(32)).astype(np.int64)
        v = (acc >> 3) + (1 << 31) - (3 << 30)
        out = np.clip(v, 0, 0xFFFFFFFF).astype(np.uint64)
    elif dist in ("zipf", "zipf_rank"):
        u = (np_hash(seed, 4, start, count) >> np.uint64(11)).astype(np.float64) * (2.0 ** -53)
        rank = np.searchsorted(zipf_cdf(), u, side="right").astype(np.uint64) + np.uint64(1)
        rank = np.minimum(rank, np.uint64(ZIPF_RANKS))
        out = _np_fmix32(rank) if dist == "zipf" else rank
    else:
        raise ValueError(dist)
    return out.astype(np.uint32)


# ----------------------------------------------------------------------------
# torch version (same integers; runs on CPU or CUDA).  int64 arithmetic wraps
# mod 2^64 exactly like uint64; logical right shifts are emulated with masks.
# ----------------------------------------------------------------------------

def _s64(x: int) -> int:
    x &= MASK64
    return x - (1 << 64) if x >= (1 << 63) else x


def _t_srl(z, s: int):
    import torch
    return (z >> s) & ((1 << (64 - s)) - 1)


def t_hash(seed: int, stream: int, start: int, count: int, device):
    import torch
    i = torch.arange(start + 1, start + count + 1, dtype=torch.int64, device=device)
    z = i * _s64(GOLDEN) + _s64(_salt(seed, stream))
    z = (z ^ _t_srl(z, 30)) * _s64(M1)
    z = (z ^ _t_srl(z, 27)) * _s64(M2)
    z = z ^ _t_srl(z, 31)
    return z


def _t_fmix32(x):
    x = x & 0xFFFFFFFF
    x = x ^ (x >> 16)
    x = (x * 0x85EBCA6B) & 0xFFFFFFFF
    x = x ^ (x >> 13)
    x = (x * 0xC2B2AE35) & 0xFFFFFFFF
    x = x ^ (x >> 16)
    return x


def _t_sorted_u32(n: int, start: int, count: int, device):
    import torch
    i = torch.arange(start, start + count, dtype=torch.int64, device=device)
    nn = max(n, 1)
    a = torch.div(i << 16, nn, rounding_mode="floor")
    ra = torch.remainder(i << 16, nn)
    return (a << 16) + torch.div(ra << 16, nn, rounding_mode="floor")


def _t_to_u32_storage(v):
    """int64 tensor holding values in [0, 2^32) -> uint32 tensor (same bits)."""
    import torch
    v = torch.where(v >= (1 << 31), v - (1 << 32), v)
    return v.to(torch.int32).view(torch.uint32)


def t_generate_into(out, n: int, key_type: str = "u32", dist: str = "uniform", seed: int = 1,
                    start: int = 0, block: int = 1 << 26):
    """Fill the 1-D tensor `out` (dtype of the key type's width) with keys
    [start, start+len(out)) of the length-n workload, in blocks (bounded temp memory)."""
    import torch
    total = out.numel()
    device = out.device
    flat_bits = out.view(torch.int32) if KEY_BYTES[key_type] == 4 else out.view(torch.int64)
    for off in range(0, total, block):
        cnt = min(block, total - off)
        s = start + off
        if key_type == "u64":
            if dist != "uniform":
                raise ValueError("u64 workloads are uniform")
            flat_bits[off:off + cnt] = t_hash(seed, 0, s, cnt, device)
            continue
        if key_type in ("f32", "f64"):
            if dist != "uniform":
                raise ValueError("float workloads are uniform + 1% specials")
            h = t_hash(seed, 0, s, cnt, device)
            x = -1000.0 + 2000.0 * (_t_srl(h, 11).to(torch.float64) * (2.0 ** -53))
            pick = (_t_srl(t_hash(seed, 1, s, cnt, device), 1) % 100) == 0
            which = _t_srl(t_hash(seed, 2, s, cnt, device), 1) % 16
            if key_type == "f32":
                bits = x.to(torch.float32).view(torch.int32).clone()
                sp = torch.from_numpy(F32_SPECIALS.view(np.int32).copy()).to(device)
            else:
                bits = x.view(torch.int64).clone()
                sp = torch.from_numpy(F64_SPECIALS.view(np.int64).copy()).to(device)
            bits[pick] = sp[which[pick]]
            flat_bits[off:off + cnt] = bits
            continue
        if dist == "uniform":
            v = _t_srl(t_hash(seed, 0, s, cnt, device), 32)
        elif dist == "sorted":
            v = _t_sorted_u32(n, s, cnt, device)
        elif dist == "reverse":
            v = 0xFFFFFFFF - _t_sorted_u32(n, s, cnt, device)
        elif dist == "nearly":
            v = _t_sorted_u32(n, s, cnt, device)
            pick = (_t_srl(t_hash(seed, 2, s, cnt, device), 1) % 100) == 0
            v = torch.where(pick, _t_srl(t_hash(seed, 3, s, cnt, device), 32), v)
        elif dist == "normal":
            acc = torch.zeros(cnt, dtype=torch.int64, device=device)
            for j in range(12):
                acc += _t_srl(t_hash(seed, 10 + j, s, cnt, device), 32)
            v = torch.clamp((acc >> 3) + (1 << 31) - (3 << 30), 0, 0xFFFFFFFF)
        elif dist in ("zipf", "zipf_rank"):
            u = _t_srl(t_hash(seed, 4, s, cnt, device), 11).to(torch.float64) * (2.0 ** -53)
            cdf = torch.from_numpy(zipf_cdf()).to(device)
            rank = torch.searchsorted(cdf, u, right=True) + 1
            rank = torch.clamp(rank, max=ZIPF_RANKS)
            v = _t_fmix32(rank) if dist == "zipf" else rank
        else:
            raise ValueError(dist)
        flat_bits[off:off + cnt] = _t_to_u32_storage(v).view(torch.int32)
    return out


def torch_dtype(key_type: str):
    import torch
    return {"u32": torch.uint32, "u64": torch.uint64, "f32": torch.float32, "f64": torch.float64}[key_type]


def t_generate(n: int, key_type: str = "u32", dist: str = "uniform", seed: int = 1, device="cpu"):
    import torch
    out = torch.empty(n, dtype=torch_dtype(key_type), device=device)
    return t_generate_into(out, n, key_type, dist, seed)
