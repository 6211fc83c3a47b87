"""HET sort baseline (comparison only; §5.3):
g chunks are sorted on the GPU(s) with libmsort's radix sort (the same chunk
sort the P2P path uses), copied back to the host, and merged on the CPU with a
parallel multiway merge (libstdc++ parallel mode, a loser tree) on all host
cores.  Timed end to end from pinned host keys like msort_sort_host."""
from __future__ import annotations

import ctypes
import os
import subprocess
import time

HERE = os.path.dirname(os.path.abspath(__file__))
LIB = os.path.join(HERE, "libhet_merge.so")


def build() -> str:
    src = os.path.join(HERE, "het_merge.cpp")
    if not os.path.exists(LIB) or os.path.getmtime(LIB) < os.path.getmtime(src):
        subprocess.run(["g++", "-O3", "-march=x86-64-v3", "-fopenmp", "-shared", "-fPIC", "-o", LIB, src], check=True)
    return LIB


def het_sort_host(host_keys, key_type: str, chunks: int = 8, devices: list[int] | None = None, threads: int = 0):
    """Sort the pinned host tensor `host_keys` (1-D) in place via HET; returns a dict of phase times."""
    import torch

    import paper_conf_sigmod_maltenbergeritr22_b200 as ms
    lib = ctypes.CDLL(build())
    lib.het_multiway_merge.argtypes = [ctypes.POINTER(ctypes.c_void_p), ctypes.POINTER(ctypes.c_uint64), ctypes.c_int,
                                       ctypes.c_void_p, ctypes.c_int, ctypes.c_int]
    n = host_keys.numel()
    devices = devices or [0]
    c = (n + chunks - 1) // chunks
    t0 = time.perf_counter()
    bufs, lens = [], []
    for i in range(chunks):
        lo, hi = i * c, min(n, (i + 1) * c)
        if hi <= lo:
            continue
        dev = torch.device("cuda", devices[i % len(devices)])
        d = host_keys[lo:hi].to(dev, non_blocking=True)
        aux = torch.empty_like(d)
        wsb = ms.msort_radix_workspace_bytes(hi - lo, key_type)
        ws = torch.empty(wsb, dtype=torch.uint8, device=dev)
        with torch.cuda.device(dev):
            ms.msort_radix_sort(ms.tensor_ptr(d), ms.tensor_ptr(aux), hi - lo, key_type, ms.tensor_ptr(ws), wsb,
                                torch.cuda.current_stream(dev))
        bufs.append(d)
        lens.append(hi - lo)
    runs = [torch.empty(b.numel(), dtype=b.dtype, pin_memory=True) for b in bufs]
    for r, b in zip(runs, bufs):
        r.copy_(b, non_blocking=True)
    torch.cuda.synchronize()
    t1 = time.perf_counter()
    ptrs = (ctypes.c_void_p * len(runs))(*[r.data_ptr() for r in runs])
    ls = (ctypes.c_uint64 * len(runs))(*lens)
    kt = ms.KEY_TYPES[key_type]
    rc = lib.het_multiway_merge(ptrs, ls, len(runs), ctypes.c_void_p(host_keys.data_ptr()), kt, threads)
    if rc:
        raise RuntimeError("het merge failed")
    t2 = time.perf_counter()
    return {"gpu_sort_and_copies_s": t1 - t0, "cpu_merge_s": t2 - t1, "total_s": t2 - t0, "chunks": len(runs),
            "threads": threads or os.cpu_count()}
