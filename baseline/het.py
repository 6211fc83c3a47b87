"""CPU-side comparison baselines (never the product path).

HET sort (§5.3): the keys are split into
`chunks` chunks, the chunks are sorted on the GPUs (chunk i on devices[i % g],
all GPUs at once) with libmsort's radix sort - the same chunk
sort the P2P path uses - copied back to the host, and merged on the CPU with a
parallel multiway merge (libstdc++ parallel mode, a loser tree)
on all host cores.  `HetSort` allocates every device and pinned buffer up
front (the paper pre-allocates), so `run` times only the
transfers, the GPU sorts and the CPU merge.

cpu_parallel_sort: GNU parallel mode's sort on the host cores (the paper's CPU
library baseline family, §6), reported beside the oracle.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import time

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
LIB = os.path.join(HERE, "libhet_merge.so")
OOC_LIB = os.path.join(HERE, "libhet_ooc.so")
PKG = os.path.join(ROOT, "paper_conf_sigmod_maltenbergeritr22_b200")
CUDA = "/usr/local/cuda"
_lib = None
_ooc = None


def _stale(lib, *srcs):
    return not os.path.exists(lib) or any(os.path.getmtime(lib) < os.path.getmtime(s) for s in srcs)


def build() -> str:
    src = os.path.join(HERE, "het_merge.cpp")
    if _stale(LIB, src):
        subprocess.run(["g++", "-O3", "-march=x86-64-v3", "-fopenmp", "-shared", "-fPIC", "-o", LIB, src], check=True)
    # NEXT-4: the out-of-core (2n) HET pipeline - CUDA runtime (static) + libmsort's C ABI
    osrc = os.path.join(HERE, "het_ooc.cpp")
    if _stale(OOC_LIB, osrc, os.path.join(PKG, "libmsort.so")):
        subprocess.run(["g++", "-O3", "-march=x86-64-v3", "-fopenmp", "-shared", "-fPIC", "-std=c++17", "-o", OOC_LIB,
                        osrc, f"-I{CUDA}/include", f"-L{CUDA}/lib64", "-lcudart_static", f"-L{PKG}", "-lmsort",
                        "-Wl,-rpath,$ORIGIN/../paper_conf_sigmod_maltenbergeritr22_b200", "-ldl", "-lrt", "-lpthread"],
                       check=True)
    return LIB


def _load():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        _lib.het_multiway_merge.argtypes = [ctypes.POINTER(ctypes.c_void_p), ctypes.POINTER(ctypes.c_uint64),
                                            ctypes.c_int, ctypes.c_void_p, ctypes.c_int, ctypes.c_int]
        _lib.cpu_parallel_sort.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int, ctypes.c_int]
        _lib.het_max_threads.restype = ctypes.c_int
    return _lib


class het_ooc_stats(ctypes.Structure):
    _fields_ = [("gpu_phase_s", ctypes.c_double), ("merge_s", ctypes.c_double), ("total_s", ctypes.c_double),
                ("chunks", ctypes.c_uint64), ("chunk_groups", ctypes.c_uint64), ("threads", ctypes.c_int)]


def het_ooc_sort(host_keys, key_type: str, chunk_keys: int, devices: list[int], host_out, threads: int = 0) -> dict:
    """NEXT-4: sort the pinned host tensor `host_keys` in chunk groups of len(devices)
    chunks of `chunk_keys` keys with two chunk buffers per GPU (the 2n-approach), then merge every
    sorted chunk on the CPU into `host_out`; returns the phase times."""
    global _ooc
    import paper_conf_sigmod_maltenbergeritr22_b200 as ms
    if _ooc is None:
        build()
        _ooc = ctypes.CDLL(OOC_LIB)
        _ooc.het_ooc_sort.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int, ctypes.c_int,
                                      ctypes.POINTER(ctypes.c_int), ctypes.c_uint64, ctypes.c_void_p, ctypes.c_int,
                                      ctypes.POINTER(het_ooc_stats)]
        _ooc.het_ooc_last_error.restype = ctypes.c_char_p
    devs = (ctypes.c_int * len(devices))(*devices)
    st = het_ooc_stats()
    rc = _ooc.het_ooc_sort(ctypes.c_void_p(host_keys.data_ptr()), host_keys.numel(), ms.KEY_TYPES[key_type],
                           len(devices), devs, chunk_keys, ctypes.c_void_p(host_out.data_ptr()), threads,
                           ctypes.byref(st))
    if rc:
        raise RuntimeError(f"het_ooc_sort: {rc}: {_ooc.het_ooc_last_error().decode()}")
    return {k: getattr(st, k) for k, _ in het_ooc_stats._fields_}


def max_threads() -> int:
    return int(_load().het_max_threads())


def cpu_parallel_sort(keys_ptr: int, n: int, key_type: int, threads: int = 0) -> None:
    """__gnu_parallel::sort of n keys at host address keys_ptr (T order)."""
    if _load().cpu_parallel_sort(ctypes.c_void_p(keys_ptr), n, key_type, threads):
        raise RuntimeError("cpu_parallel_sort failed")


class HetSort:
    """Pre-allocated HET sort of n keys of key_type in `chunks` chunks on `devices`."""

    def __init__(self, n: int, key_type: str, chunks: int = 8, devices: list[int] | None = None, threads: int = 0):
        import torch

        import paper_conf_sigmod_maltenbergeritr22_b200 as ms
        self.ms, self.torch = ms, torch
        self.n, self.key_type, self.threads = n, key_type, threads
        self.devices = devices or [0]
        dt = {"u32": torch.int32, "f32": torch.int32, "u64": torch.int64, "f64": torch.int64}[key_type]
        c = (n + chunks - 1) // chunks
        self.parts = []
        for i in range(chunks):
            lo, hi = i * c, min(n, (i + 1) * c)
            if hi <= lo:
                continue
            dev = torch.device("cuda", self.devices[i % len(self.devices)])
            wsb = ms.msort_radix_workspace_bytes(hi - lo, key_type)
            self.parts.append({
                "lo": lo, "hi": hi, "dev": dev, "stream": torch.cuda.Stream(device=dev),
                "d": torch.empty(hi - lo, dtype=dt, device=dev), "aux": torch.empty(hi - lo, dtype=dt, device=dev),
                "ws": torch.empty(wsb, dtype=torch.uint8, device=dev), "wsb": wsb,
                "run": torch.empty(hi - lo, dtype=dt, pin_memory=True)})
        lib = _load()
        self.lib = lib
        self.ptrs = (ctypes.c_void_p * len(self.parts))(*[p["run"].data_ptr() for p in self.parts])
        self.lens = (ctypes.c_uint64 * len(self.parts))(*[p["hi"] - p["lo"] for p in self.parts])

    def run(self, host_keys) -> dict:
        """Sort the pinned 1-D host tensor `host_keys` (n keys, same element width) in place."""
        torch, ms = self.torch, self.ms
        src = host_keys.view(self.parts[0]["d"].dtype) if self.parts else host_keys
        t0 = time.perf_counter()
        for p in self.parts:  # H2D + radix sort + D2H per chunk, every GPU concurrently (its own stream)
            with torch.cuda.device(p["dev"]), torch.cuda.stream(p["stream"]):
                p["d"].copy_(src[p["lo"]:p["hi"]], non_blocking=True)
                ms.msort_radix_sort(ms.tensor_ptr(p["d"]), ms.tensor_ptr(p["aux"]), p["hi"] - p["lo"], self.key_type,
                                    ms.tensor_ptr(p["ws"]), p["wsb"], p["stream"])
                p["run"].copy_(p["d"], non_blocking=True)
        for p in self.parts:
            p["stream"].synchronize()
        t1 = time.perf_counter()
        kt = ms.KEY_TYPES[self.key_type]
        rc = self.lib.het_multiway_merge(self.ptrs, self.lens, len(self.parts), ctypes.c_void_p(host_keys.data_ptr()),
                                         kt, self.threads)
        if rc:
            raise RuntimeError("het merge failed")
        t2 = time.perf_counter()
        return {"gpu_sort_and_copies_s": t1 - t0, "cpu_merge_s": t2 - t1, "total_s": t2 - t0,
                "chunks": len(self.parts), "gpus": len(set(str(p["dev"]) for p in self.parts)),
                "threads": self.threads or max_threads()}


def het_sort_host(host_keys, key_type: str, chunks: int = 8, devices: list[int] | None = None, threads: int = 0):
    """One-shot HET sort of the pinned host tensor `host_keys` (allocations included)."""
    return HetSort(host_keys.numel(), key_type, chunks, devices, threads).run(host_keys)
