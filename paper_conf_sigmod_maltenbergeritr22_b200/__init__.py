"""Python binding of libmsort (the B200-native multi-GPU P2P sort).

Argument marshalling only: every step of the sort runs in the CUDA kernels of
libmsort.so (csrc/).  There is no CPU fallback; importing this package fails
loudly if the shared library is missing (run __graft_entry__.build() or
`python paper_conf_sigmod_maltenbergeritr22_b200/build.py`).

Function names follow the C ABI in include/msort.h.  Pointers are plain ints
(CUDA device addresses or host addresses); `tensor_ptr` / `key_type_of` help
callers that hold torch tensors (torch is plumbing: memory and streams).
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libmsort.so")

if not os.path.exists(LIB_PATH):
    raise ImportError(f"libmsort.so not built at {LIB_PATH}; run __graft_entry__.build() (no CPU fallback exists)")

_lib = ctypes.CDLL(LIB_PATH)

MSORT_U32, MSORT_U64, MSORT_F32, MSORT_F64 = 0, 1, 2, 3
KEY_TYPES = {"u32": MSORT_U32, "u64": MSORT_U64, "f32": MSORT_F32, "f64": MSORT_F64}
KEY_BYTES = {0: 4, 1: 8, 2: 4, 3: 8}
MSORT_MAX_GPUS = 8
MSORT_MAX_STAGES = 7
MSORT_DIST_HANDLE_BYTES = 512
MSORT_OPT_TIMING, MSORT_OPT_EXCHANGE, MSORT_OPT_SKIP_TRIVIAL, MSORT_OPT_HOST_PIPELINE, MSORT_OPT_SMALL_GRAPH = 0, 1, 2, 3, 4
MSORT_OPT_RADIX_EPOCH, MSORT_OPT_STOP_AFTER_STAGE = 100, 101  # testing only
EXCHANGE_FUSED, EXCHANGE_SWAP, EXCHANGE_ALLTOALL, EXCHANGE_ALLTOALL_PULL, EXCHANGE_NCCL = 0, 1, 2, 3, 4
MSORT_NCCL_ID_BYTES = 128
MSORT_PASS_ENCODE_IN, MSORT_PASS_DECODE_OUT = 1, 2

STATUS = {0: "MSORT_OK", 1: "MSORT_ERR_INVALID_ARGUMENT", 2: "MSORT_ERR_DEVICE", 3: "MSORT_ERR_OUT_OF_MEMORY",
          4: "MSORT_ERR_CUDA", 5: "MSORT_ERR_NCCL", 6: "MSORT_ERR_INTERNAL", 7: "MSORT_ERR_TIMEOUT"}

EXPORTED = [
    "msort_sort", "msort_create", "msort_destroy", "msort_set_option", "msort_sort_host", "msort_sort_device",
    "msort_get_timings", "msort_status_string", "msort_last_error", "msort_version", "msort_rank_mode",
    "msort_radix_workspace_bytes", "msort_step_histogram", "msort_step_radix_pass", "msort_radix_sort",
    "msort_step_pivot", "msort_merge_workspace_bytes", "msort_step_merge", "msort_step_splitters",
    "msort_plan_num_stages", "msort_plan_stage", "msort_plan_exchange",
    "msort_dist_create", "msort_dist_export", "msort_dist_import", "msort_dist_sort", "msort_dist_sort_host",
    "msort_plan_chunk", "msort_release_cached", "msort_measure_links", "msort_nccl_unique_id",
    "msort_dist_nccl_init",
]


class msort_timings(ctypes.Structure):
    _fields_ = [
        ("h2d_ms", ctypes.c_double), ("sort_ms", ctypes.c_double), ("merge_ms", ctypes.c_double),
        ("d2h_ms", ctypes.c_double), ("total_ms", ctypes.c_double), ("hist_ms", ctypes.c_double),
        ("pass_ms_sum", ctypes.c_double), ("passes_run", ctypes.c_int), ("passes_total", ctypes.c_int),
        ("n_gpus", ctypes.c_int), ("n_stages", ctypes.c_int), ("keys_per_gpu", ctypes.c_uint64),
        ("stage_label", ctypes.c_int * MSORT_MAX_STAGES),
        ("stage_pivot", (ctypes.c_uint64 * (MSORT_MAX_GPUS // 2)) * MSORT_MAX_STAGES),
        ("stage_max_x", ctypes.c_uint64 * MSORT_MAX_STAGES),
        ("stage_keys_exchanged", ctypes.c_uint64 * MSORT_MAX_STAGES),
        ("stage_ms", ctypes.c_double * MSORT_MAX_STAGES),
        ("stage_exchange_ms", ctypes.c_double * MSORT_MAX_STAGES),
        ("kernel_launches", ctypes.c_int), ("exchange_mode", ctypes.c_int), ("peer_bulk_ok", ctypes.c_int),
        ("stage_swap_ms", ctypes.c_double * MSORT_MAX_STAGES),
        ("stage_pivot_ms", ctypes.c_double * MSORT_MAX_STAGES),
    ]

    def as_dict(self) -> dict:
        S = self.n_stages
        return {
            "h2d_ms": self.h2d_ms, "sort_ms": self.sort_ms, "merge_ms": self.merge_ms, "d2h_ms": self.d2h_ms,
            "total_ms": self.total_ms, "hist_ms": self.hist_ms, "pass_ms_sum": self.pass_ms_sum,
            "passes_run": self.passes_run, "passes_total": self.passes_total, "n_gpus": self.n_gpus,
            "n_stages": S, "keys_per_gpu": self.keys_per_gpu,
            "stage_label": list(self.stage_label[:S]),
            "stage_pivot": [list(self.stage_pivot[s][: max(1, self.n_gpus // max(1, self.stage_label[s]))]) for s in range(S)],
            "stage_max_x": list(self.stage_max_x[:S]),
            "stage_keys_exchanged": list(self.stage_keys_exchanged[:S]),
            "stage_ms": list(self.stage_ms[:S]),
            "stage_exchange_ms": list(self.stage_exchange_ms[:S]),
            "kernel_launches": self.kernel_launches, "exchange_mode": self.exchange_mode,
            "peer_bulk_ok": self.peer_bulk_ok, "stage_swap_ms": list(self.stage_swap_ms[:S]),
            "stage_pivot_ms": list(self.stage_pivot_ms[:S]),
        }


class msort_link_peaks(ctypes.Structure):
    _fields_ = [("p2p_ce_gbs", ctypes.c_double), ("p2p_sm_gbs", ctypes.c_double), ("h2d_gbs", ctypes.c_double),
                ("d2h_gbs", ctypes.c_double), ("bidir_gbs", ctypes.c_double), ("bytes", ctypes.c_uint64),
                ("pairs", ctypes.c_int), ("same_device", ctypes.c_int)]

    def as_dict(self) -> dict:
        return {k: getattr(self, k) for k, _ in self._fields_}


_P = ctypes.c_void_p
_U64 = ctypes.c_uint64
_I = ctypes.c_int


def _sig(name, res, *args):
    f = getattr(_lib, name)
    f.restype = res
    f.argtypes = list(args)
    return f


_sig("msort_sort", _I, _P, _U64, _I, _I, _P)
_sig("msort_create", _I, ctypes.POINTER(_P), _I, ctypes.POINTER(_I), _U64, _I)
_sig("msort_destroy", _I, _P)
_sig("msort_set_option", _I, _P, _I, ctypes.c_int64)
_sig("msort_sort_host", _I, _P, _P, _U64)
_sig("msort_sort_device", _I, _P, ctypes.POINTER(_P), _U64, ctypes.POINTER(_P))
_sig("msort_get_timings", _I, _P, ctypes.POINTER(msort_timings))
_sig("msort_status_string", ctypes.c_char_p, _I)
_sig("msort_last_error", ctypes.c_char_p)
_sig("msort_version", _I)
_sig("msort_rank_mode", _I, _I)
_sig("msort_radix_workspace_bytes", _U64, _U64, _I)
_sig("msort_step_histogram", _I, _P, _U64, _I, _P, _P)
_sig("msort_step_radix_pass", _I, _P, _P, _U64, _I, _I, _P, _I, _P, _U64, _P)
_sig("msort_radix_sort", _I, _P, _P, _U64, _I, _P, _U64, _P)
_sig("msort_step_pivot", _I, ctypes.POINTER(_P), _I, _U64, _I, _P, _P)
_sig("msort_merge_workspace_bytes", _U64, _U64, _I)
_sig("msort_step_merge", _I, _P, _U64, _P, _U64, _P, _I, _P, _U64, _P)
_sig("msort_step_splitters", _I, ctypes.POINTER(_P), _I, _U64, _I, _P, _P)
_sig("msort_plan_num_stages", _I, _I)
_sig("msort_plan_stage", _I, _I, _I, ctypes.POINTER(_I))
_sig("msort_plan_exchange", _I, _I, _I, _U64, ctypes.POINTER(_U64), ctypes.POINTER(_I), ctypes.POINTER(_U64),
     ctypes.POINTER(_I))
_sig("msort_dist_create", _I, ctypes.POINTER(_P), _I, _I, _I, _U64, _I)
_sig("msort_dist_export", _I, _P, _P)
_sig("msort_dist_import", _I, _P, _P)
_sig("msort_dist_sort", _I, _P, _P, _U64, _P)
_sig("msort_dist_sort_host", _I, _P, _P, _U64)
_sig("msort_plan_chunk", _I, _U64, _I, _I, ctypes.POINTER(_U64), ctypes.POINTER(_U64), ctypes.POINTER(_U64))
_sig("msort_release_cached", _I)
_sig("msort_measure_links", _I, _P, _U64, _I, ctypes.POINTER(msort_link_peaks))
_sig("msort_nccl_unique_id", _I, _P)
_sig("msort_dist_nccl_init", _I, _P, _P)


class MsortError(RuntimeError):
    def __init__(self, where: str, status: int):
        self.status = status
        detail = (_lib.msort_last_error() or b"").decode(errors="replace")
        super().__init__(f"{where}: {STATUS.get(status, status)}: {detail}")


def _check(where: str, status: int) -> None:
    if status != 0:
        raise MsortError(where, status)


def _kt(key_type) -> int:
    return KEY_TYPES[key_type] if isinstance(key_type, str) else int(key_type)


# --- torch plumbing helpers (no compute) ------------------------------------

def key_type_of(t) -> int:
    """msort key type of a tensor's dtype.  Only unsigned integers and IEEE floats
    are key types (include/msort.h; reading Q2): a signed tensor would
    sort its negative values after the positive ones, so it is rejected."""
    import torch
    m = {torch.uint32: 0, torch.uint64: 1, torch.float32: 2, torch.float64: 3}
    if t.dtype not in m:
        raise TypeError(f"msort sorts uint32/uint64/float32/float64 keys, not {t.dtype} "
                        "(signed integers would order negatives after positives)")
    return m[t.dtype]


def tensor_ptr(t) -> int:
    return int(t.data_ptr())


def stream_ptr(stream) -> int:
    if stream is None:
        return 0
    return int(getattr(stream, "cuda_stream", stream))


# --- C ABI wrappers (same names) ---------------------------------------------

def msort_sort(keys: int, n: int, key_type, n_gpus: int = 1, stream=None) -> None:
    _check("msort_sort", _lib.msort_sort(keys, n, _kt(key_type), n_gpus, stream_ptr(stream)))


def msort_version() -> int:
    return _lib.msort_version()


def msort_rank_mode(device: int = 0) -> int:
    return _lib.msort_rank_mode(device)


def msort_radix_workspace_bytes(n: int, key_type) -> int:
    return int(_lib.msort_radix_workspace_bytes(n, _kt(key_type)))


def msort_merge_workspace_bytes(total: int, key_type) -> int:
    return int(_lib.msort_merge_workspace_bytes(total, _kt(key_type)))


def msort_step_histogram(d_keys: int, n: int, key_type, d_hist: int, stream=None) -> None:
    _check("msort_step_histogram", _lib.msort_step_histogram(d_keys, n, _kt(key_type), d_hist, stream_ptr(stream)))


def msort_step_radix_pass(d_in: int, d_out: int, n: int, key_type, pass_: int, d_hist: int, flags: int,
                          d_ws: int, ws_bytes: int, stream=None) -> None:
    _check("msort_step_radix_pass", _lib.msort_step_radix_pass(d_in, d_out, n, _kt(key_type), pass_, d_hist, flags,
                                                                d_ws, ws_bytes, stream_ptr(stream)))


def msort_radix_sort(d_keys: int, d_aux: int, n: int, key_type, d_ws: int, ws_bytes: int, stream=None) -> None:
    _check("msort_radix_sort", _lib.msort_radix_sort(d_keys, d_aux, n, _kt(key_type), d_ws, ws_bytes, stream_ptr(stream)))


def msort_step_pivot(d_chunks: list[int], c: int, key_type, d_pivot: int, stream=None) -> None:
    arr = (_P * len(d_chunks))(*d_chunks)
    _check("msort_step_pivot", _lib.msort_step_pivot(arr, len(d_chunks), c, _kt(key_type), d_pivot, stream_ptr(stream)))


def msort_step_merge(d_a: int, a_len: int, d_b: int, b_len: int, d_out: int, key_type, d_ws: int, ws_bytes: int,
                     stream=None) -> None:
    _check("msort_step_merge", _lib.msort_step_merge(d_a, a_len, d_b, b_len, d_out, _kt(key_type), d_ws, ws_bytes,
                                                     stream_ptr(stream)))


def msort_step_splitters(d_chunks: list[int], c: int, key_type, d_s: int, stream=None) -> None:
    arr = (_P * len(d_chunks))(*d_chunks)
    _check("msort_step_splitters", _lib.msort_step_splitters(arr, len(d_chunks), c, _kt(key_type), d_s,
                                                             stream_ptr(stream)))


def msort_plan_num_stages(g: int) -> int:
    return _lib.msort_plan_num_stages(g)


def msort_plan_stage(g: int, s: int) -> int:
    lab = _I(0)
    _check("msort_plan_stage", _lib.msort_plan_stage(g, s, ctypes.byref(lab)))
    return lab.value


def msort_plan_exchange(g: int, s: int, c: int, pivots: list[int]):
    piv = (_U64 * max(1, len(pivots)))(*pivots)
    partner = (_I * g)()
    x = (_U64 * g)()
    side = (_I * g)()
    _check("msort_plan_exchange", _lib.msort_plan_exchange(g, s, c, piv, partner, x, side))
    return list(partner), list(x), list(side)


def msort_plan_chunk(n: int, g: int, rank: int) -> tuple[int, int, int]:
    """(c, offset, valid) of `rank` for n keys on g GPUs (include/msort.h)."""
    c, off, val = _U64(), _U64(), _U64()
    _check("msort_plan_chunk", _lib.msort_plan_chunk(n, g, rank, ctypes.byref(c), ctypes.byref(off), ctypes.byref(val)))
    return c.value, off.value, val.value


def msort_nccl_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(MSORT_NCCL_ID_BYTES)
    _check("msort_nccl_unique_id", _lib.msort_nccl_unique_id(buf))
    return buf.raw


def msort_release_cached() -> None:
    _check("msort_release_cached", _lib.msort_release_cached())


class Context:
    """msort_ctx: pre-allocated buffers/streams/events for g chunks (single process)."""

    def __init__(self, n_gpus: int, max_keys: int, key_type, device_ids: list[int] | None = None):
        self.n_gpus = n_gpus
        self.key_type = _kt(key_type)
        h = _P()
        ids = (_I * n_gpus)(*device_ids) if device_ids is not None else None
        _check("msort_create", _lib.msort_create(ctypes.byref(h), n_gpus, ids, max_keys, self.key_type))
        self._h = h

    def set_option(self, option: int, value: int) -> None:
        _check("msort_set_option", _lib.msort_set_option(self._h, option, value))

    def sort_host(self, host_ptr: int, n: int) -> None:
        _check("msort_sort_host", _lib.msort_sort_host(self._h, host_ptr, n))

    def sort_device(self, chunk_ptrs: list[int], keys_per_gpu: int, streams: list | None = None) -> None:
        arr = (_P * self.n_gpus)(*chunk_ptrs)
        sts = (_P * self.n_gpus)(*[stream_ptr(s) for s in streams]) if streams else None
        _check("msort_sort_device", _lib.msort_sort_device(self._h, arr, keys_per_gpu, sts))

    def timings(self) -> dict:
        t = msort_timings()
        _check("msort_get_timings", _lib.msort_get_timings(self._h, ctypes.byref(t)))
        return t.as_dict()

    def measure_links(self, nbytes: int, reps: int = 3) -> dict:
        pk = msort_link_peaks()
        _check("msort_measure_links", _lib.msort_measure_links(self._h, nbytes, reps, ctypes.byref(pk)))
        return pk.as_dict()

    def close(self) -> None:
        if getattr(self, "_h", None):
            _lib.msort_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class DistContext:
    """One process per GPU: msort_dist_create / export / import / sort."""

    def __init__(self, rank: int, world: int, device: int, max_keys_per_rank: int, key_type):
        self.rank, self.world, self.key_type = rank, world, _kt(key_type)
        h = _P()
        _check("msort_dist_create", _lib.msort_dist_create(ctypes.byref(h), rank, world, device, max_keys_per_rank,
                                                           self.key_type))
        self._h = h

    def export_handle(self) -> bytes:
        buf = ctypes.create_string_buffer(MSORT_DIST_HANDLE_BYTES)
        _check("msort_dist_export", _lib.msort_dist_export(self._h, buf))
        return buf.raw

    def import_handles(self, all_handles: bytes) -> None:
        if len(all_handles) != self.world * MSORT_DIST_HANDLE_BYTES:
            raise ValueError("need world * MSORT_DIST_HANDLE_BYTES bytes")
        buf = ctypes.create_string_buffer(all_handles, len(all_handles))
        _check("msort_dist_import", _lib.msort_dist_import(self._h, buf))

    def set_option(self, option: int, value: int) -> None:
        _check("msort_set_option", _lib.msort_set_option(self._h, option, value))

    def nccl_init(self, unique_id: bytes) -> None:
        """Join the NCCL communicator of all ranks (exchange mode 4); unique_id from rank 0."""
        if len(unique_id) != MSORT_NCCL_ID_BYTES:
            raise ValueError("need MSORT_NCCL_ID_BYTES bytes")
        buf = ctypes.create_string_buffer(unique_id, len(unique_id))
        _check("msort_dist_nccl_init", _lib.msort_dist_nccl_init(self._h, buf))

    def sort(self, d_chunk: int, n_total: int, stream=None) -> None:
        """d_chunk holds this rank's `valid` keys of the n_total (msort_plan_chunk)."""
        _check("msort_dist_sort", _lib.msort_dist_sort(self._h, d_chunk, n_total, stream_ptr(stream)))

    def sort_host(self, host_ptr: int, n_total: int) -> None:
        _check("msort_dist_sort_host", _lib.msort_dist_sort_host(self._h, host_ptr, n_total))

    def timings(self) -> dict:
        t = msort_timings()
        _check("msort_get_timings", _lib.msort_get_timings(self._h, ctypes.byref(t)))
        return t.as_dict()

    def measure_links(self, nbytes: int, reps: int = 3) -> dict:
        """Collective: every rank calls it; this rank's rates."""
        pk = msort_link_peaks()
        _check("msort_measure_links", _lib.msort_measure_links(self._h, nbytes, reps, ctypes.byref(pk)))
        return pk.as_dict()

    def close(self) -> None:
        if getattr(self, "_h", None):
            _lib.msort_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
