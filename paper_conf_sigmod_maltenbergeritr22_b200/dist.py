"""One-process-per-GPU plumbing for msort (torch.distributed only moves the
opaque IPC handle bytes; every step of the sort runs in libmsort's kernels).

    ctx = dist_context(rank, world, device, max_keys_per_rank, "u32")
    ctx.sort(d_chunk_ptr, c)          # rank r ends with global ranks [r*c, (r+1)*c)

The chunking rule is the paper's (equal chunks) with DESIGN.md
reading Q3 (c rounded up to a multiple of 4, the tail padded with the largest
key under the T order).
"""
from __future__ import annotations

from dataclasses import dataclass

MSORT_DIST_HANDLE_BYTES = 512
PAD_BITS = {"u32": 0xFFFFFFFF, "u64": 0xFFFFFFFFFFFFFFFF, "f32": 0x7FFFFFFF, "f64": 0x7FFFFFFFFFFFFFFF}


@dataclass(frozen=True)
class Chunking:
    n: int           # total keys
    world: int       # GPUs
    c: int           # keys per GPU (padded)

    def valid(self, rank: int) -> int:
        """Real (unpadded) keys held by `rank`."""
        return max(0, min(self.n - rank * self.c, self.c))

    def offset(self, rank: int) -> int:
        return rank * self.c


def chunking(n: int, world: int) -> Chunking:
    c = -(-n // world) if world else 0
    return Chunking(n, world, (c + 3) // 4 * 4)


def exchange_handles(local: bytes, group=None) -> bytes:
    """All-gather every rank's handle bytes in rank order (any torch.distributed backend)."""
    import torch.distributed as dist
    if len(local) != MSORT_DIST_HANDLE_BYTES:
        raise ValueError("handle must be MSORT_DIST_HANDLE_BYTES long")
    world = dist.get_world_size(group)
    out = [None] * world
    dist.all_gather_object(out, local, group=group)
    if any(len(x) != MSORT_DIST_HANDLE_BYTES for x in out):
        raise RuntimeError("malformed handle from a peer")
    return b"".join(out)


def dist_context(rank: int, world: int, device: int, max_keys_per_rank: int, key_type, group=None):
    """Create this rank's msort context and map every peer's buffers."""
    from . import DistContext
    ctx = DistContext(rank, world, device, max_keys_per_rank, key_type)
    ctx.import_handles(exchange_handles(ctx.export_handle(), group))
    return ctx
