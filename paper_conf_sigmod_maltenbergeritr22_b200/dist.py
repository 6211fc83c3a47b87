"""One-process-per-GPU plumbing for msort (torch.distributed only moves the
opaque IPC handle bytes; every step of the sort runs in libmsort's kernels).

    c, off, valid = msort_plan_chunk(n, world, rank)     # the library's chunking rule
    ctx = dist_context(rank, world, device, c, "u32")
    ctx.sort(d_chunk_ptr, n)      # d_chunk: this rank's `valid` keys (room for c)

The chunking rule (equal chunks, reading Q3) and the
tail padding live in libmsort (msort_plan_chunk, msort_dist_sort).
"""
from __future__ import annotations

MSORT_DIST_HANDLE_BYTES = 512


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


def dist_context(rank: int, world: int, device: int, max_keys_per_rank: int, key_type, group=None,
                 nccl: bool = False):
    """Create this rank's msort context and map every peer's buffers; with
    nccl=True also join an NCCL communicator of all ranks (exchange mode 4),
    bootstrapped from an id rank 0 broadcasts over torch.distributed."""
    import torch.distributed as dist

    from . import DistContext, msort_nccl_unique_id
    ctx = DistContext(rank, world, device, max_keys_per_rank, key_type)
    ctx.import_handles(exchange_handles(ctx.export_handle(), group))
    if nccl:
        obj = [msort_nccl_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0, group=group)
        ctx.nccl_init(obj[0])
    return ctx
