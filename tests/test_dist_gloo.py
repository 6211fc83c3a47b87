"""Host-side logic of the one-process-per-GPU path, world_size 2 over gloo on CPU:
IPC-handle all-gather in rank order, identical chunking and identical Alg.2
plans on every rank.  (The CUDA calls themselves are covered by test_gpu_dist.py.)"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, out_dir):
    import sys
    sys.path.insert(0, ROOT)
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_sigmod_maltenbergeritr22_b200 import dist as md
    import paper_conf_sigmod_maltenbergeritr22_b200 as m
    local = bytes([rank + 1]) * 7 + bytes(md.MSORT_DIST_HANDLE_BYTES - 7)
    allh = md.exchange_handles(local)
    chunks = [m.msort_plan_chunk(1_000_003, world, r) for r in range(world)]
    c = chunks[0][0]
    plans = []
    for s in range(m.msort_plan_num_stages(world)):
        label = m.msort_plan_stage(world, s)
        piv = [(s * 7919 + j * 104729) % (c * label // 2 + 1) for j in range(world // label)]
        plans.append(m.msort_plan_exchange(world, s, c, piv))
    no_gpu_error = None
    if not torch.cuda.is_available():
        try:
            md.dist_context(rank, world, 0, 1000, "u32")
        except m.MsortError as e:
            no_gpu_error = e.status
    np.save(os.path.join(out_dir, f"r{rank}.npy"), np.frombuffer(allh, dtype=np.uint8))
    with open(os.path.join(out_dir, f"r{rank}.txt"), "w") as f:
        f.write(repr((c, chunks, plans, no_gpu_error)))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 4])
def test_dist_host_logic_gloo(tmp_path, world):
    mp.spawn(_worker, args=(world, _free_port(), str(tmp_path)), nprocs=world, join=True)
    from paper_conf_sigmod_maltenbergeritr22_b200 import dist as md
    ref = None
    for r in range(world):
        h = np.load(tmp_path / f"r{r}.npy").tobytes()
        assert len(h) == world * md.MSORT_DIST_HANDLE_BYTES
        for q in range(world):
            blk = h[q * md.MSORT_DIST_HANDLE_BYTES:(q + 1) * md.MSORT_DIST_HANDLE_BYTES]
            assert blk[:7] == bytes([q + 1]) * 7       # rank order preserved
        txt = (tmp_path / f"r{r}.txt").read_text()
        body = txt.rsplit(",", 1)[0]                    # everything but the error status
        if ref is None:
            ref = body
        assert body == ref                              # every rank derives the same chunking and plans
        if not torch.cuda.is_available():
            assert txt.rstrip(")").endswith("2")        # MSORT_ERR_DEVICE, no CPU fallback


def test_chunking_covers_input():
    """msort_plan_chunk (the library's chunking rule, include/msort.h) against the
    oracle's reading Q3 (oracle.p2p.chunk_size): equal chunks of c keys, c a
    multiple of 4, consecutive slices covering the n keys exactly once."""
    import paper_conf_sigmod_maltenbergeritr22_b200 as m
    from oracle import p2p
    for n in (0, 1, 7, 8, 9, 1000, 65_537, 4_000_000_000, (1 << 32) + 3):
        for g in (1, 2, 4, 8):
            seen = 0
            for r in range(g):
                c, off, valid = m.msort_plan_chunk(n, g, r)
                assert c == p2p.chunk_size(n, g) and c % 4 == 0 and c * g >= n
                assert off == min(n, r * c) and 0 <= valid <= c
                if valid:
                    assert off == seen
                seen += valid
            assert seen == n
    with pytest.raises(m.MsortError):
        m.msort_plan_chunk(10, 3, 0)
    with pytest.raises(m.MsortError):
        m.msort_plan_chunk(10, 2, 2)
