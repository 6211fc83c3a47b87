"""One process per rank (msort_dist_*): CUDA-IPC peer mapping, device-side
barriers and the fused peer-read merge, with every rank on cuda:0 (the only
GPU of the test box; IPC works between processes on one device).  Output of
all ranks together must equal the oracle bit for bit."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import msort_inputs as mi
from oracle import codec, sort

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, n, kt, distn, out_dir, host, exchange=0):
    import sys
    sys.path.insert(0, ROOT)
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    os.environ.setdefault("MSORT_BARRIER_TIMEOUT_S", "120")
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import paper_conf_sigmod_maltenbergeritr22_b200 as m
    from paper_conf_sigmod_maltenbergeritr22_b200 import dist as md
    ch = md.chunking(n, world)
    ctx = md.dist_context(rank, world, 0, ch.c, kt)
    ctx.set_option(m.MSORT_OPT_EXCHANGE, exchange)
    a = mi.np_generate(n, kt, distn, seed=5)
    mine = np.full(ch.c, md.PAD_BITS[kt], dtype=codec.UINT[kt])
    v = ch.valid(rank)
    mine[:v] = codec.bits_of(a[ch.offset(rank):ch.offset(rank) + v], kt)
    if host:
        h = torch.from_numpy(mine.view(np.uint8).copy()).pin_memory()
        ctx.sort_host(m.tensor_ptr(h), ch.c)
        res = h.numpy()
    else:
        d = torch.from_numpy(mine.view(np.uint8).copy()).cuda()
        ctx.sort(m.tensor_ptr(d), ch.c)
        torch.cuda.synchronize()
        res = d.cpu().numpy()
    np.save(os.path.join(out_dir, f"r{rank}.npy"), res)
    tm = ctx.timings()
    with open(os.path.join(out_dir, f"t{rank}.txt"), "w") as f:
        f.write(repr(tm["stage_label"]))
    ctx.close()
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,n,kt,distn,host,exchange", [
    (2, 100_003, "u32", "uniform", False, 0),
    (2, 50_000, "f32", "uniform", True, 0),
    (4, 200_001, "u32", "zipf", False, 0),
    (4, 120_000, "u32", "reverse", False, 0),
    (8, 64_003, "u64", "uniform", False, 0),
    (4, 200_001, "u32", "uniform", False, 2),
    (8, 80_000, "f32", "uniform", True, 2),
    (4, 200_001, "u32", "zipf", False, 3),
    (2, 90_001, "u64", "uniform", True, 3),
    # chunks of >= 2^20 keys: msort_dist_sort_host takes the pipelined S0 (pieces sorted as they land)
    (2, 2_500_001, "u32", "uniform", True, 0),
    (4, 4_400_000, "f32", "uniform", True, 2),
    (2, 2_200_002, "u32", "zipf", True, 3),
])
def test_dist_sort_matches_oracle(tmp_path, world, n, kt, distn, host, exchange):
    mp.spawn(_worker, args=(world, _free_port(), n, kt, distn, str(tmp_path), host, exchange), nprocs=world,
             join=True)
    from paper_conf_sigmod_maltenbergeritr22_b200 import dist as md
    ch = md.chunking(n, world)
    out = np.concatenate([np.load(tmp_path / f"r{r}.npy").view(codec.UINT[kt]) for r in range(world)])[:n]
    a = mi.np_generate(n, kt, distn, seed=5)
    assert np.array_equal(out, codec.bits_of(sort.oracle_sort(a, kt), kt))
    labels = eval((tmp_path / "t0.txt").read_text())
    assert len(labels) == (world - 1 if exchange < 2 else 1)
