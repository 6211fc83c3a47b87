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


def _worker(rank, world, port, n, kt, distn, out_dir, host, exchange=0, nccl=False, distinct=False):
    import sys
    sys.path.insert(0, ROOT)
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    os.environ.setdefault("MSORT_BARRIER_TIMEOUT_S", "120")
    dev = rank if distinct else 0
    torch.cuda.set_device(dev)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import paper_conf_sigmod_maltenbergeritr22_b200 as m
    from paper_conf_sigmod_maltenbergeritr22_b200 import dist as md
    c, off, v = m.msort_plan_chunk(n, world, rank)
    try:
        ctx = md.dist_context(rank, world, dev, c, kt, nccl=nccl)
    except m.MsortError as e:
        if nccl and e.status == 5:  # MSORT_ERR_NCCL: e.g. NCCL refuses two ranks on one GPU
            with open(os.path.join(out_dir, f"nccl{rank}.txt"), "w") as f:
                f.write(str(e))
            dist.barrier()
            dist.destroy_process_group()
            return
        raise
    ctx.set_option(m.MSORT_OPT_EXCHANGE, exchange)
    a = mi.np_generate(n, kt, distn, seed=5)
    mine = codec.bits_of(a[off:off + v], kt).copy()   # this rank's slice; the library pads (reading Q3)
    if host == "pageable":  # a plain numpy array: the bounce-buffer path
        h = mine.view(np.uint8).copy()
        ctx.sort_host(h.ctypes.data, n)
        res = h
    elif host:
        h = torch.from_numpy(mine.view(np.uint8).copy()).pin_memory()
        ctx.sort_host(m.tensor_ptr(h), n)
        res = h.numpy()
    else:
        d = torch.zeros(c * mi.KEY_BYTES[kt], dtype=torch.uint8, device=f"cuda:{dev}")
        d[: v * mi.KEY_BYTES[kt]] = torch.from_numpy(mine.view(np.uint8).copy()).to(f"cuda:{dev}")
        ctx.sort(m.tensor_ptr(d), n)
        torch.cuda.synchronize()
        res = d[: v * mi.KEY_BYTES[kt]].cpu().numpy()
    np.save(os.path.join(out_dir, f"r{rank}.npy"), res)
    tm = ctx.timings()
    with open(os.path.join(out_dir, f"t{rank}.txt"), "w") as f:
        f.write(repr((tm["stage_label"], tm["exchange_mode"], tm["peer_bulk_ok"])))
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
    # pageable host keys: bounce buffers, below and above the pipelining threshold
    (2, 60_001, "u64", "uniform", "pageable", 0),
    (2, 2_500_001, "u32", "uniform", "pageable", 0),
])
def test_dist_sort_matches_oracle(tmp_path, world, n, kt, distn, host, exchange):
    mp.spawn(_worker, args=(world, _free_port(), n, kt, distn, str(tmp_path), host, exchange), nprocs=world,
             join=True)
    out = np.concatenate([np.load(tmp_path / f"r{r}.npy").view(codec.UINT[kt]) for r in range(world)])
    assert len(out) == n
    a = mi.np_generate(n, kt, distn, seed=5)
    assert np.array_equal(out, codec.bits_of(sort.oracle_sort(a, kt), kt))
    labels, mode, bulk_ok = eval((tmp_path / "t0.txt").read_text())
    assert len(labels) == (world - 1 if exchange in (0, 1, 4) else 1)
    assert bulk_ok == 1 and mode == exchange   # the peer bulk-copy self-test passed: no fallback


def test_dist_nccl_swap(tmp_path):
    """Exchange mode 4 in dist mode: an NCCL communicator bootstrapped from rank 0's
    unique id (torch.distributed broadcast), grouped ncclSend/ncclRecv per
    mirrored pair.  Two ranks on the test box's one GPU: if NCCL refuses that
    (duplicate GPU), the refusal must come back as MSORT_ERR_NCCL, cleanly."""
    world, n, kt = 2, 100_003, "u32"
    mp.spawn(_worker, args=(world, _free_port(), n, kt, "uniform", str(tmp_path), False, 4, True), nprocs=world,
             join=True)
    refused = [(tmp_path / f"nccl{r}.txt").exists() for r in range(world)]
    if all(refused):
        pytest.skip("NCCL refused two ranks on one GPU: " + (tmp_path / "nccl0.txt").read_text()[:200])
    assert not any(refused)
    out = np.concatenate([np.load(tmp_path / f"r{r}.npy").view(codec.UINT[kt]) for r in range(world)])
    a = mi.np_generate(n, kt, "uniform", seed=5)
    assert np.array_equal(out, codec.bits_of(sort.oracle_sort(a, kt), kt))


def _worker_big(rank, world, port, n, kt, distn, exchange, out_dir):
    """Full-size rank: this rank's chunk of the seeded workload generated on the GPU, sorted through
    msort_dist_sort, summarised by properties that hold at any size (oracle.checks)."""
    import json
    import sys
    sys.path.insert(0, ROOT)
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    os.environ.setdefault("MSORT_BARRIER_TIMEOUT_S", "300")
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import paper_conf_sigmod_maltenbergeritr22_b200 as m
    from paper_conf_sigmod_maltenbergeritr22_b200 import dist as md
    from oracle import checks
    c, off, v = m.msort_plan_chunk(n, world, rank)
    t = torch.empty(c, dtype=mi.torch_dtype(kt), device="cuda")
    mi.t_generate_into(t[:v], n, kt, distn, seed=9, start=off, block=1 << 27)
    blk = 1 << 26

    def fp(x, lim):
        f = [0, 0, 0]
        for off in range(0, lim, blk):
            a, b, cc = checks.fingerprint(x[off:min(off + blk, lim)].cpu().numpy(), kt)
            f = [f[0] + a, (f[1] + b) % (1 << 64), f[2] ^ cc]
        return f
    fp_in = fp(t, v)
    ctx = md.dist_context(rank, world, 0, c, kt)
    ctx.set_option(m.MSORT_OPT_EXCHANGE, exchange)
    ctx.sort(m.tensor_ptr(t), n)
    torch.cuda.synchronize()
    keep = v  # this rank's sorted keys: global ranks [off, off + v)
    ok, first, last = True, None, None
    for off in range(0, keep, blk):
        codes = codec.encode(t[off:min(off + blk, keep)].cpu().numpy(), kt)
        ok &= checks.is_sorted_codes(codes)
        ok &= last is None or int(last) <= int(codes[0])
        first = int(codes[0]) if first is None else first
        last = int(codes[-1])
    res = {"fp_in": fp_in, "fp_out": fp(t, keep), "sorted": bool(ok), "first": first, "last": last}
    with open(os.path.join(out_dir, f"big{rank}.json"), "w") as f:
        json.dump(res, f)
    ctx.close()
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,n,kt,distn,exchange", [
    (4, 1_000_000_003, "u32", "uniform", 2),   # bench.py's N > 1 path (NEXT-1 fused), ranks sharing one GPU
    (2, 1_000_000_000, "u32", "zipf", 0),      # the paper's Alg.2 with the fused peer-read merge
])
def test_dist_sort_full_size(tmp_path, world, n, kt, distn, exchange):
    """One process per rank at full size: every rank's output non-decreasing, rank boundaries ordered, and the
    union a permutation of the input (fingerprints) - together equality with the unique sorted result
    (oracle/checks.py)."""
    import json
    mp.spawn(_worker_big, args=(world, _free_port(), n, kt, distn, exchange, str(tmp_path)), nprocs=world, join=True)
    rs = [json.loads((tmp_path / f"big{r}.json").read_text()) for r in range(world)]
    assert all(r["sorted"] for r in rs)
    for a, b in zip(rs, rs[1:]):
        if a["last"] is not None and b["first"] is not None:
            assert a["last"] <= b["first"]

    def tot(k):
        f = [0, 0, 0]
        for r in rs:
            f = [f[0] + r[k][0], (f[1] + r[k][1]) % (1 << 64), f[2] ^ r[k][2]]
        return f
    assert tot("fp_in") == tot("fp_out") and tot("fp_in")[0] == n


@pytest.mark.parametrize("exchange", [0, 2, 4])
def test_dist_sort_distinct_gpus(tmp_path, exchange):
    """One process per GPU on distinct GPUs (skipped on one-GPU boxes): IPC over NVLink, device barriers,
    the NCCL communicator of mode 4 - equal to the oracle."""
    world = min(torch.cuda.device_count(), 8)
    world = 1 << (world.bit_length() - 1) if world else 0
    if world < 2:
        pytest.skip("needs 2 or more GPUs")
    n, kt = 1_000_003, "u32"
    mp.spawn(_worker, args=(world, _free_port(), n, kt, "uniform", str(tmp_path), False, exchange, exchange == 4, True),
             nprocs=world, join=True)
    out = np.concatenate([np.load(tmp_path / f"r{r}.npy").view(codec.UINT[kt]) for r in range(world)])
    a = mi.np_generate(n, kt, "uniform", seed=5)
    assert np.array_equal(out, codec.bits_of(sort.oracle_sort(a, kt), kt))
    labels, mode, bulk_ok = eval((tmp_path / "t0.txt").read_text())
    assert bulk_ok == 1 and mode == exchange


def _worker_soak(rank, world, port, out_dir, iters):
    """Many back-to-back dist sorts of random sizes, distributions and exchange modes in ONE context per
    rank: the device barriers (release/acquire on IPC-mapped flags), the epoch-tagged look-back and the
    device-resident stages under repeated reuse of the same buffers."""
    import sys
    sys.path.insert(0, ROOT)
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    os.environ.setdefault("MSORT_BARRIER_TIMEOUT_S", "120")
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import paper_conf_sigmod_maltenbergeritr22_b200 as m
    from paper_conf_sigmod_maltenbergeritr22_b200 import dist as md
    cap = 1 << 19
    ctx = md.dist_context(rank, world, 0, cap, "u32")
    rng = np.random.default_rng(77)          # the same sequence on every rank
    bad = []
    for it in range(iters):
        n = int(rng.integers(world, world * cap))
        distn = ["uniform", "zipf", "reverse", "sorted", "nearly"][int(rng.integers(0, 5))]
        ex = [0, 1, 2, 3][int(rng.integers(0, 4))]
        ctx.set_option(m.MSORT_OPT_EXCHANGE, ex)
        c, off, v = m.msort_plan_chunk(n, world, rank)
        a = mi.np_generate(n, "u32", distn, seed=it)
        d = torch.zeros(c, dtype=torch.int32, device="cuda")
        d[:v] = torch.from_numpy(a[off:off + v].view(np.int32).copy()).cuda()
        ctx.sort(m.tensor_ptr(d), n)
        torch.cuda.synchronize()
        want = sort.oracle_sort(a, "u32")[off:off + v]
        if not np.array_equal(d[:v].cpu().numpy().view(np.uint32), want):
            bad.append((it, n, distn, ex))
    with open(os.path.join(out_dir, f"soak{rank}.txt"), "w") as f:
        f.write(repr(bad))
    ctx.close()
    dist.barrier()
    dist.destroy_process_group()


def test_dist_soak(tmp_path):
    world, iters = 4, 40
    mp.spawn(_worker_soak, args=(world, _free_port(), str(tmp_path), iters), nprocs=world, join=True)
    for r in range(world):
        assert (tmp_path / f"soak{r}.txt").read_text() == "[]", r
