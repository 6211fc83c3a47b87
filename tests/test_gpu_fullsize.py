"""Parity at BASELINE.json's full sizes, in the launch configurations bench.py
times, checked by the oracle's any-size properties (oracle/checks.py):
non-decreasing under T, a permutation of the input (multiset fingerprint), and
sampled outputs equal to the oracle's order statistics computed one by one.
Together these imply byte equality with the (unique) oracle result.

configs[2]: 4e9 uniform u32 on one GPU (the bench's N=1 workload); configs[4]'s u64 / f32 at 2e9 on one GPU;
configs[1]: 2^28 uniform u32 on 2 chunks (virtual ranks on one GPU);
configs[3]/[4]: 2e9 keys on 8 chunks (virtual ranks): zipf / reverse / nearly-sorted / sorted / normal
u32, f32, u64, NEXT-1 on zipf, and the NCCL swap (mode 4) on reverse.
"""
import os

import numpy as np
import pytest
import torch

import msort_inputs as mi
from oracle import checks, codec

pytestmark = [pytest.mark.gpu, pytest.mark.slow]

BLOCK = 1 << 27


def _gen_chunks(n, g, kt, dist, seed):
    c = n // g
    chunks = [torch.empty(c, dtype=mi.torch_dtype(kt), device="cuda") for _ in range(g)]
    for i in range(g):
        mi.t_generate_into(chunks[i], n, kt, dist, seed=seed, start=i * c, block=BLOCK)
    return chunks, c


def _host_blocks(chunks):
    for ch in chunks:
        for off in range(0, ch.numel(), BLOCK):
            yield ch[off:off + BLOCK].cpu().numpy()


def _block_stats(blk, kt, sv):
    """Per-block oracle work (numpy releases the GIL: blocks run on a thread pool)."""
    t = codec.encode(blk, kt)
    m = len(sv)
    lt = np.cumsum(np.bincount(np.searchsorted(sv, t, side="right"), minlength=m + 1))[:m]
    le = np.cumsum(np.bincount(np.searchsorted(sv, t, side="left"), minlength=m + 1))[:m]
    return checks.fingerprint(blk, kt), lt, le


def _out_stats(blk, kt):
    t = codec.encode(blk, kt)
    return checks.is_sorted_codes(t), t[0], t[-1], checks.fingerprint(blk, kt)


def _fp_add(a, f):
    return [a[0] + f[0], (a[1] + f[1]) % (1 << 64), a[2] ^ f[2]]


def _check(out_chunks, n, kt, dist, seed, nsamples=24):
    from concurrent.futures import ThreadPoolExecutor
    rng = np.random.default_rng(seed)
    ranks = np.sort(rng.choice(n, size=nsamples, replace=False))
    ranks[0], ranks[-1] = 0, n - 1
    pool = ThreadPoolExecutor(max_workers=min(16, (os.cpu_count() or 4)))
    # output: sortedness (within and across blocks), fingerprint, sampled values
    futs, samples, pos = [], {}, 0
    for blk in _host_blocks(out_chunks):
        futs.append(pool.submit(_out_stats, blk, kt))
        for r in ranks[(ranks >= pos) & (ranks < pos + len(blk))]:
            samples[int(r)] = blk[int(r) - pos]
        pos += len(blk)
    assert pos == n
    fp_out, prev = [0, 0, 0], None
    for i, f in enumerate(futs):
        ok, first, last, fp = f.result()
        assert ok, f"not sorted inside output block {i}"
        assert prev is None or prev <= first, f"not sorted across output blocks at {i}"
        prev = last
        fp_out = _fp_add(fp_out, fp)
    # input: fingerprint and order statistics of the sampled outputs, block by block
    sv = codec.encode(np.array([samples[int(r)] for r in ranks], dtype=mi.NP_DTYPE[kt]), kt)
    futs = []
    tmp = torch.empty(BLOCK, dtype=mi.torch_dtype(kt), device="cuda")
    for off in range(0, n, BLOCK):
        cnt = min(BLOCK, n - off)
        mi.t_generate_into(tmp[:cnt], n, kt, dist, seed=seed, start=off, block=BLOCK)
        futs.append(pool.submit(_block_stats, tmp[:cnt].cpu().numpy(), kt, sv))
    fp_in = [0, 0, 0]
    lt = np.zeros(len(ranks), dtype=np.int64)
    le = np.zeros(len(ranks), dtype=np.int64)
    for f in futs:
        fp, a, b = f.result()
        fp_in = _fp_add(fp_in, fp)
        lt += a
        le += b
    pool.shutdown()
    assert fp_in == fp_out, "output is not a permutation of the input"
    assert np.all((lt <= ranks) & (ranks < le)), "a sampled output differs from the oracle's order statistic"


def test_config3_4e9_u32_one_gpu():
    import paper_conf_sigmod_maltenbergeritr22_b200 as ms
    n = 4_000_000_000
    chunks, c = _gen_chunks(n, 1, "u32", "uniform", 1)
    ctx = ms.Context(1, n, "u32", device_ids=[0])
    ctx.sort_device([ms.tensor_ptr(chunks[0])], c)
    torch.cuda.synchronize()
    ctx.close()
    _check(chunks, n, "u32", "uniform", 1)


@pytest.mark.parametrize("kt", ["u64", "f32"])
def test_config4_2e9_one_gpu(kt):
    """configs[4]'s key types as bench.py times them at N = 1 (2e9 keys in one chunk: 8-byte keys with the
    7680-key tiles of 512 threads, float keys with the codec fused into the first / last pass)."""
    import paper_conf_sigmod_maltenbergeritr22_b200 as ms
    n = 2_000_000_000
    chunks, c = _gen_chunks(n, 1, kt, "uniform", 5)
    ctx = ms.Context(1, n, kt, device_ids=[0])
    ctx.sort_device([ms.tensor_ptr(chunks[0])], c)
    torch.cuda.synchronize()
    ctx.close()
    _check(chunks, n, kt, "uniform", 5)


def test_max_chunk_u32_one_gpu():
    """The largest chunk the 32-bit per-chunk indexing contract allows (include/msort.h: keys per GPU < 2^32,
    rounded to a multiple of 4, reading Q3): n = 2^32 - 4 uint32 keys on one GPU, sorted device-resident and
    checked like configs[2]; one key more per GPU is refused with MSORT_ERR_INVALID_ARGUMENT, not truncated."""
    import paper_conf_sigmod_maltenbergeritr22_b200 as ms
    n = (1 << 32) - 4
    chunks, c = _gen_chunks(n, 1, "u32", "uniform", 3)
    ctx = ms.Context(1, n, "u32", device_ids=[0])
    ctx.sort_device([ms.tensor_ptr(chunks[0])], c)
    torch.cuda.synchronize()
    ctx.close()
    _check(chunks, n, "u32", "uniform", 3)
    with pytest.raises(ms.MsortError) as e:
        ms.Context(1, n + 1, "u32", device_ids=[0])
    assert "INVALID_ARGUMENT" in str(e.value)


def test_config3_4e9_u32_one_gpu_end_to_end():
    """configs[2] end to end (bench.py's e2e call): pinned host keys -> msort_sort_host
    (pipelined transfers, MSORT_OPT_HOST_PIPELINE default) -> host; checked on the GPU."""
    import paper_conf_sigmod_maltenbergeritr22_b200 as ms
    n = 4_000_000_000
    chunks, c = _gen_chunks(n, 1, "u32", "uniform", 1)
    host = torch.empty(n, dtype=chunks[0].dtype, pin_memory=True)
    host.copy_(chunks[0][:n])
    ctx = ms.Context(1, n, "u32", device_ids=[0])
    ctx.sort_host(ms.tensor_ptr(host), n)
    ctx.close()
    chunks[0][:n].copy_(host)
    del host
    torch.cuda.synchronize()
    _check(chunks, n, "u32", "uniform", 1)


@pytest.mark.parametrize("n,g,kt,dist,exchange", [
    (1 << 28, 2, "u32", "uniform", 0),          # configs[1]
    (2_000_000_000, 8, "u32", "zipf", 0),        # configs[3] (pivot imbalance stress)
    (2_000_000_000, 8, "u32", "reverse", 0),     # configs[3]: x_d = c on every pair, every stage
    (2_000_000_000, 8, "u32", "nearly", 0),      # configs[3]
    (2_000_000_000, 8, "u32", "sorted", 0),      # configs[3]: p = 0 every stage (no key moves)
    (2_000_000_000, 8, "u32", "normal", 0),      # Fig.16's "normal" at g > 1
    (2_000_000_000, 8, "u32", "reverse", 4),     # the NCCL send/recv swap (mode 4, self p2p on one GPU)
    (2_000_000_000, 8, "f32", "uniform", 0),     # configs[4] float keys
    (2_000_000_000, 8, "u64", "uniform", 0),     # configs[4] 64-bit keys
    (2_000_000_000, 8, "u32", "zipf", 2),        # NEXT-1 (fused all-to-all) at full size
    (4_000_000_000, 8, "u32", "uniform", 2),     # configs[2] as bench.py measures it at N = 8 (NEXT-1 default)
    (4_000_000_000, 4, "u32", "uniform", 2),     # ... at N = 4
    (1 << 28, 2, "u32", "uniform", 2),           # configs[1] with NEXT-1
    (2_000_000_000, 8, "u64", "uniform", 2),     # configs[4] 64-bit keys, NEXT-1
    (2_000_000_000, 8, "f32", "uniform", 3),     # configs[4] float keys, NEXT-1 pull-then-merge
])
def test_p2p_virtual_full_size(n, g, kt, dist, exchange):
    import paper_conf_sigmod_maltenbergeritr22_b200 as ms
    chunks, c = _gen_chunks(n, g, kt, dist, 3)
    ctx = ms.Context(g, n, kt, device_ids=[0] * g)
    ctx.set_option(ms.MSORT_OPT_EXCHANGE, exchange)
    ctx.sort_device([ms.tensor_ptr(t) for t in chunks], c)
    torch.cuda.synchronize()
    tm = ctx.timings()
    ctx.close()
    assert tm["n_stages"] == (g - 1 if exchange in (0, 1, 4) else 1)
    _check(chunks, n, kt, dist, 3)
