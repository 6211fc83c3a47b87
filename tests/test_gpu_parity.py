"""GPU parity: the CUDA path (through the C ABI) vs the CPU oracle, bit-exact.

Every row of SURVEY §8(a): S1+S2 histogram, S3 onesweep pass, S1-S3 radix sort,
S4 pivot, S6 merge, S5+S6 fused exchange, S7 stage schedule (virtual ranks on
one GPU), S0/S8 host round trip.  Sizes span several tiles and a ragged tail.
"""
import json
import os

import numpy as np
import pytest
import torch

import msort_inputs as mi
from oracle import codec, p2p, radix, sort

pytestmark = pytest.mark.gpu

GOLD = os.path.join(os.path.dirname(__file__), "golden")
KT = {"u32": 0, "u64": 1, "f32": 2, "f64": 3}


@pytest.fixture(scope="module")
def ms():
    if not torch.cuda.is_available():
        pytest.fail("GPU tests need CUDA")
    import paper_conf_sigmod_maltenbergeritr22_b200 as m
    return m


def dev_keys(a: np.ndarray) -> torch.Tensor:
    return torch.from_numpy(a.view(np.uint8).copy()).cuda()


def host_keys(t: torch.Tensor, kt: str) -> np.ndarray:
    return t.cpu().numpy().view(mi.NP_DTYPE[kt])


def bits(a, kt):
    return codec.bits_of(a, kt)


SIZES = [0, 1, 2, 3, 5, 100, 7679, 7680, 7681, 4608 * 3 + 17, 1 << 20, (1 << 20) + 13]


@pytest.mark.parametrize("kt", ["u32", "u64", "f32", "f64"])
@pytest.mark.parametrize("n", SIZES)
def test_radix_sort_single_gpu(ms, kt, n):
    a = mi.np_generate(n, kt, "uniform", seed=11)
    d = dev_keys(a)
    ms.msort_sort(ms.tensor_ptr(d), n, kt, 1)
    torch.cuda.synchronize()
    assert np.array_equal(bits(host_keys(d, kt), kt), bits(sort.oracle_sort(a, kt), kt))


@pytest.mark.parametrize("g", [1, 4])
def test_repeated_sorts_one_context(ms, g):
    """Look-back status words are not zeroed between sorts of one context (they
    carry a per-sort epoch tag): back-to-back sorts of different sizes and
    inputs in one context must each match the oracle."""
    cap = 4 * 60000
    ctx = ms.Context(g, cap, "u32", device_ids=[0] * g)
    for i, n in enumerate([cap, 4 * 7000, cap, 4 * 123, cap - 4 * 999, cap]):
        c = n // g
        a = mi.np_generate(g * c, "u32", ["uniform", "zipf", "reverse"][i % 3], seed=100 + i)
        chunks = [dev_keys(a[j * c:(j + 1) * c]) for j in range(g)]
        ctx.sort_device([ms.tensor_ptr(t) for t in chunks], c)
        torch.cuda.synchronize()
        got = np.concatenate([host_keys(t, "u32") for t in chunks])
        assert np.array_equal(got, sort.oracle_sort(a, "u32")), (i, n)
    ctx.close()


def test_epoch_wrap_zeroes_whole_workspace(ms):
    """the look-back words carry an epoch tag that comes round again
    after 512 sorts; when the epoch wraps to 0 the WHOLE workspace is zeroed, so
    a large sort at epoch E, a small one across the wrap, and a large one at
    epoch E again must all be right (stale E-tagged words past the small sort's
    tiles would otherwise be read as published)."""
    big, small = 4 * 300_000, 4 * 1000
    ctx = ms.Context(1, big, "u32", device_ids=[0])
    ctx.set_option(ms.MSORT_OPT_SMALL_GRAPH, 0)
    E = 300
    for i, (n, before) in enumerate([(big, E - 1), (small, 511), (big, E - 1), (small, 511), (big, E - 1)]):
        ctx.set_option(ms.MSORT_OPT_RADIX_EPOCH, before)
        a = mi.np_generate(n, "u32", ["uniform", "zipf"][i % 2], seed=40 + i)
        d = dev_keys(a)
        ctx.sort_device([ms.tensor_ptr(d)], n)
        torch.cuda.synchronize()
        assert np.array_equal(host_keys(d, "u32"), sort.oracle_sort(a, "u32")), (i, n)
    ctx.close()


@pytest.mark.parametrize("dist", mi.DISTRIBUTIONS)
def test_radix_sort_distributions(ms, dist):
    n = 3 * (1 << 18) + 77
    a = mi.np_generate(n, "u32", dist, seed=2)
    d = dev_keys(a)
    ms.msort_sort(ms.tensor_ptr(d), n, "u32", 1)
    torch.cuda.synchronize()
    assert np.array_equal(host_keys(d, "u32"), sort.oracle_sort(a, "u32"))


@pytest.mark.parametrize("shape", ["small_ints", "high_word", "few_doubles"])
def test_radix_sort_skewed_8byte(ms, shape):
    """Skewed 8-byte keys through the 512-thread u64/f64 tiles: every skew path of the pass (trivial passes
    skipped, a dominant digit ranked by the hot path, moderately skewed digits by peer match), over several
    7680-key tiles and a ragged one."""
    n = 5 * 7680 + 3 * (1 << 16) + 11
    z = mi.np_generate(n, "u32", "zipf_rank", seed=21).astype(np.uint64)
    if shape == "small_ints":      # high bytes zero (trivial passes), bytes 1-2 dominated by one value
        a, kt = z, "u64"
    elif shape == "high_word":     # the skew sits in the upper passes, the low word is uniform
        a, kt = (z << np.uint64(32)) | mi.np_generate(n, "u32", "uniform", seed=22).astype(np.uint64), "u64"
    else:                          # 40 distinct doubles, zipf-weighted, with -0.0 / +0.0 among them
        vals = np.concatenate([np.array([-0.0, 0.0]), np.linspace(-1e3, 1e3, 38)])
        a, kt = vals[(z % np.uint64(40)).astype(np.int64)], "f64"
    d = dev_keys(a)
    ms.msort_sort(ms.tensor_ptr(d), n, kt, 1)
    torch.cuda.synchronize()
    assert np.array_equal(bits(host_keys(d, kt), kt), bits(sort.oracle_sort(a, kt), kt))


def test_radix_sort_constant_and_special(ms):
    # all-equal keys (every pass trivial) and the IEEE special-value table
    for a, kt in [(np.full(50000, 7, np.uint32), "u32"), (np.full(9999, 0x7FC00000, np.uint32).view(np.float32), "f32")]:
        d = dev_keys(a)
        ms.msort_sort(ms.tensor_ptr(d), len(a), kt, 1)
        torch.cuda.synchronize()
        assert np.array_equal(bits(host_keys(d, kt), kt), bits(sort.oracle_sort(a, kt), kt))
    with open(os.path.join(GOLD, "float_total_order_f32.json")) as f:
        table = np.array([int(h, 16) for h in json.load(f)["ascending_bits_hex"]], dtype=np.uint32)
    rng = np.random.default_rng(0)
    a = table[rng.integers(0, len(table), 100000)].view(np.float32)
    d = dev_keys(a)
    ms.msort_sort(ms.tensor_ptr(d), len(a), "f32", 1)
    torch.cuda.synchronize()
    assert np.array_equal(host_keys(d, "f32").view(np.uint32), sort.oracle_sort(a, "f32").view(np.uint32))


@pytest.mark.parametrize("kt", ["u32", "u64", "f32", "f64"])
def test_step_histogram(ms, kt):
    n = 123457
    a = mi.np_generate(n, kt, "uniform", seed=3)
    d = dev_keys(a)
    P = radix.num_passes(kt)
    h = torch.zeros(P * 256, dtype=torch.int32, device="cuda")
    ms.msort_step_histogram(ms.tensor_ptr(d), n, kt, ms.tensor_ptr(h))
    torch.cuda.synchronize()
    got = h.cpu().numpy().view(np.uint32).reshape(P, 256)
    assert np.array_equal(got.astype(np.uint64), radix.histograms(a, kt))


@pytest.mark.parametrize("kt", ["u64", "f64"])
def test_step_histogram_8byte_skewed_large(ms, kt):
    """4e8 8-byte keys (~2600 per thread of 148 x 1024, so every private counter column sees thousands of
    adds), all but 1 in 997 on ONE bin per pass, read from one key past a 16-byte boundary (head and tail
    keys).  Expected: the oracle's histogram of the random keys plus the constant key's bins times its
    count (closed form)."""
    n = 400_000_003
    const = np.array([0x40091EB851EB851F], dtype=np.uint64)  # (as f64: 3.14; codec T applied by the oracle)
    d = torch.full((n,), int(const.view(np.int64)[0]), dtype=torch.int64, device="cuda")
    idx = torch.arange(1, n, 997, device="cuda")
    rnd = mi.np_generate(len(idx), kt, "uniform", seed=11)
    d[idx] = torch.from_numpy(rnd.view(np.int64).copy()).cuda()
    P = radix.num_passes(kt)
    h = torch.zeros(P * 256, dtype=torch.int32, device="cuda")
    ms.msort_step_histogram(ms.tensor_ptr(d) + 8, n - 1, kt, ms.tensor_ptr(h))  # keys d[1:]
    torch.cuda.synchronize()
    got = h.cpu().numpy().view(np.uint32).reshape(P, 256).astype(np.uint64)
    n_const = (n - 1) - len(idx)
    want = radix.histograms(rnd.view(mi.NP_DTYPE[kt]), kt) + radix.histograms(const.view(mi.NP_DTYPE[kt]), kt) * n_const
    assert np.array_equal(got, want)


@pytest.mark.parametrize("kt", ["u32", "u64", "f32"])
def test_step_radix_pass(ms, kt):
    n = 50001
    a = mi.np_generate(n, kt, "uniform", seed=4)
    P = radix.num_passes(kt)
    hist = torch.from_numpy(radix.histograms(a, kt).astype(np.uint32).view(np.int32).reshape(-1).copy()).cuda()
    ws_bytes = ms.msort_radix_workspace_bytes(n, kt)
    ws = torch.empty(ws_bytes, dtype=torch.uint8, device="cuda")
    codes = codec.encode(a, kt)
    cur_dev = dev_keys(a)  # raw keys for pass 0
    for p in range(P):
        out = torch.empty_like(cur_dev)
        flags = (ms.MSORT_PASS_ENCODE_IN if p == 0 else 0)
        ms.msort_step_radix_pass(ms.tensor_ptr(cur_dev), ms.tensor_ptr(out), n, kt, p, ms.tensor_ptr(hist), flags,
                                 ms.tensor_ptr(ws), ws_bytes)
        torch.cuda.synchronize()
        codes = radix.counting_pass(codes, p)
        got = out.cpu().numpy().view(codec.UINT[kt])
        assert np.array_equal(got, codes), f"pass {p}"
        cur_dev = out


def _chunks_to_dev(chunks, kt):
    return [dev_keys(c) for c in chunks]


@pytest.mark.parametrize("kt", ["u32", "u64", "f32"])
@pytest.mark.parametrize("nchunks", [2, 4, 8])
def test_step_pivot(ms, kt, nchunks):
    rng = np.random.default_rng(nchunks)
    for trial in range(12):
        c = int(rng.integers(1, 3000))
        dist = ["uniform", "sorted", "reverse"][trial % 3]
        if kt == "u32":
            data = mi.np_generate(c * nchunks, kt, "uniform", seed=trial)
            if trial % 4 == 3:
                data = (data % np.uint32(5)).astype(np.uint32)   # duplicate-heavy
        else:
            data = mi.np_generate(c * nchunks, kt, "uniform", seed=trial)
        h = nchunks // 2
        # A (left half) and B (right half) must each be sorted as concatenations
        # (what the earlier merge stages guarantee)
        A = sort.oracle_sort(data[: h * c], kt)
        B = sort.oracle_sort(data[h * c:], kt)
        if dist == "sorted":
            s = sort.oracle_sort(data, kt)
            A, B = s[: h * c], s[h * c:]
        elif dist == "reverse":
            s = sort.oracle_sort(data, kt)
            A, B = s[h * c:], s[: h * c]
        chunks = [A[i * c:(i + 1) * c] for i in range(h)] + [B[i * c:(i + 1) * c] for i in range(h)]
        codes = [codec.encode(x, kt) for x in chunks]
        expect = p2p.select_pivot(p2p.Concat(codes[:h]), p2p.Concat(codes[h:]))
        devs = _chunks_to_dev(chunks, kt)
        out = torch.zeros(1, dtype=torch.int64, device="cuda")
        ms.msort_step_pivot([ms.tensor_ptr(t) for t in devs], c, kt, ms.tensor_ptr(out))
        torch.cuda.synchronize()
        assert int(out.item()) == expect


def test_step_pivot_paper_figures(ms):
    with open(os.path.join(GOLD, "fig8.json")) as f:
        fx8 = json.load(f)
    with open(os.path.join(GOLD, "fig9.json")) as f:
        fx9 = json.load(f)
    out = torch.zeros(1, dtype=torch.int64, device="cuda")
    devs = [dev_keys(np.array(r, dtype=np.uint32)) for r in fx8["before"]]
    ms.msort_step_pivot([ms.tensor_ptr(t) for t in devs], 4, "u32", ms.tensor_ptr(out))
    torch.cuda.synchronize()
    assert out.item() == fx8["pivot_p"]
    devs = [dev_keys(np.array(r, dtype=np.uint32)) for r in fx9["after_stage1"]]
    ms.msort_step_pivot([ms.tensor_ptr(t) for t in devs], 4, "u32", ms.tensor_ptr(out))
    torch.cuda.synchronize()
    assert out.item() == fx9["stage2_pivot_p"]


@pytest.mark.parametrize("kt", ["u32", "u64", "f32", "f64"])
def test_step_merge(ms, kt):
    rng = np.random.default_rng(5)
    for al, bl in [(0, 0), (0, 5), (7, 0), (1, 1), (3839, 1), (3840, 3840), (100000, 3), (54321, 65432)]:
        a = sort.oracle_sort(mi.np_generate(al, kt, "uniform", seed=al + 1), kt)
        b = sort.oracle_sort(mi.np_generate(bl, kt, "uniform", seed=bl + 2), kt)
        if kt == "u32" and al and bl:
            a = sort.oracle_sort((a % np.uint32(50)).astype(np.uint32), kt)   # ties across runs
            b = sort.oracle_sort((b % np.uint32(50)).astype(np.uint32), kt)
        da, db = dev_keys(a), dev_keys(b)
        out = torch.zeros(max(1, (al + bl)) * mi.KEY_BYTES[kt], dtype=torch.uint8, device="cuda")
        wsb = ms.msort_merge_workspace_bytes(al + bl, kt)
        ws = torch.empty(wsb, dtype=torch.uint8, device="cuda")
        ms.msort_step_merge(ms.tensor_ptr(da), al, ms.tensor_ptr(db), bl, ms.tensor_ptr(out), kt, ms.tensor_ptr(ws), wsb)
        torch.cuda.synchronize()
        got = host_keys(out, kt)[: al + bl]
        expect = sort.oracle_sort(np.concatenate([a, b]), kt)
        assert np.array_equal(bits(got, kt), bits(expect, kt)), (al, bl)


@pytest.mark.parametrize("kt", ["u32", "u64"])
def test_step_merge_unaligned(ms, kt):
    """Runs and output starting at any key offset (the merge bulk-copies each
    range from its 16-byte-aligned start to the 16-byte boundary after its end;
    the ragged output goes through the scalar store path)."""
    K = mi.KEY_BYTES[kt]
    for (oa, ob, oo), (al, bl) in [((1, 2, 0), (40000, 33333)), ((3, 0, 1), (3841, 7681)), ((2, 3, 3), (5, 100001)),
                                    ((1, 1, 2), (65536, 65536)), ((0, 1, 0), (1, 123457))]:
        a = sort.oracle_sort(mi.np_generate(al, kt, "uniform", seed=oa + 11), kt)
        b = sort.oracle_sort(mi.np_generate(bl, kt, "uniform", seed=ob + 13), kt)
        da = dev_keys(np.concatenate([np.zeros(oa, a.dtype), a]))
        db = dev_keys(np.concatenate([np.zeros(ob, b.dtype), b]))
        out = torch.zeros((al + bl + oo) * K, dtype=torch.uint8, device="cuda")
        wsb = ms.msort_merge_workspace_bytes(al + bl, kt)
        ws = torch.empty(wsb, dtype=torch.uint8, device="cuda")
        ms.msort_step_merge(ms.tensor_ptr(da) + oa * K, al, ms.tensor_ptr(db) + ob * K, bl, ms.tensor_ptr(out) + oo * K,
                            kt, ms.tensor_ptr(ws), wsb)
        torch.cuda.synchronize()
        got = host_keys(out, kt)[oo: oo + al + bl]
        expect = sort.oracle_sort(np.concatenate([a, b]), kt)
        assert np.array_equal(bits(got, kt), bits(expect, kt)), (oa, ob, oo, al, bl)


def _virtual_sort(ms, a, kt, g, exchange=0):
    """g virtual ranks on GPU 0, device-resident chunks of c keys."""
    n = len(a)
    c = n // g
    ctx = ms.Context(g, n, kt, device_ids=[0] * g)
    ctx.set_option(ms.MSORT_OPT_EXCHANGE, exchange)
    chunks = [dev_keys(a[i * c:(i + 1) * c]) for i in range(g)]
    ctx.sort_device([ms.tensor_ptr(t) for t in chunks], c)
    torch.cuda.synchronize()
    out = np.concatenate([host_keys(t, kt) for t in chunks])
    tm = ctx.timings()
    ctx.close()
    return out, tm


@pytest.mark.parametrize("g", [2, 4, 8])
@pytest.mark.parametrize("dist", ["uniform", "sorted", "reverse", "nearly", "zipf", "normal"])
def test_p2p_sort_virtual_ranks(ms, g, dist):
    c = 3 * 7680 + 44
    a = mi.np_generate(g * c, "u32", dist, seed=g)
    out, tm = _virtual_sort(ms, a, "u32", g)
    assert np.array_equal(out, sort.oracle_sort(a, "u32"))
    # stage-level parity with the oracle's Alg.2 model: labels and every pivot
    chunks = [np.sort(a[i * c:(i + 1) * c]) for i in range(g)]
    stages = p2p.run_stages(chunks)
    assert tm["stage_label"] == p2p.stage_labels(g)
    for s, st in enumerate(stages):
        assert tm["stage_pivot"][s][: len(st)] == [op.p for op in st]
        assert tm["stage_max_x"][s] == max(max(op.xs) for op in st)
    # per-stage timings: the pivot search is part of the stage, the exchange too
    for pv, ex, st in zip(tm["stage_pivot_ms"], tm["stage_exchange_ms"], tm["stage_ms"]):
        assert 0 < pv <= st and 0 <= ex <= st


def _staged_chunks(ms, a, kt, g, exchange, stop):
    """Virtual-rank Alg.2 stopped after stage `stop` (MSORT_OPT_STOP_AFTER_STAGE): every chunk."""
    n = len(a)
    c = n // g
    ctx = ms.Context(g, n, kt, device_ids=[0] * g)
    ctx.set_option(ms.MSORT_OPT_EXCHANGE, exchange)
    ctx.set_option(ms.MSORT_OPT_STOP_AFTER_STAGE, stop)
    chunks = [dev_keys(a[i * c:(i + 1) * c]) for i in range(g)]
    ctx.sort_device([ms.tensor_ptr(t) for t in chunks], c)
    torch.cuda.synchronize()
    out = [host_keys(t, kt) for t in chunks]
    tm = ctx.timings()
    ctx.close()
    return out, tm


@pytest.mark.parametrize("exchange", [0, 1, 4])
@pytest.mark.parametrize("g", [2, 4, 8])
@pytest.mark.parametrize("dist", ["uniform", "reverse", "dups", "zipf"])
def test_alg2_every_stage_matches_stage_model(ms, g, dist, exchange):
    """SURVEY §8(c) S7 pin: after EVERY Alg.2 stage, every GPU's chunk equals the
    oracle's stage model (oracle.p2p.run_stages, Alg.2 P:1804-1818 in its
    concurrent form, reading Q7) - the fused device-resident exchange (0), the
    paper's copy-then-merge swap (1) and the NCCL send/recv swap (4)."""
    c = 2 * 4864 + 52   # several merge tiles and a ragged one
    if dist == "dups":
        a = (mi.np_generate(g * c, "u32", "uniform", seed=g + 3) % np.uint32(97)).astype(np.uint32)
    else:
        a = mi.np_generate(g * c, "u32", dist, seed=g + 3)
    codes = [np.sort(codec.encode(a[i * c:(i + 1) * c], "u32")) for i in range(g)]
    stages = p2p.run_stages(codes)
    for s, st in enumerate(stages):
        expect = [None] * g
        for op in st:
            for k, ch in enumerate(op.after):
                expect[op.lo + k] = ch
        out, tm = _staged_chunks(ms, a, "u32", g, exchange, s)
        assert tm["n_stages"] == s + 1
        assert tm["stage_pivot"][s][: len(st)] == [op.p for op in st]
        for q in range(g):
            assert np.array_equal(out[q], expect[q]), (s, q)


@pytest.mark.parametrize("exchange", [0, 1, 4])
@pytest.mark.parametrize("c", [1, 3, 5003, 4864 + 1])
def test_p2p_sort_ragged_chunks(ms, c, exchange):
    """Chunks whose size is not a multiple of 4 keys (a ragged tail after the last
    16-byte unit) through every Alg.2 exchange mode."""
    g = 4
    a = mi.np_generate(g * c, "u32", "uniform", seed=c)
    out, _ = _virtual_sort(ms, a, "u32", g, exchange=exchange)
    assert np.array_equal(out, sort.oracle_sort(a, "u32"))


@pytest.mark.parametrize("g", [2, 4, 8])
@pytest.mark.parametrize("dist", ["uniform", "sorted", "reverse", "zipf"])
def test_p2p_sort_nccl_swap(ms, g, dist):
    """Exchange mode 4: the swap as grouped ncclSend/ncclRecv per mirrored pair (one
    communicator on the one GPU: NCCL self send/recv), then the local merge."""
    c = 3 * 7680 + 44
    a = mi.np_generate(g * c, "u32", dist, seed=g + 11)
    out, tm = _virtual_sort(ms, a, "u32", g, exchange=4)
    assert np.array_equal(out, sort.oracle_sort(a, "u32"))
    assert tm["stage_label"] == p2p.stage_labels(g)
    assert tm["exchange_mode"] == 4
    for mx, sw, ex in zip(tm["stage_max_x"], tm["stage_swap_ms"], tm["stage_exchange_ms"]):
        if mx:  # the NCCL transfer alone is timed, and it is part of the stage's exchange + merge
            assert 0 < sw <= ex


@pytest.mark.parametrize("kt", ["u64", "f32", "f64"])
def test_p2p_sort_nccl_swap_key_types(ms, kt):
    g, c = 4, 5003
    a = mi.np_generate(g * c, kt, "uniform", seed=23)
    out, _ = _virtual_sort(ms, a, kt, g, exchange=4)
    assert np.array_equal(bits(out, kt), bits(sort.oracle_sort(a, kt), kt))


@pytest.mark.parametrize("kt", ["u64", "f32", "f64"])
def test_p2p_sort_virtual_key_types(ms, kt):
    g, c = 4, 5000
    a = mi.np_generate(g * c, kt, "uniform", seed=21)
    out, _ = _virtual_sort(ms, a, kt, g)
    assert np.array_equal(bits(out, kt), bits(sort.oracle_sort(a, kt), kt))


@pytest.mark.parametrize("g", [2, 8])
def test_p2p_sort_swap_mode(ms, g):
    c = 20000
    a = mi.np_generate(g * c, "u32", "uniform", seed=31)
    out, tm = _virtual_sort(ms, a, "u32", g, exchange=1)
    assert np.array_equal(out, sort.oracle_sort(a, "u32"))


@pytest.mark.parametrize("g", [1, 2, 4, 8])
@pytest.mark.parametrize("n", [2, 7, 1001, 65536 + 3])
def test_sort_host_end_to_end(ms, g, n):
    a = mi.np_generate(n, "u32", "uniform", seed=n)
    h = torch.from_numpy(a.copy()).pin_memory()
    ctx = ms.Context(g, n, "u32", device_ids=[0] * g)
    ctx.sort_host(ms.tensor_ptr(h), n)
    ctx.close()
    assert np.array_equal(h.numpy(), sort.oracle_sort(a, "u32"))


@pytest.mark.parametrize("kt,dist,n", [("u32", "uniform", (1 << 22) + 3), ("u32", "zipf", (1 << 21) + 1),
                                       ("u32", "reverse", 1 << 20), ("u64", "uniform", (1 << 21) + 2),
                                       ("f32", "uniform", 3_000_001), ("f64", "uniform", (1 << 20) + 7)])
@pytest.mark.parametrize("pipeline", [1, 0])
def test_sort_host_pipelined(ms, kt, dist, n, pipeline):
    """msort_sort_host on one GPU with MSORT_OPT_HOST_PIPELINE (4 pieces sorted as
    they land, merged, the final merge sliced and copied back slice by slice) and
    without it: both equal the oracle (the sorted multiset is unique, §8(c))."""
    a = mi.np_generate(n, kt, dist, seed=5)
    h = torch.from_numpy(a.copy()).pin_memory()
    ctx = ms.Context(1, n, kt, device_ids=[0])
    ctx.set_option(ms.MSORT_OPT_HOST_PIPELINE, pipeline)
    ctx.sort_host(ms.tensor_ptr(h), n)
    t = ctx.timings()
    ctx.close()
    assert bits(h.numpy(), kt).tobytes() == bits(sort.oracle_sort(a, kt), kt).tobytes()
    assert t["total_ms"] > 0 and t["h2d_ms"] > 0 and t["d2h_ms"] > 0


def _shaped(n, kt, dist, seed):
    """distribution shapes for every key type (u64 / f32 from the u32 shapes' bits)"""
    if kt in ("u32",) or dist == "uniform":
        return mi.np_generate(n, kt, dist, seed=seed)
    a = mi.np_generate(n, "u32", dist, seed=seed)
    return {"u64": a.astype(np.uint64) * np.uint64(0x10001), "f32": a.view(np.float32),
            "f64": (a.astype(np.uint64) << np.uint64(32)).view(np.float64)}[kt]


@pytest.mark.parametrize("kt", ["u32", "u64", "f32", "f64"])
def test_small_sort_graph_replay(ms, kt):
    """Repeated one-GPU sorts of one buffer (MSORT_OPT_SMALL_GRAPH: the second call
    captures the radix sort as a CUDA graph, later calls replay it) on new data each
    time, skewed and sorted shapes included, then a new size (re-capture): every
    result equals the oracle (§8(c))."""
    K = mi.KEY_BYTES[kt]
    for n in ((1 << 20) + 5, 300_001):
        buf = torch.empty(n * K, dtype=torch.uint8, device="cuda")
        ctx = ms.Context(1, n, kt, device_ids=[0])
        for trial, dist in enumerate(["uniform", "zipf", "uniform", "reverse", "sorted", "uniform"]):
            a = _shaped(n, kt, dist, seed=trial)
            buf.copy_(torch.from_numpy(a.view(np.uint8).copy()))
            ctx.sort_device([ms.tensor_ptr(buf)], n)
            got = buf.cpu().numpy().view(codec.UINT[kt])
            assert got.tobytes() == bits(sort.oracle_sort(a, kt), kt).tobytes(), (n, trial, dist)
        t = ctx.timings()
        assert t["passes_run"] == radix.num_passes(kt)
        ctx.close()


@pytest.mark.parametrize("n,kt", [(100003, "f32"), ((1 << 21) + 1, "u32"), ((1 << 20) + 6, "u64")])
def test_msort_sort_host_pointer(ms, n, kt):
    """The north-star entry msort_sort on PAGEABLE host memory (numpy), below and above the pipelining
    threshold (2^20 keys): the copies are staged by the driver, the result is the oracle's."""
    a = mi.np_generate(n, kt, "uniform", seed=9)
    h = a.copy()
    ms.msort_sort(h.ctypes.data, n, kt, 1)
    assert bits(h, kt).tobytes() == bits(sort.oracle_sort(a, kt), kt).tobytes()


@pytest.mark.parametrize("n,kt,g", [(50_000_003, "u32", 1), (20_000_001, "f64", 2), (33_554_437, "u64", 4),
                                    (300_000_001, "u32", 1), (100_000_003, "u64", 1)])
def test_pageable_host_bounce(ms, n, kt, g):
    """Pageable host keys (numpy) spanning several 64 MiB pinned bounce buffers: the host threads' copies,
    the bounce ring's events and the padding of the last chunk, through msort_sort (the north-star entry,
    g = 1: the pipelined path, the host staging piece i+1 while the GPU sorts piece i, each piece and each
    D2H slice several bounce buffers long) and a context (virtual ranks)."""
    a = mi.np_generate(n, kt, "uniform", seed=n % 97)
    h = a.copy()
    if g == 1:
        ms.msort_sort(h.ctypes.data, n, kt, 1)
    else:
        ctx = ms.Context(g, n, kt, device_ids=[0] * g)
        ctx.sort_host(h.ctypes.data, n)
        ctx.close()
    assert bits(h, kt).tobytes() == bits(sort.oracle_sort(a, kt), kt).tobytes()


def test_errors(ms):
    with pytest.raises(ms.MsortError):
        ms.msort_sort(0, 10, "u32", 1)
    with pytest.raises(ms.MsortError):
        ms.msort_sort(1234, 10, "u32", 3)
    with pytest.raises(ms.MsortError):
        ms.msort_sort(1234, 10, 9, 1)
    ms.msort_sort(0, 0, "u32", 1)   # n = 0 is a no-op


def test_out_of_memory_is_reported_and_recoverable(ms):
    """A context larger than HBM (8 virtual ranks x (2^32 - 4) u64 keys: 3 chunk buffers of 32 GB each per
    rank) fails with MSORT_ERR_OUT_OF_MEMORY (include/msort.h: no CPU fallback) and leaves the device usable:
    what it had allocated is freed and the next context sorts correctly."""
    n = 8 * ((1 << 32) - 4)
    with pytest.raises(ms.MsortError) as e:
        ms.Context(8, n, "u64", device_ids=[0] * 8)
    assert "OUT_OF_MEMORY" in str(e.value)
    a = mi.np_generate(100_003, "u64", "uniform", seed=8)
    d = dev_keys(a)
    ctx = ms.Context(1, a.size, "u64", device_ids=[0])
    ctx.sort_device([ms.tensor_ptr(d)], a.size)
    torch.cuda.synchronize()
    ctx.close()
    assert np.array_equal(host_keys(d, "u64"), sort.oracle_sort(a, "u64"))


# ---------------------------------------------------------------------------
# NEXT-1: single all-to-all exchange (MSORT_OPT_EXCHANGE = 2 fused, 3 pull-then-merge)
# ---------------------------------------------------------------------------

@pytest.mark.parametrize("g", [2, 4, 8])
def test_step_splitters(ms, g):
    rng = np.random.default_rng(g + 100)
    for trial in range(6):
        c = int(rng.integers(1, 5000))
        kt = ["u32", "u64", "f32"][trial % 3]
        data = mi.np_generate(g * c, kt, "uniform", seed=trial)
        if kt == "u32" and trial % 2:
            data = (data % np.uint32(7)).astype(np.uint32)   # heavy ties across chunks
        chunks = [sort.oracle_sort(data[i * c:(i + 1) * c], kt) for i in range(g)]
        codes = [codec.encode(x, kt) for x in chunks]
        expect = [p2p.multiway_splitter(codes, j * c) for j in range(g + 1)]
        devs = [dev_keys(x) for x in chunks]
        out = torch.zeros((g + 1) * g, dtype=torch.int64, device="cuda")
        ms.msort_step_splitters([ms.tensor_ptr(t) for t in devs], c, kt, ms.tensor_ptr(out))
        torch.cuda.synchronize()
        got = out.cpu().numpy().reshape(g + 1, g).tolist()
        assert got == expect, (kt, c)


@pytest.mark.parametrize("exchange", [2, 3])  # 2: pulls fused into the first merge round, 3: pull, then merge
@pytest.mark.parametrize("g", [2, 4, 8])
@pytest.mark.parametrize("dist", ["uniform", "sorted", "reverse", "zipf", "zipf_rank"])
def test_alltoall_virtual_ranks(ms, g, dist, exchange):
    c = 3 * 7168 + 52
    a = mi.np_generate(g * c, "u32", dist, seed=g + 7)
    out, tm = _virtual_sort(ms, a, "u32", g, exchange=exchange)
    assert np.array_equal(out, sort.oracle_sort(a, "u32"))
    assert tm["n_stages"] == 1 and tm["stage_label"] == [g]


@pytest.mark.parametrize("exchange", [2, 3])
@pytest.mark.parametrize("kt", ["u64", "f32", "f64"])
def test_alltoall_virtual_key_types(ms, kt, exchange):
    g, c = 8, 4001
    a = mi.np_generate(g * c, kt, "uniform", seed=33)
    out, _ = _virtual_sort(ms, a, kt, g, exchange=exchange)
    assert np.array_equal(bits(out, kt), bits(sort.oracle_sort(a, kt), kt))


def test_rank_mode_probe(ms):
    # the lane-order self-test ran; report which ranking the passes use
    mode = ms.msort_rank_mode(0)
    assert mode in (0, 1)
    print("onesweep ranking:", "atomic (lane-ordered)" if mode == 1 else "peer match")


def test_soak_mixed_sizes_one_context(ms):
    """Stress of the cross-block protocols racecheck cannot see (the global-memory
    decoupled look-back with epoch-tagged status words, the device-resident merge
    stages): 120 back-to-back sorts in two long-lived contexts with random sizes
    around tile and group boundaries, random distributions and key types, each
    equal to the oracle."""
    rng = np.random.default_rng(2024)
    cap = 1 << 21
    ctxs = {g: ms.Context(g, cap, "u32", device_ids=[0] * g) for g in (1, 4)}
    ctxs[1].set_option(ms.MSORT_OPT_SMALL_GRAPH, 0)
    for it in range(120):
        g = 1 if it % 3 else 4
        tiles = int(rng.integers(1, (cap // g) // 7168))
        c = max(4, tiles * 7168 + int(rng.integers(-300, 300))) // 4 * 4
        dist = ["uniform", "zipf", "sorted", "reverse", "nearly", "normal"][int(rng.integers(0, 6))]
        a = mi.np_generate(g * c, "u32", dist, seed=it)
        chunks = [dev_keys(a[i * c:(i + 1) * c]) for i in range(g)]
        ctxs[g].sort_device([ms.tensor_ptr(t) for t in chunks], c)
        torch.cuda.synchronize()
        got = np.concatenate([host_keys(t, "u32") for t in chunks])
        assert np.array_equal(got, sort.oracle_sort(a, "u32")), (it, g, c, dist)
    for c in ctxs.values():
        c.close()


def test_rank_mode_is_atomic_on_b200(ms):
    """On sm_100 the lane-order probe AND the production-kernel check (one stable pass
    with atomic ranking equals the same pass with peer-match ranking, both key widths)
    pass, so the passes rank with one shared atomic per key (reading Q16)."""
    assert ms.msort_rank_mode(0) == 1


# ---------------------------------------------------------------------------
# Distinct GPUs (skipped on one-GPU boxes): the same paths over NVLink
# ---------------------------------------------------------------------------

@pytest.mark.parametrize("exchange", [0, 1, 2, 4])
@pytest.mark.parametrize("g", [2, 4, 8])
def test_p2p_sort_distinct_gpus(ms, g, exchange):
    """Chunk i on GPU i (peer access over NVLink): every exchange mode equals the oracle, every Alg.2 stage
    equals the stage model, and the peer bulk-copy self-test ran between distinct devices."""
    if torch.cuda.device_count() < g:
        pytest.skip(f"needs {g} GPUs")
    c = 2 * 7168 + 36
    a = mi.np_generate(g * c, "u32", "uniform", seed=g * 10 + exchange)
    ctx = ms.Context(g, g * c, "u32", device_ids=list(range(g)))
    ctx.set_option(ms.MSORT_OPT_EXCHANGE, exchange)
    chunks = [torch.from_numpy(a[i * c:(i + 1) * c].view(np.uint8).copy()).to(f"cuda:{i}") for i in range(g)]
    ctx.sort_device([ms.tensor_ptr(t) for t in chunks], c)
    for i in range(g):
        torch.cuda.synchronize(i)
    out = np.concatenate([t.cpu().numpy().view(np.uint32) for t in chunks])
    tm = ctx.timings()
    assert np.array_equal(out, sort.oracle_sort(a, "u32"))
    assert tm["peer_bulk_ok"] == 1 and tm["exchange_mode"] == exchange
    if exchange in (0, 1, 4):
        codes = [np.sort(a[i * c:(i + 1) * c]) for i in range(g)]
        stages = p2p.run_stages(codes)
        for s, st in enumerate(stages):
            assert tm["stage_pivot"][s][: len(st)] == [op.p for op in st]
    ctx.close()


@pytest.mark.parametrize("exchange", [0, 1, 2, 4])
def test_timing_off_every_mode(ms, exchange):
    """MSORT_OPT_TIMING = 0 (no per-phase events) leaves every exchange mode's result and stage
    statistics intact."""
    g, c = 4, 3 * 7168 + 8
    a = mi.np_generate(g * c, "u32", "reverse", seed=exchange + 50)
    ctx = ms.Context(g, g * c, "u32", device_ids=[0] * g)
    ctx.set_option(ms.MSORT_OPT_TIMING, 0)
    ctx.set_option(ms.MSORT_OPT_EXCHANGE, exchange)
    chunks = [dev_keys(a[i * c:(i + 1) * c]) for i in range(g)]
    ctx.sort_device([ms.tensor_ptr(t) for t in chunks], c)
    torch.cuda.synchronize()
    out = np.concatenate([host_keys(t, "u32") for t in chunks])
    tm = ctx.timings()
    ctx.close()
    assert np.array_equal(out, sort.oracle_sort(a, "u32"))
    if exchange != 2:  # reverse input: every mirrored pair swaps whole chunks in every stage (x_d = c)
        assert tm["stage_max_x"] == [c] * (g - 1)
