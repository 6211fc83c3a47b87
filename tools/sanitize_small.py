"""Small end-to-end workload for compute-sanitizer (memcheck / racecheck / synccheck)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import msort_inputs as mi
import paper_conf_sigmod_maltenbergeritr22_b200 as ms
from oracle import sort as osort
def dev(a): return torch.from_numpy(a.view(np.uint8).copy()).cuda()
ok = True
# (g > 1, mode 0: the device-resident Alg.2 stages; mode 4: the NCCL send/recv swap; 4 x 5003: ragged chunks)
for kt, n, g, ex in [("u32", 20011, 1, 0), ("f32", 30000, 4, 0), ("u64", 9001 * 2, 2, 1), ("u32", 24000, 4, 2),
                     ("u64", 16000, 8, 2), ("u32", 24000, 4, 3), ("u32", 4 * 5003, 4, 0), ("u32", 32000, 8, 0),
                     ("u32", 4 * 5003, 4, 4), ("f64", 12000, 2, 4)]:
    a = mi.np_generate(n, kt, "uniform", seed=2)
    c = n // g
    ctx = ms.Context(g, n, kt, device_ids=[0] * g)
    ctx.set_option(ms.MSORT_OPT_EXCHANGE, ex)
    ch = [dev(a[i * c:(i + 1) * c]) for i in range(g)]
    ctx.sort_device([ms.tensor_ptr(t) for t in ch], c)
    torch.cuda.synchronize()
    out = np.concatenate([t.cpu().numpy() for t in ch]).view(mi.NP_DTYPE[kt])
    good = np.array_equal(out.view(np.uint8), osort.oracle_sort(a[:g * c], kt).view(np.uint8))
    ok &= good
    print(kt, n, g, ex, "ok" if good else "MISMATCH", flush=True)
    ctx.close()
# pipelined host sort (pieces sorted as they land, sliced final merge) and the small-sort graph replay
for kt, n in [("u32", (1 << 20) + 3), ("f64", (1 << 20) + 1)]:
    a = mi.np_generate(n, kt, "uniform", seed=7)
    h = torch.from_numpy(a.copy()).pin_memory()
    ctx = ms.Context(1, n, kt, device_ids=[0])
    ctx.sort_host(ms.tensor_ptr(h), n)
    good = np.array_equal(h.numpy().view(np.uint8), osort.oracle_sort(a, kt).view(np.uint8))
    ok &= good
    print("pipelined host", kt, n, "ok" if good else "MISMATCH", flush=True)
    d = dev(a)
    for rep in range(3):  # 2nd call captures, 3rd replays
        d.copy_(dev(a))
        ctx.sort_device([ms.tensor_ptr(d)], n)
        torch.cuda.synchronize()
        good = np.array_equal(d.cpu().numpy(), osort.oracle_sort(a, kt).view(np.uint8))
        ok &= good
    print("graph replay", kt, n, "ok" if good else "MISMATCH", flush=True)
    ctx.close()
# merge step on runs/output at odd key offsets (bulk copies over-fetch to 16-byte bounds)
for kt, oa, ob, oo, al, bl in [("u32", 1, 3, 2, 9001, 7777), ("u64", 1, 0, 1, 5003, 6007)]:
    K = mi.KEY_BYTES[kt]
    a = osort.oracle_sort(mi.np_generate(al, kt, "uniform", seed=3), kt)
    b = osort.oracle_sort(mi.np_generate(bl, kt, "uniform", seed=4), kt)
    da = dev(np.concatenate([np.zeros(oa, a.dtype), a]))
    db = dev(np.concatenate([np.zeros(ob, b.dtype), b]))
    out = torch.zeros((al + bl + oo) * K, dtype=torch.uint8, device="cuda")
    wsb = ms.msort_merge_workspace_bytes(al + bl, kt)
    ws = torch.empty(wsb, dtype=torch.uint8, device="cuda")
    ms.msort_step_merge(ms.tensor_ptr(da) + oa * K, al, ms.tensor_ptr(db) + ob * K, bl, ms.tensor_ptr(out) + oo * K, kt,
                        ms.tensor_ptr(ws), wsb)
    torch.cuda.synchronize()
    got = out.cpu().numpy().view(mi.NP_DTYPE[kt])[oo:oo + al + bl]
    good = np.array_equal(got.view(np.uint8), osort.oracle_sort(np.concatenate([a, b]), kt).view(np.uint8))
    ok &= good
    print("merge", kt, al, bl, "ok" if good else "MISMATCH", flush=True)
# interconnect measurement and the out-of-core HET baseline (NEXT-4)
ctx = ms.Context(2, 1 << 20, "u32", device_ids=[0, 0])
print("links", ctx.measure_links(1 << 20, 1), flush=True)
ctx.close()
from baseline import het
a = mi.np_generate(300_001, "u32", "uniform", seed=9)
h = torch.from_numpy(a.copy()).pin_memory()
o = torch.empty_like(h)
het.het_ooc_sort(h, "u32", 1 << 16, [0, 0], o)
good = np.array_equal(o.numpy(), osort.oracle_sort(a, "u32"))
ok &= good
print("het ooc", "ok" if good else "MISMATCH", flush=True)
print("ALL OK" if ok else "FAIL")
