import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import msort_inputs as mi
import paper_conf_sigmod_maltenbergeritr22_b200 as ms
from oracle import sort as osort
def dev(a): return torch.from_numpy(a.view(np.uint8).copy()).cuda()
for lg in (16, 20, 22, 24, 25, 26):
    n = 1 << lg
    for g in (2,):
        a = mi.np_generate(n, "u32", "uniform", seed=3)
        c = n // g
        ch = [dev(a[i*c:(i+1)*c]) for i in range(g)]
        ctx = ms.Context(g, n, "u32", device_ids=[0]*g)
        ctx.sort_device([ms.tensor_ptr(t) for t in ch], c)
        torch.cuda.synchronize()
        out = np.concatenate([t.cpu().numpy().view(np.uint32) for t in ch])
        ref = np.sort(a)
        bad = np.nonzero(out != ref)[0]
        print("p2p", lg, g, "ok" if len(bad) == 0 else f"BAD {len(bad)} first {bad[:5]}", ctx.timings()["stage_max_x"], flush=True)
        ctx.close()
    # direct merge step
    al = bl = n // 2
    A = np.sort(mi.np_generate(al, "u32", "uniform", seed=7)); B = np.sort(mi.np_generate(bl, "u32", "uniform", seed=8))
    da, db = dev(A), dev(B)
    out = torch.zeros(n * 4, dtype=torch.uint8, device="cuda")
    wsb = ms.msort_merge_workspace_bytes(n, "u32"); ws = torch.empty(wsb, dtype=torch.uint8, device="cuda")
    ms.msort_step_merge(ms.tensor_ptr(da), al, ms.tensor_ptr(db), bl, ms.tensor_ptr(out), "u32", ms.tensor_ptr(ws), wsb)
    torch.cuda.synchronize()
    o = out.cpu().numpy().view(np.uint32); ref = np.sort(np.concatenate([A, B]))
    bad = np.nonzero(o != ref)[0]
    print("merge", lg, "ok" if len(bad) == 0 else f"BAD {len(bad)} first {bad[:5]}", flush=True)
