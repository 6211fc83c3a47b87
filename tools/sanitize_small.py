"""Small end-to-end workload for compute-sanitizer (memcheck / racecheck / synccheck)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import msort_inputs as mi
import paper_conf_sigmod_maltenbergeritr22_b200 as ms
from oracle import sort as osort
def dev(a): return torch.from_numpy(a.view(np.uint8).copy()).cuda()
ok = True
for kt, n, g, ex in [("u32", 20011, 1, 0), ("f32", 30000, 4, 0), ("u64", 9001 * 2, 2, 1), ("u32", 24000, 4, 2)]:
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
print("ALL OK" if ok else "FAIL")
