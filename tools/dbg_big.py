import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import msort_inputs as mi
import paper_conf_sigmod_maltenbergeritr22_b200 as ms
for lg in (27, 28):
    n = 1 << lg; g = 2; c = n // g
    chunks = [torch.empty(c, dtype=torch.uint32, device="cuda") for _ in range(g)]
    for i in range(g): mi.t_generate_into(chunks[i], n, "u32", "uniform", seed=3, start=i*c, block=1<<27)
    a = np.concatenate([t.cpu().numpy() for t in chunks])
    ctx = ms.Context(g, n, "u32", device_ids=[0]*g)
    ctx.sort_device([ms.tensor_ptr(t) for t in chunks], c)
    torch.cuda.synchronize()
    out = np.concatenate([t.cpu().numpy() for t in chunks])
    ref = np.sort(a)
    bad = np.nonzero(out != ref)[0]
    print(lg, "ok" if len(bad) == 0 else f"BAD {len(bad)} first {bad[:8]} out {out[bad[:4]]} ref {ref[bad[:4]]}", ctx.timings()["stage_max_x"], ctx.timings()["stage_pivot"], flush=True)
    # also radix-only of each chunk
    ctx.close()
