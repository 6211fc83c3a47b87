import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import numpy as np, torch
import msort_inputs as mi
import paper_conf_sigmod_maltenbergeritr22_b200 as ms
import test_gpu_fullsize as T
from oracle import checks
first = sys.argv[1] if len(sys.argv) > 1 else "big"
if first == "big":
    n = 4_000_000_000
    chunks, c = T._gen_chunks(n, 1, "u32", "uniform", 1)
    ctx = ms.Context(1, n, "u32", device_ids=[0]); ctx.sort_device([ms.tensor_ptr(chunks[0])], c); torch.cuda.synchronize(); ctx.close()
    del chunks
n = 1 << 28; g = 2
chunks, c = T._gen_chunks(n, g, "u32", "uniform", 3)
a = np.concatenate([t.cpu().numpy() for t in chunks])
ctx = ms.Context(g, n, "u32", device_ids=[0] * g)
ctx.sort_device([ms.tensor_ptr(t) for t in chunks], c)
torch.cuda.synchronize()
print(ctx.timings()["stage_pivot"], ctx.timings()["stage_max_x"])
out = np.concatenate([t.cpu().numpy() for t in chunks])
ref = np.sort(a)
bad = np.nonzero(out != ref)[0]
print("exact:", "ok" if len(bad) == 0 else f"BAD {len(bad)} first {bad[:8]} out {out[bad[:4]]} ref {ref[bad[:4]]}", flush=True)
print("fp out", checks.fingerprint(out, "u32"), "fp in", checks.fingerprint(a, "u32"))
ctx.close()
