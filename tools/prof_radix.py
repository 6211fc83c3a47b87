"""Sort n keys a few times on cuda:0 through the C ABI (for ncu captures)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import msort_inputs as mi
import paper_conf_sigmod_maltenbergeritr22_b200 as ms
n = int(float(sys.argv[1])) if len(sys.argv) > 1 else 1 << 28
kt = sys.argv[2] if len(sys.argv) > 2 else "u32"
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 3
dist = sys.argv[4] if len(sys.argv) > 4 else "uniform"
src = torch.empty(n, dtype=mi.torch_dtype(kt), device="cuda")
mi.t_generate_into(src, n, kt, dist, seed=1, block=1 << 27)
work = torch.empty_like(src)
ctx = ms.Context(1, n, kt, device_ids=[0])
for _ in range(reps):
    work.copy_(src)
    ctx.sort_device([ms.tensor_ptr(work)], n)
torch.cuda.synchronize()
print(ctx.timings())
