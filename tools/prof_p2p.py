"""Virtual-rank P2P sort on cuda:0 through the C ABI (for ncu captures of the merge phase).
usage: prof_p2p.py N G KT EXCHANGE [REPS]"""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import msort_inputs as mi
import paper_conf_sigmod_maltenbergeritr22_b200 as ms
n, g, kt, ex = int(float(sys.argv[1])), int(sys.argv[2]), sys.argv[3], int(sys.argv[4])
reps = int(sys.argv[5]) if len(sys.argv) > 5 else 2
c = n // g
src = [torch.empty(c, dtype=mi.torch_dtype(kt), device="cuda") for _ in range(g)]
for i, t in enumerate(src):
    mi.t_generate_into(t, n, kt, "uniform", seed=1, start=i * c, block=1 << 27)
work = [torch.empty_like(t) for t in src]
ctx = ms.Context(g, n, kt, device_ids=[0] * g)
ctx.set_option(ms.MSORT_OPT_EXCHANGE, ex)
for _ in range(reps):
    for w, s in zip(work, src):
        w.copy_(s)
    ctx.sort_device([ms.tensor_ptr(w) for w in work], c)
torch.cuda.synchronize()
print(ctx.timings())
