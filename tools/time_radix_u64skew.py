"""Time the radix sort of n uint64 keys whose HIGH word is zipf (fmix32-scattered ranks) and low word uniform:
the four upper passes are moderately skewed (peer-match ranking), the four lower ones uniform.
usage: time_radix_u64skew.py N [REPS]   (MSORT_PKG_ROOT selects a tools/_ablate build)"""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
if os.environ.get("MSORT_PKG_ROOT"): sys.path.insert(0, os.environ["MSORT_PKG_ROOT"])
import torch
import msort_inputs as mi
import paper_conf_sigmod_maltenbergeritr22_b200 as ms
n = int(float(sys.argv[1])); reps = int(sys.argv[2]) if len(sys.argv) > 2 else 5
hi = torch.empty(n, dtype=torch.int32, device="cuda")
lo = torch.empty(n, dtype=torch.int32, device="cuda")
mi.t_generate_into(hi.view(torch.uint32), n, "u32", "zipf", seed=1, block=1 << 27)
mi.t_generate_into(lo.view(torch.uint32), n, "u32", "uniform", seed=2, block=1 << 27)
src = (hi.to(torch.int64) << 32) | (lo.to(torch.int64) & 0xFFFFFFFF)
del hi, lo
work = torch.empty_like(src)
ctx = ms.Context(1, n, "u64", device_ids=[0])
tot = ps = 0.0; pc = 0
for r in range(reps + 2):
    work.copy_(src)
    ctx.sort_device([ms.tensor_ptr(work)], n)
    t = ctx.timings()
    if r >= 2:
        tot += t["sort_ms"]; ps += t["pass_ms_sum"]; pc += t["passes_run"]
print(json.dumps({"n": n, "kt": "u64", "dist": "zipf_hi", "sort_ms": tot / reps, "pass_ms": ps / pc, "hist_ms": 0.0}))
