"""Time the radix sort (device-resident) of n keys on cuda:0; prints one line:
cfg n kt dist total_ms hist_ms pass_ms_avg GB/s(pass) frac."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
if os.environ.get("MSORT_PKG_ROOT"): sys.path.insert(0, os.environ["MSORT_PKG_ROOT"])
import torch
import msort_inputs as mi
import paper_conf_sigmod_maltenbergeritr22_b200 as ms
n = int(float(sys.argv[1])); kt = sys.argv[2]; dist = sys.argv[3] if len(sys.argv) > 3 else "uniform"
reps = int(sys.argv[4]) if len(sys.argv) > 4 else 5
src = torch.empty(n, dtype=mi.torch_dtype(kt), device="cuda")
mi.t_generate_into(src, n, kt, dist, seed=1, block=1 << 27)
work = torch.empty_like(src)
ctx = ms.Context(1, n, kt, device_ids=[0])
K = mi.KEY_BYTES[kt]
tot = hist = ps = 0.0; pc = 0
for r in range(reps + 2):
    work.copy_(src)
    ctx.sort_device([ms.tensor_ptr(work)], n)
    t = ctx.timings()
    if r >= 2:
        tot += t["sort_ms"]; hist += t["hist_ms"]; ps += t["pass_ms_sum"]; pc += t["passes_run"]
pavg = ps / pc
gbs = 2 * K * n / (pavg / 1e3) / 1e9
print(json.dumps({"cfg": os.environ.get("MSORT_OS_CFG", "0"), "n": n, "kt": kt, "dist": dist, "sort_ms": tot / reps,
                  "hist_ms": hist / reps, "hist_gbs": K * n / (hist / reps / 1e3) / 1e9, "pass_ms": pavg, "pass_gbs": gbs,
                  "pass_frac": gbs / 6554.2, "gkeys_s": n / (tot / reps / 1e3) / 1e9}))
