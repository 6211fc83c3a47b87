"""Virtual-rank P2P sort timing on one GPU: g chunks on cuda:0 (merge kernels read
'peer' chunks that are local).  Prints per-phase and per-stage times."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import msort_inputs as mi
import paper_conf_sigmod_maltenbergeritr22_b200 as ms
n = int(float(sys.argv[1])); g = int(sys.argv[2]); kt = sys.argv[3] if len(sys.argv) > 3 else "u32"
dist = sys.argv[4] if len(sys.argv) > 4 else "uniform"
exch = int(sys.argv[5]) if len(sys.argv) > 5 else 0
reps = 3
c = n // g
K = mi.KEY_BYTES[kt]
src = [torch.empty(c, dtype=mi.torch_dtype(kt), device="cuda") for _ in range(g)]
for i in range(g):
    mi.t_generate_into(src[i], n, kt, dist, seed=1, start=i * c, block=1 << 27)
work = [torch.empty_like(s) for s in src]
ctx = ms.Context(g, n, kt, device_ids=[0] * g)
ctx.set_option(ms.MSORT_OPT_EXCHANGE, exch)
acc = None
for r in range(reps + 1):
    for w, s in zip(work, src):
        w.copy_(s)
    torch.cuda.synchronize()
    ctx.sort_device([ms.tensor_ptr(w) for w in work], c)
    t = ctx.timings()
    if r == 0:
        continue
    if acc is None:
        acc = {k: (list(v) if isinstance(v, list) else v) for k, v in t.items()}
        for k in ("sort_ms", "merge_ms", "stage_ms", "stage_exchange_ms"):
            acc[k] = t[k] if not isinstance(t[k], list) else list(t[k])
    else:
        acc["sort_ms"] += t["sort_ms"]; acc["merge_ms"] += t["merge_ms"]
        acc["stage_ms"] = [a + b for a, b in zip(acc["stage_ms"], t["stage_ms"])]
        acc["stage_exchange_ms"] = [a + b for a, b in zip(acc["stage_exchange_ms"], t["stage_exchange_ms"])]
out = {"n": n, "g": g, "kt": kt, "dist": dist, "exchange": exch, "sort_ms": acc["sort_ms"] / reps, "merge_ms": acc["merge_ms"] / reps,
       "stage_label": acc["stage_label"], "stage_max_x": acc["stage_max_x"],
       "stage_ms": [x / reps for x in acc["stage_ms"]], "stage_exchange_ms": [x / reps for x in acc["stage_exchange_ms"]],
       "gkeys_s": n / ((acc["sort_ms"] + acc["merge_ms"]) / reps / 1e3) / 1e9}
# merge kernel HBM: every merging rank reads c keys and writes c keys
tot_ms = sum(out["stage_exchange_ms"])
out["merge_phase_gbs_if_all_merge"] = (2 * K * n * len(out["stage_label"])) / (sum(out["stage_ms"]) / 1e3) / 1e9 if out["stage_ms"] else None
print(json.dumps(out))
