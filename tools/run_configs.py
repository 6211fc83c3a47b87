"""Device-resident timing of every BASELINE.json config on ONE GPU (chunks of
g > 1 configs run as virtual ranks: the same g-chunk algorithm, 'peer' reads are
local HBM reads, so stage times are not NVLink numbers).  One JSON line each.
Parity at these sizes is tests/test_gpu_fullsize.py; this tool only times.
Usage: python tools/run_configs.py [REPS]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import msort_inputs as mi
import paper_conf_sigmod_maltenbergeritr22_b200 as ms

REPS = int(sys.argv[1]) if len(sys.argv) > 1 else 3
CONFIGS = [  # (BASELINE.json configs index, n, g, key type, distribution, exchange)
    (0, 1 << 20, 1, "u32", "uniform", 0),
    (1, 1 << 28, 2, "u32", "uniform", 0),
    (2, 4_000_000_000, 1, "u32", "uniform", 0),
    (2, 4_000_000_000, 2, "u32", "uniform", 0),
    (2, 4_000_000_000, 2, "u32", "uniform", 2),
    (2, 4_000_000_000, 4, "u32", "uniform", 0),
    (2, 4_000_000_000, 4, "u32", "uniform", 2),
    (2, 4_000_000_000, 8, "u32", "uniform", 0),
    (2, 4_000_000_000, 8, "u32", "uniform", 2),
    (3, 2_000_000_000, 8, "u32", "zipf", 0),
    (3, 2_000_000_000, 8, "u32", "sorted", 0),
    (3, 2_000_000_000, 8, "u32", "reverse", 0),
    (3, 2_000_000_000, 8, "u32", "nearly", 0),
    (3, 2_000_000_000, 8, "u32", "zipf", 2),
    (3, 2_000_000_000, 8, "u32", "reverse", 2),
    (4, 2_000_000_000, 8, "u64", "uniform", 0),
    (4, 2_000_000_000, 8, "u64", "uniform", 2),
    (4, 2_000_000_000, 8, "f32", "uniform", 0),
    (4, 2_000_000_000, 8, "f32", "uniform", 2),
    (1, 1 << 28, 2, "u32", "uniform", 1),        # the paper's copy-then-merge swap
    (1, 1 << 28, 2, "u32", "uniform", 4),        # the NCCL send/recv swap (self p2p on one GPU)
    (3, 2_000_000_000, 8, "u32", "reverse", 4),
    (3, 2_000_000_000, 8, "u32", "normal", 0),
]
only = os.environ.get("CONFIGS")
for idx, n, g, kt, dist, ex in CONFIGS:
    if only and str(idx) not in only.split(","):
        continue
    c = n // g
    src = [torch.empty(c, dtype=mi.torch_dtype(kt), device="cuda") for _ in range(g)]
    for i in range(g):
        mi.t_generate_into(src[i], n, kt, dist, seed=1, start=i * c, block=1 << 27)
    work = [torch.empty_like(s) for s in src]
    ctx = ms.Context(g, n, kt, device_ids=[0] * g)
    ctx.set_option(ms.MSORT_OPT_EXCHANGE, ex)
    st = torch.cuda.current_stream()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    times, tm = [], None
    for r in range(REPS + 2):
        for w, s in zip(work, src):
            w.copy_(s)
        e0.record(st)
        ctx.sort_device([ms.tensor_ptr(w) for w in work], c, streams=[st] * g)
        e1.record(st)
        torch.cuda.synchronize()
        if r >= 2:
            times.append(e0.elapsed_time(e1))
            tm = ctx.timings()
    ms_avg = sum(times) / len(times)
    print(json.dumps({"config": idx, "n": n, "g": g, "kt": kt, "dist": dist, "exchange": ex, "ms": ms_avg,
                      "keys_per_s": n / (ms_avg / 1e3), "sort_ms": tm["sort_ms"], "merge_ms": tm["merge_ms"],
                      "stage_label": tm["stage_label"], "stage_max_x": tm["stage_max_x"],
                      "stage_ms": [round(x, 3) for x in tm["stage_ms"]],
                      "stage_swap_ms": [round(x, 3) for x in tm["stage_swap_ms"]],
                      "exchange_mode_run": tm["exchange_mode"], "virtual_ranks": g > 1}), flush=True)
    ctx.close()
    del src, work
    torch.cuda.empty_cache()
