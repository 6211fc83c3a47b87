"""Latency of small one-GPU device sorts, MSORT_OPT_SMALL_GRAPH on vs off,
interleaved in one process.  usage: python tools/time_small.py N KT REPS"""
import os, sys, json, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import msort_inputs as mi
import paper_conf_sigmod_maltenbergeritr22_b200 as ms
n = int(float(sys.argv[1])); kt = sys.argv[2]; reps = int(sys.argv[3]) if len(sys.argv) > 3 else 200
src = torch.empty(n, dtype=mi.torch_dtype(kt), device="cuda")
mi.t_generate_into(src, n, kt, "uniform", seed=1)
work = torch.empty_like(src)
ctx = ms.Context(1, n, kt, device_ids=[0])
out = {}
for graph in (1, 0, 1, 0):
    ctx.set_option(ms.MSORT_OPT_SMALL_GRAPH, graph)
    wall, dev = [], []
    for r in range(reps + 3):
        work.copy_(src)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        ctx.sort_device([ms.tensor_ptr(work)], n)
        el = time.perf_counter() - t0
        if r >= 3:
            wall.append(el * 1e3)
            dev.append(ctx.timings()["sort_ms"])
    wall.sort(); dev.sort()
    out[graph] = {"graph": graph, "n": n, "kt": kt, "wall_ms_median": wall[len(wall) // 2],
                  "device_ms_median": dev[len(dev) // 2], "keys_per_s_wall": n / (wall[len(wall) // 2] / 1e3)}
for g in (1, 0):
    print(json.dumps(out[g]))
