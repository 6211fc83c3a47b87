"""A/B of msort_sort_host on one GPU: MSORT_OPT_HOST_PIPELINE 1 vs 0, interleaved in one
process (PCIe / host-memory rates vary between boxes, so only same-process pairs compare).
usage: python tools/time_e2e.py N KT REPS"""
import os, sys, json, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import msort_inputs as mi
import paper_conf_sigmod_maltenbergeritr22_b200 as ms
n = int(float(sys.argv[1])); kt = sys.argv[2]; reps = int(sys.argv[3]) if len(sys.argv) > 3 else 3
if len(sys.argv) > 4 and sys.argv[4] == "numa":  # pin to the GPU's NUMA-local CPUs before any host allocation
    import pynvml
    pynvml.nvmlInit()
    h = pynvml.nvmlDeviceGetHandleByIndex(0)
    words = pynvml.nvmlDeviceGetCpuAffinity(h, (os.cpu_count() + 63) // 64)
    cpus = {w * 64 + b for w, m in enumerate(words) for b in range(64) if (m >> b) & 1}
    print(json.dumps({"affinity_before": len(os.sched_getaffinity(0)), "gpu_local_cpus": len(cpus)}))
    os.sched_setaffinity(0, cpus & os.sched_getaffinity(0) or cpus)
src = torch.empty(n, dtype=mi.torch_dtype(kt), device="cuda")
mi.t_generate_into(src, n, kt, "uniform", seed=1, block=1 << 27)
pristine = src.cpu()
del src
host = torch.empty(n, dtype=pristine.dtype, pin_memory=True)
ctx = ms.Context(1, n, kt, device_ids=[0])
res = {0: [], 1: []}
for r in range(reps + 1):
    for pipe in (1, 0):
        ctx.set_option(ms.MSORT_OPT_HOST_PIPELINE, pipe)
        host.copy_(pristine)
        t0 = time.perf_counter()
        ctx.sort_host(ms.tensor_ptr(host), n)
        el = time.perf_counter() - t0
        t = ctx.timings()
        if r > 0:
            res[pipe].append({"wall_ms": el * 1e3, "h2d": t["h2d_ms"], "sort": t["sort_ms"], "merge": t["merge_ms"],
                              "d2h": t["d2h_ms"], "total": t["total_ms"]})
for pipe in (1, 0):
    avg = {k: sum(x[k] for x in res[pipe]) / len(res[pipe]) for k in res[pipe][0]}
    print(json.dumps({"pipeline": pipe, "n": n, "kt": kt, **{k: round(v, 2) for k, v in avg.items()},
                      "gkeys_s": n / avg["wall_ms"] / 1e6}))
