"""msort_sort (north-star entry) on PAGEABLE host memory (numpy) vs pinned, one GPU.
usage: time_pageable.py N"""
import os, sys, time, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import msort_inputs as mi
import paper_conf_sigmod_maltenbergeritr22_b200 as ms
n = int(float(sys.argv[1]))
src = torch.empty(n, dtype=torch.int32, device="cuda")
mi.t_generate_into(src.view(torch.uint32), n, "u32", "uniform", seed=1, block=1 << 27)
host_np = src.cpu().numpy()
pinned = torch.empty(n, dtype=torch.int32, pin_memory=True)
res = {"n": n}
for rep, kind in enumerate(("pageable", "pinned", "pageable", "pinned")):
    if kind == "pageable":
        a = host_np.copy(); ptr = a.ctypes.data
    else:
        pinned.copy_(torch.from_numpy(host_np)); ptr = pinned.data_ptr()
    t0 = time.perf_counter()
    ms.msort_sort(ptr, n, "u32", 1)
    el = time.perf_counter() - t0
    res[f"{kind}_{rep // 2}"] = {"s": el, "gkeys_s": n / el / 1e9}
print(json.dumps(res))
