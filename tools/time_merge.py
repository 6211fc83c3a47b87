"""Merge kernel (S6) timing through the C ABI (msort_step_merge): two sorted
runs of total keys, CUDA events, GB/s = 2*K*total (read both runs + write) per
launch.  Usage: python tools/time_merge.py TOTAL KT [REPS] [SPLIT]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import msort_inputs as mi
import paper_conf_sigmod_maltenbergeritr22_b200 as ms

total = int(float(sys.argv[1]))
kt = sys.argv[2] if len(sys.argv) > 2 else "u32"
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 10
split = float(sys.argv[4]) if len(sys.argv) > 4 else 0.5
K = mi.KEY_BYTES[kt]
al = int(total * split)
bl = total - al
dt = torch.int32 if K == 4 else torch.int64
# sorted runs of unsigned codes (u32/u64 only: plain integer order of the bit patterns)
g = torch.Generator(device="cuda").manual_seed(1)
def run(n):
    x = torch.randint(0, 2**31 - 1 if K == 4 else 2**62, (n,), device="cuda", dtype=torch.int64, generator=g)
    return torch.sort(x)[0].to(dt)
a, b = run(al), run(bl)
out = torch.empty(total, dtype=dt, device="cuda")
wsb = ms.msort_merge_workspace_bytes(total, kt)
ws = torch.empty(wsb, dtype=torch.uint8, device="cuda")
st = torch.cuda.current_stream()
def once():
    ms.msort_step_merge(ms.tensor_ptr(a), al, ms.tensor_ptr(b), bl, ms.tensor_ptr(out), kt, ms.tensor_ptr(ws), wsb,
                        stream=st)
for _ in range(3):
    once()
torch.cuda.synchronize()
ok = bool(torch.equal(out, torch.sort(torch.cat([a, b]))[0]))
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record(st)
for _ in range(reps):
    once()
e1.record(st)
torch.cuda.synchronize()
ms_per = e0.elapsed_time(e1) / reps
print(json.dumps({"total": total, "kt": kt, "split": split, "version": "default",
                  "ms": ms_per, "gbs": 2 * K * total / (ms_per / 1e3) / 1e9, "ok": ok}))
