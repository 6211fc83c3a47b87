import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import numpy as np, torch
import msort_inputs as mi
from oracle import checks
import test_gpu_fullsize as T
n = 1 << 28; g = 2
chunks, c = T._gen_chunks(n, g, "u32", "uniform", 3)
a = np.concatenate([t.cpu().numpy() for t in chunks])
print("fp chunks", checks.fingerprint(a, "u32"))
tmp = torch.empty(T.BLOCK, dtype=torch.uint32, device="cuda")
parts = []
for off in range(0, n, T.BLOCK):
    cnt = min(T.BLOCK, n - off)
    mi.t_generate_into(tmp[:cnt], n, "u32", "uniform", seed=3, start=off, block=T.BLOCK)
    parts.append(tmp[:cnt].cpu().numpy())
b = np.concatenate(parts)
print("fp regen", checks.fingerprint(b, "u32"), "equal arrays", np.array_equal(a, b))
bad = np.nonzero(a != b)[0]; print(len(bad), bad[:5], a[bad[:3]], b[bad[:3]])
