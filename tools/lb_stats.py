"""Look-back statistics from the MSORT_ABLATE=8 build (tools/ablate_build.py 8):
window rounds and polls per (tile, digit) of one radix sort of n keys."""
import ctypes, os, sys
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tools", "_ablate", "8"))
sys.path.insert(1, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import msort_inputs as mi
import paper_conf_sigmod_maltenbergeritr22_b200 as ms
n = int(float(sys.argv[1])); kt = sys.argv[2]; dist = sys.argv[3] if len(sys.argv) > 3 else "uniform"
src = torch.empty(n, dtype=mi.torch_dtype(kt), device="cuda")
mi.t_generate_into(src, n, kt, dist, seed=1, block=1 << 27)
ctx = ms.Context(1, n, kt, device_ids=[0])
st = (ctypes.c_ulonglong * 4)()
for r in range(3):
    ms._lib.msort_debug_lb_stats(st, 1)
    work = src.clone()
    ctx.sort_device([ms.tensor_ptr(work)], n)
    torch.cuda.synchronize()
    ms._lib.msort_debug_lb_stats(st, 1)
    print(f"{os.environ.get('MSORT_OS_CFG','0')} rep {r}: tile-digits {st[0]} rounds/td {st[1]/max(st[0],1):.3f} polls/td {st[2]/max(st[0],1):.3f}")
