timeout 600 ncu --set full --clock-control none --import-source on -k regex:onesweep -s 5 -c 1 -o gpurun_out/os_cfg0 python tools/prof_radix.py 268435456 u32 2 > /dev/null 2>&1
MSORT_OS_CFG=1 timeout 600 ncu --set full --clock-control none --import-source on -k regex:onesweep -s 5 -c 1 -o gpurun_out/os_cfg1 python tools/prof_radix.py 268435456 u32 2 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:hist -s 1 -c 1 -o gpurun_out/hist_r2 python tools/prof_radix.py 268435456 u32 2 > /dev/null 2>&1
python - <<'PY'
import torch, time
for n in (10**9,):
    x = torch.randint(-2**31, 2**31-1, (n,), dtype=torch.int32, device="cuda")
    for dt in (torch.int32,):
        y = x.to(dt)
        for i in range(3): torch.sort(y)
        torch.cuda.synchronize()
        e0=torch.cuda.Event(enable_timing=True); e1=torch.cuda.Event(enable_timing=True)
        e0.record()
        for i in range(5): torch.sort(y)
        e1.record(); torch.cuda.synchronize()
        print("torch.sort (CUB) int32", n, e0.elapsed_time(e1)/5, "ms  (values+indices)")
        e0.record()
        for i in range(5): torch.sort(y, stable=True)
        e1.record(); torch.cuda.synchronize()
        print("torch.sort stable int32", n, e0.elapsed_time(e1)/5, "ms")
PY
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv python -c "
import torch
x = torch.randint(-2**31, 2**31-1, (10**9,), dtype=torch.int32, device='cuda')
torch.sort(x); torch.cuda.synchronize()
" 2>/dev/null | grep -v "^==" | tail -25 > gpurun_out/torch_sort_launches.csv
