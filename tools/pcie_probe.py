"""PCIe copy-rate probe: 16 GB pinned H2D / D2H as one copy vs split over 2 / 4 streams."""
import time, json, torch
n = 4_000_000_000
h = torch.empty(n, dtype=torch.int32, pin_memory=True)
h.fill_(1)
d = torch.empty(n, dtype=torch.int32, device="cuda")
for direction in ("h2d", "d2h"):
    for k in (1, 2, 4):
        sts = [torch.cuda.Stream() for _ in range(k)]
        best = 1e9
        for rep in range(3):
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            step = n // k
            for i, s in enumerate(sts):
                lo, hi = i * step, (n if i == k - 1 else (i + 1) * step)
                with torch.cuda.stream(s):
                    if direction == "h2d":
                        d[lo:hi].copy_(h[lo:hi], non_blocking=True)
                    else:
                        h[lo:hi].copy_(d[lo:hi], non_blocking=True)
            torch.cuda.synchronize()
            best = min(best, time.perf_counter() - t0)
        print(json.dumps({"dir": direction, "streams": k, "ms": best * 1e3, "GB_s": 16e9 / best / 1e9}), flush=True)
