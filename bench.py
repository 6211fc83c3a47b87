#!/usr/bin/env python3
"""bench.py - keys/s of the B200 P2P sort (BASELINE.json metric) in one JSON line.

Workload (BASELINE.json configs[2], paper Fig.1 shape): 4e9 uniform uint32 keys
(16 GB), sorted on N = 1/2/4/8 GPUs (strong scaling: the total is fixed).  A
"step" is one whole sort: per-GPU radix sort (S1-S3) and, for N > 1, the merge
phase: by default NEXT-1, the paper's future work for NVSwitch systems
(one all-to-all exchange fused into a local merge tree), with the
paper's own g-1 merge stages (Alg.2, S4-S7) timed beside it as `alg2`
(`--exchange 0` makes Alg.2 the measured path).

  value  device-resident keys/s: chunks already in HBM; CUDA events on the
         stream the sort is ordered on, max over ranks; the input is restored
         from a pristine copy between steps OUTSIDE the event pair (inputs are
         16 GB >> 126 MB L2, so no L2 flush is needed)
  e2e    the same metric through the public host-pointer API (msort_sort_host /
         msort_dist_sort_host): pinned host keys -> H2D -> sort -> D2H, timed
         per call; N = 1: the pipelined path (transfers overlapped with the
         sort), the sequential one interleaved with it as `e2e.sequential`
  roofline  dominant kernel = the onesweep pass (S3): algorithmic bytes
         2*K*c per launch / mean launch time (library CUDA events around each
         launch) vs MEASURED_PEAKS.json hbm_gbs
  cpu_baseline  the oracle (np.sort on T codes, single thread) on a bounded
         sample of the same workload, on this host

`--impl reference` times the oracle itself (the reference arm of this tier).
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

N_DEFAULT = 4_000_000_000
PEAKS_PATH = os.path.join(ROOT, "MEASURED_PEAKS.json")
FALLBACK_HBM = 6650.0
PAPER_CONTEXT = {
    "source": "PAPER.md P:124-141 (Fig.1), DGX A100, 16 GB = 4e9 ints, end-to-end",
    "thrust_1gpu_s": 1.47, "p2p_2gpu_s": 0.75, "p2p_4gpu_s": 0.45, "het_2gpu_s": 1.09, "het_4gpu_s": 0.75,
    "paradis_cpu_s": 2.25,
}


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="msort", choices=["msort", "reference"])
    ap.add_argument("--keys", dest="n", type=float, default=N_DEFAULT, help="total keys (default 4e9, BASELINE configs[2])")
    ap.add_argument("--key-type", default="u32")
    ap.add_argument("--dist", default="uniform")
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--seed", type=int, default=1)
    ap.add_argument("--exchange", type=int, default=None,
                    help="merge phase for N>1: 0 the paper's Alg.2 with fused exchange+merge, 1 Alg.2 swap then "
                         "merge (single process only), 2 (default for N>1) NEXT-1 - the paper's future work for "
                         "NVSwitch systems, P:3416-3424 - single all-to-all fused into the merge, 3 NEXT-1 pull then "
                         "merge. With 2 or 3, Alg.2 (0) is timed too and reported as `alg2`")
    ap.add_argument("--no-alg2", action="store_true", help="N>1: skip the Alg.2 comparison timing")
    ap.add_argument("--het", action="store_true", help="also time the HET-sort baseline (GPU chunk sort + CPU merge)")
    ap.add_argument("--het-chunks", type=int, default=8)
    ap.add_argument("--cpu-seconds", type=float, default=10.0)
    return ap.parse_args()


def hbm_peak():
    try:
        with open(PEAKS_PATH) as f:
            return float(json.load(f)["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return FALLBACK_HBM, "fallback (B200_PROFILING.md)"


class ClockSampler:
    """SM clocks and clock-event (throttle) reasons sampled through NVML every
    ~5 ms in a background thread during the timed region (the first sample is
    taken before the region opens, so even a 0.2 s region is covered);
    nvidia-smi is the fallback when NVML is unavailable."""

    NAMES = (("hw_slowdown", "nvmlClocksEventReasonHwSlowdown"),
             ("hw_thermal_slowdown", "nvmlClocksEventReasonHwThermalSlowdown"),
             ("sw_thermal_slowdown", "nvmlClocksEventReasonSwThermalSlowdown"),
             ("sw_power_cap", "nvmlClocksEventReasonSwPowerCap"),
             ("hw_power_brake", "nvmlClocksEventReasonHwPowerBrakeSlowdown"))

    def __init__(self, index: int, pci_bus_id: str | None = None):
        self.index = index
        self.pci = pci_bus_id
        self.rows = []  # (sm_mhz, max_mhz, reasons bitmask)
        self.stop = threading.Event()
        self.nv = None
        self.t = None

    def _handle(self):
        import pynvml as nv
        nv.nvmlInit()
        self.nv = nv
        if self.pci:
            try:
                return nv.nvmlDeviceGetHandleByPciBusId(self.pci)
            except Exception:
                pass
        return nv.nvmlDeviceGetHandleByIndex(self.index)

    def _sample(self, h):
        nv = self.nv
        sm = nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM)
        mx = nv.nvmlDeviceGetMaxClockInfo(h, nv.NVML_CLOCK_SM)
        rs = nv.nvmlDeviceGetCurrentClocksEventReasons(h)
        self.rows.append((float(sm), float(mx), int(rs)))

    def _loop(self, h):
        while not self.stop.is_set():
            try:
                self._sample(h)
            except Exception:
                pass
            self.stop.wait(0.005)

    def __enter__(self):
        try:
            h = self._handle()
            self._sample(h)
            self.t = threading.Thread(target=self._loop, args=(h,), daemon=True)
            self.t.start()
        except Exception:
            self.nv = None
            self._smi()
        return self

    def _smi(self):
        q = "clocks.sm,clocks.max.sm"
        try:
            r = subprocess.run(["nvidia-smi", "-i", str(self.index), f"--query-gpu={q}", "--format=csv,noheader,nounits"],
                               capture_output=True, text=True, timeout=20)
            sm, mx = [float(x) for x in r.stdout.strip().split(",")[:2]]
            self.rows.append((sm, mx, 0))
        except Exception:
            pass

    def __exit__(self, *a):
        self.stop.set()
        if self.t:
            self.t.join(timeout=2)
        if self.nv is None:
            self._smi()

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unavailable"]}
        sm = sorted(r[0] for r in self.rows)
        reasons = set()
        if self.nv is not None:
            for nm, attr in self.NAMES:
                bit = getattr(self.nv, attr, 0)
                if any(r[2] & bit for r in self.rows):
                    reasons.add(nm)
        return {"sm_mhz": sm[len(sm) // 2], "sm_max_mhz": max(r[1] for r in self.rows), "reasons": sorted(reasons),
                "samples": len(self.rows), "source": "nvml" if self.nv is not None else "nvidia-smi"}


def cpu_baseline(n_total: int, key_type: str, dist: str, seed: int, seconds: float):
    """The oracle as it stands (np.sort on T codes, one thread) on a bounded sample."""
    import numpy as np

    import msort_inputs as mi
    from oracle import sort as osort
    sample = min(n_total, 1 << 26)
    a = mi.np_generate(n_total, key_type, dist, seed=seed, start=0, count=sample)
    done, t0 = 0, time.perf_counter()
    while True:
        osort.oracle_sort(a, key_type)
        done += sample
        el = time.perf_counter() - t0
        if el >= seconds:
            break
    return {"value": done / el, "unit": "keys/s", "cores": 1, "kind": "oracle",
            "sample": f"first {sample} keys of the {n_total}-key {dist} {key_type} workload, "
                      f"oracle.sort.oracle_sort (np.sort of T codes) repeated {done // sample}x in {el:.1f} s"}


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    cb = cpu_baseline(args.n, args.key_type, args.dist, args.seed, max(1.0, args.cpu_seconds / 2))
    import numpy as np

    import msort_inputs as mi
    from oracle import sort as osort
    sample = min(args.n, 1 << 25)
    a = mi.np_generate(args.n, args.key_type, args.dist, seed=args.seed, start=0, count=sample)
    for _ in range(args.warmup):
        osort.oracle_sort(a, args.key_type)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        osort.oracle_sort(a, args.key_type)
    el = time.perf_counter() - t0
    v = sample * args.steps / el
    cb["value"] = v
    cb["sample"] = f"first {sample} keys of the {args.n}-key workload per step, oracle.sort.oracle_sort, 1 thread"
    print(json.dumps({
        "impl": "reference", "metric": "keys/sec", "value": v, "unit": "keys/s", "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * el / args.steps, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": args.key_type, "data": "synthetic",
        "config": {"workload": f"{args.n} {args.dist} {args.key_type} keys (sample of {sample} per step)",
                   "n": args.n, "key_type": args.key_type, "distribution": args.dist},
        "cpu_baseline": cb, "e2e": {"value": v, "unit": "keys/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }))


def main():
    args = parse()
    args.n = int(args.n)
    if args.impl == "reference":
        run_reference(args)
        return
    import numpy as np
    import torch

    import msort_inputs as mi
    import paper_conf_sigmod_maltenbergeritr22_b200 as ms

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus:
        if world == 1 and args.gpus > 1:
            raise SystemExit("--gpus N > 1 runs under torchrun (one process per GPU)")
    # MSORT_BENCH_SAME_GPU=1 maps every rank to cuda:0 (testing the N>1 path on a
    # one-GPU box: CUDA IPC works between processes on one device)
    if os.environ.get("MSORT_BENCH_SAME_GPU") == "1":
        local = 0
    torch.cuda.set_device(local)
    dist = None
    if world > 1:
        import torch.distributed as dist
        # plumbing only (IPC-handle all-gather, barriers, a max-reduce of the
        # step times): gloo is enough, the sort itself needs no collective
        dist.init_process_group("gloo")
    g = world
    kt = args.key_type
    K = mi.KEY_BYTES[kt]
    n = args.n
    c = ((n + g - 1) // g + 3) // 4 * 4
    n_valid_local = max(0, min(n - rank * c, c))
    dev = torch.device("cuda", local)
    tdt = mi.torch_dtype(kt)

    # --- input: this rank's chunk of the global seeded workload, generated on the GPU
    pristine = torch.empty(c, dtype=tdt, device=dev)
    mi.t_generate_into(pristine[:n_valid_local], n, kt, args.dist, seed=args.seed, start=rank * c, block=1 << 27)
    if n_valid_local < c:
        # reading Q3 padding: largest key under T
        pad = {"u32": -1, "u64": -1, "f32": 0x7FFFFFFF, "f64": 0x7FFFFFFFFFFFFFFF}[kt]
        pristine.view(torch.int32 if K == 4 else torch.int64)[n_valid_local:] = pad
    work = torch.empty_like(pristine)
    stream = torch.cuda.Stream(device=dev)

    if g == 1:
        ctx = ms.Context(1, c, kt, device_ids=[local])
        sort_dev = lambda: ctx.sort_device([ms.tensor_ptr(work)], c, streams=[stream])  # noqa: E731
    else:
        from paper_conf_sigmod_maltenbergeritr22_b200 import dist as mdist
        ctx = mdist.dist_context(rank, g, local, c, kt)
        sort_dev = lambda: ctx.sort(ms.tensor_ptr(work), c, stream=stream)  # noqa: E731
    if args.exchange is None:
        args.exchange = 2 if g > 1 else 0
    if g > 1:
        if args.exchange == 1:
            raise SystemExit("--exchange 1 (swap then merge) is a single-process option")
        ctx.set_option(ms.MSORT_OPT_EXCHANGE, args.exchange)

    def barrier():
        torch.cuda.synchronize()
        if dist:
            dist.barrier()

    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    # warm-up (untimed)
    for _ in range(args.warmup):
        with torch.cuda.stream(stream):
            work.copy_(pristine)
        sort_dev()
    barrier()
    pass_ms, pass_cnt, stage_info, launches = 0.0, 0, None, 0
    hist_ms = 0.0
    try:
        pp = torch.cuda.get_device_properties(dev)
        pci = f"{pp.pci_domain_id:08X}:{pp.pci_bus_id:02X}:{pp.pci_device_id:02X}.0"
    except Exception:
        pci = None
    with ClockSampler(local, pci) as clk:
        barrier()
        t_wall = time.perf_counter()
        for i in range(args.steps):
            with torch.cuda.stream(stream):
                work.copy_(pristine)      # restore input: outside the event pair
                ev[i][0].record(stream)
            sort_dev()
            with torch.cuda.stream(stream):
                ev[i][1].record(stream)
            tm = ctx.timings()
            pass_ms += tm["pass_ms_sum"]
            pass_cnt += tm["passes_run"]
            hist_ms += tm["hist_ms"]
            stage_info = tm
            launches += tm["kernel_launches"]
        barrier()
        wall = time.perf_counter() - t_wall
    step_ms = [a.elapsed_time(b) for a, b in ev]
    tot = sum(step_ms)
    if dist:
        tt = torch.tensor([tot], dtype=torch.float64)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        tot = float(tt.item())
    ms_per_step = tot / args.steps
    value = n / (ms_per_step / 1e3)

    # --- N>1 with NEXT-1: the paper's own merge phase (Alg.2) timed the same way, as context
    alg2 = None
    if g > 1 and args.exchange in (2, 3) and not args.no_alg2:
        ctx.set_option(ms.MSORT_OPT_EXCHANGE, 0)
        for _ in range(2):
            with torch.cuda.stream(stream):
                work.copy_(pristine)
            sort_dev()
        barrier()
        ev2 = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
        for i in range(args.steps):
            with torch.cuda.stream(stream):
                work.copy_(pristine)
                ev2[i][0].record(stream)
            sort_dev()
            with torch.cuda.stream(stream):
                ev2[i][1].record(stream)
        barrier()
        t2 = sum(a.elapsed_time(b) for a, b in ev2)
        tt = torch.tensor([t2], dtype=torch.float64)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        ms2 = float(tt.item()) / args.steps
        at = ctx.timings()
        alg2 = {"value": n / (ms2 / 1e3), "unit": "keys/s", "ms_per_step": ms2,
                "exchange": "Alg.2 (paper P:1763-1854), fused peer-read merge", "merge_phase_ms": at["merge_ms"],
                "stage_label": at["stage_label"], "stage_max_x": at["stage_max_x"]}
        ctx.set_option(ms.MSORT_OPT_EXCHANGE, args.exchange)

    # --- roofline of the dominant kernel (onesweep pass)
    peak, peak_src = hbm_peak()
    pass_avg_ms = pass_ms / max(1, pass_cnt)
    alg_bytes = 2 * K * c
    achieved = alg_bytes / (pass_avg_ms / 1e3) / 1e9 if pass_avg_ms > 0 else None
    traffic = None
    smem_pipe = None
    # one capture per key type: onesweep_traffic.json (u32), onesweep_traffic_<kt>.json (others)
    prof = os.path.join(ROOT, "profiles", "onesweep_traffic.json" if kt == "u32" else f"onesweep_traffic_{kt}.json")
    if os.path.exists(prof):
        try:
            with open(prof) as f:
                pj = json.load(f)
            if pj.get("keys_per_launch") and pj.get("key_type", "u32") == kt:  # (a capture of the same key type only)
                traffic = pj["dram_bytes_per_launch"] * c / pj["keys_per_launch"]
                if pj.get("smem_wavefronts_per_32_keys"):
                    # the pass's binding resource (ncu, same capture): shared-memory wavefronts
                    smem_pipe = {"wavefronts_per_32_keys": pj["smem_wavefronts_per_32_keys"],
                                 "pct_of_peak": pj.get("smem_wavefronts_pct_of_peak_sustained_elapsed"),
                                 "bank_conflicts_per_launch": pj.get("smem_bank_conflicts_per_launch"),
                                 "source": os.path.relpath(prof, ROOT) + " (ncu --set full capture)"}
        except Exception:
            traffic = None
    roofline = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                "frac": (achieved / peak) if achieved else None, "traffic": traffic,
                "kernel": "onesweep_kernel (S3 pass)", "alg_bytes_per_launch": alg_bytes,
                "mean_launch_ms": pass_avg_ms, "peak_source": peak_src, "smem_pipe": smem_pipe,
                "whole_sort_hbm_frac": ((1 + 2 * (K * 8 // 8)) * K * c / (ms_per_step / 1e3) / 1e9 / peak) if g == 1 else None}

    # --- end to end through the public host API
    e2e = None
    if not args.no_e2e and args.e2e_steps > 0:
        host = torch.empty(c if g > 1 else n, dtype=tdt, pin_memory=True)
        host_pristine = pristine[: (c if g > 1 else n)].cpu()
        # one GPU: the pipelined host path (MSORT_OPT_HOST_PIPELINE, the default)
        # is the e2e number; the sequential path (H2D, sort, D2H one after the
        # other) runs interleaved with it in the same process as context (PCIe
        # and host-memory rates differ between boxes, so only same-run pairs compare)
        variants = (1, 0) if g == 1 else (None,)
        times = {v: [] for v in variants}
        phases = {}
        for i in range(args.e2e_steps + 1):
            for v in variants:
                if v is not None:
                    ctx.set_option(ms.MSORT_OPT_HOST_PIPELINE, v)
                host.copy_(host_pristine)
                barrier()
                t0 = time.perf_counter()
                if g == 1:
                    ctx.sort_host(ms.tensor_ptr(host), n)
                else:
                    ctx.sort_host(ms.tensor_ptr(host), c)
                el = time.perf_counter() - t0
                if dist:
                    tt = torch.tensor([el], dtype=torch.float64)
                    dist.all_reduce(tt, op=dist.ReduceOp.MAX)
                    el = float(tt.item())
                if i > 0:
                    times[v].append(el)
                    et = ctx.timings()
                    phases[v] = {"h2d": et["h2d_ms"], "sort": et["sort_ms"], "merge": et["merge_ms"], "d2h": et["d2h_ms"]}
        main = variants[0]
        tm = sum(times[main]) / len(times[main])
        e2e = {"value": n / tm, "unit": "keys/s", "h2d_bytes_per_step": n * K,
               "d2h_bytes_per_step": n * K, "ms_per_step": 1e3 * tm, "phases_ms": phases[main],
               "steps": len(times[main])}
        if g == 1:
            e2e["path"] = "pipelined (4 H2D pieces sorted as they land, sliced final merge overlapped with D2H)"
            ts = sum(times[0]) / len(times[0])
            e2e["sequential"] = {"value": n / ts, "ms_per_step": 1e3 * ts, "phases_ms": phases[0]}
        del host, host_pristine

    cpu = None
    if rank == 0 and g == 1 and not args.no_cpu:
        cpu = cpu_baseline(n, kt, args.dist, args.seed, args.cpu_seconds)

    het = None
    if args.het and g == 1:
        from baseline import het as hetmod
        hk = pristine[:n].cpu().pin_memory()
        hetmod.het_sort_host(hk, kt, chunks=args.het_chunks)           # warm-up (allocations, OpenMP start)
        hk.copy_(pristine[:n].cpu())
        info = hetmod.het_sort_host(hk, kt, chunks=args.het_chunks)
        het = {"value": n / info["total_s"], "unit": "keys/s", "kind": "HET sort (paper §5.3): libmsort radix per "
               f"chunk on 1 GPU + D2H + CPU multiway merge (libstdc++ parallel, {info['threads']} threads)",
               "chunks": info["chunks"], "gpu_sort_and_copies_s": info["gpu_sort_and_copies_s"],
               "cpu_merge_s": info["cpu_merge_s"]}
        del hk

    if rank == 0:
        out = {
            "metric": "keys/sec", "value": value, "unit": "keys/s", "n_gpus": g, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": kt, "data": "synthetic",
            "config": {"workload": f"{n} {args.dist} {kt} keys (BASELINE.json configs[2], paper Fig.1 shape), "
                                   f"device-resident P2P sort on {g} GPU(s)",
                       "n": n, "keys_per_gpu": c, "key_type": kt, "distribution": args.dist, "seed": args.seed,
                       "parallelism": f"p2p{g}", "l2": "inputs 16 GB >> 126 MB L2 (no flush needed)",
                       "exchange": ["Alg.2, fused peer-read merge", "Alg.2, swap then merge",
                                    "NEXT-1 single all-to-all fused into the merge", "NEXT-1 single all-to-all, pull then merge"][args.exchange] if g > 1 else "none (1 GPU)"},
            "roofline": roofline, "cpu_baseline": cpu, "e2e": e2e, "gpu_launches": launches,
            "clocks": clk.summary(), "wall_s_timed_region": wall,
            "step_ms": {"min": min(step_ms), "max": max(step_ms)},
            "phases_ms": {"hist": hist_ms / args.steps, "onesweep_passes": pass_ms / args.steps,
                          "merge_phase": stage_info["merge_ms"] if stage_info else None},
            "stages": {k: stage_info[k] for k in ("stage_label", "stage_pivot", "stage_max_x", "stage_ms",
                                                  "stage_exchange_ms")} if stage_info and g > 1 else None,
            "paper_context": PAPER_CONTEXT,
            "het_baseline": het,
            "alg2": alg2,
        }
        print(json.dumps(out))
    if dist:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
