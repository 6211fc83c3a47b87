#!/usr/bin/env python3
"""bench.py - keys/s of the B200 P2P sort (BASELINE.json metric) in one JSON line.

Workload (BASELINE.json configs[2], paper Fig.1 shape): 4e9 uniform uint32 keys
(16 GB), sorted on N = 1/2/4/8 GPUs (strong scaling: the total is fixed).  A
"step" is one whole sort: per-GPU radix sort (S1-S3) and, for N > 1, the merge
phase - the paper's g-1 merge stages (Alg.2, S4-S7) with the
exchange fused into the merge and every stage decided on the GPUs; NEXT-1, the
paper's future work for NVSwitch systems (one all-to-all exchange),
is timed beside it as `next1` with equal standing (`--exchange 2` makes it the
headline).

  value  device-resident keys/s: chunks already in HBM; CUDA events on the
         stream the sort is ordered on, max over ranks; the input is restored
         from a pristine copy between steps OUTSIDE the event pair (inputs are
         16 GB >> 126 MB L2, so no L2 flush is needed); the output of the last
         step is verified (sorted + multiset fingerprint) -> `verified`
  e2e    the same metric through the public host-pointer API (msort_sort_host /
         msort_dist_sort_host): pinned host keys -> H2D -> sort -> D2H, timed
         per call; N = 1: the pipelined path (transfers overlapped with the
         sort), the sequential one interleaved with it as `e2e.sequential`;
         `e2e.pcie` = the achieved H2D / D2H rates against the in-run measured
         parallel PCIe peaks (msort_measure_links, P:664-709 pattern)
  roofline  dominant kernel = the onesweep pass (S3): algorithmic bytes
         2*K*c per launch / mean launch time (library CUDA events around each
         launch) vs MEASURED_PEAKS.json hbm_gbs
  nvlink N > 1: per Alg.2 stage the busiest mirrored pair's bytes (x_d * K) /
         the stage's exchange time (max over ranks) against 900 GB/s per
         direction and against the in-run measured mirrored-pair peak
         (msort_measure_links: GPU i <-> GPU g-1-i concurrently)
  cpu_baseline  the oracle (np.sort on T codes, single thread) on a bounded
         sample of the same workload, on this host; `.parallel` = GNU parallel
         mode's sort on all host cores on a >= 2^28-key sample

`--impl reference` times the oracle itself (the reference arm of this tier).
"""
from __future__ import annotations

import argparse
import json
import os
import platform
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

N_DEFAULT = 4_000_000_000
PEAKS_PATH = os.path.join(ROOT, "MEASURED_PEAKS.json")
FALLBACK_HBM = 6650.0
NVLINK_NOMINAL_GBS = 900.0  # NVLink 5 per direction per GPU (north_star)
EXCHANGE_NAMES = ["Alg.2, fused peer-read merge, stages decided on the GPUs", "Alg.2, swap then merge",
                  "NEXT-1 single all-to-all fused into the merge", "NEXT-1 single all-to-all, pull then merge"]
PAPER_CONTEXT = {
    "source": "PAPER.md P:124-141 (Fig.1), DGX A100, 16 GB = 4e9 ints, end-to-end",
    "thrust_1gpu_s": 1.47, "p2p_2gpu_s": 0.75, "p2p_4gpu_s": 0.45, "het_2gpu_s": 1.09, "het_4gpu_s": 0.75,
    "paradis_cpu_s": 2.25,
}


def parse(argv=None):
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
    ap.add_argument("--no-links", action="store_true", help="skip the interconnect peak measurement")
    ap.add_argument("--seed", type=int, default=1)
    ap.add_argument("--exchange", type=int, default=0,
                    help="merge phase for N>1: 0 (default) the paper's Alg.2, fused exchange+merge, decided on the "
                         "GPUs; 2 NEXT-1 (P:3416-3424) single all-to-all fused into the merge; 3 NEXT-1 pull then "
                         "merge. The other of {0, 2} is timed too and reported beside it")
    ap.add_argument("--no-compare", action="store_true", help="N>1: skip the second merge-phase variant")
    ap.add_argument("--no-nccl", action="store_true",
                    help="N>1: skip the NCCL send/recv swap (exchange mode 4) leg (only runs on distinct GPUs)")
    ap.add_argument("--het", action="store_true", help="also time the HET-sort baseline (GPU chunk sorts + CPU merge)")
    ap.add_argument("--het-chunks", type=int, default=8)
    ap.add_argument("--het-gpus", type=int, default=0, help="GPUs for the HET chunk sorts (0: all visible)")
    ap.add_argument("--het-ooc-chunk", type=float, default=0,
                    help="also time the out-of-core HET sort (NEXT-4, 2n-approach) with chunks of this many keys "
                         "(two chunk buffers per GPU: a device budget below the input)")
    ap.add_argument("--cpu-seconds", type=float, default=10.0)
    ap.add_argument("--cpu-parallel-keys", type=float, default=float(1 << 28))
    return ap.parse_args(argv)


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


class stdout_to_stderr:
    """fd-level redirect of stdout to stderr (NCCL prints its version line on stdout at init; the bench's
    stdout carries exactly one JSON line)."""

    def __enter__(self):
        sys.stdout.flush()
        self.saved = os.dup(1)
        os.dup2(2, 1)
        return self

    def __exit__(self, *a):
        sys.stdout.flush()
        os.dup2(self.saved, 1)
        os.close(self.saved)


def cpu_model() -> str:
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except Exception:
        pass
    return platform.processor() or "unknown"


def cpu_baseline(n_total: int, key_type: str, dist: str, seed: int, seconds: float):
    """The oracle as it stands (np.sort on T codes, one thread) on a bounded sample."""
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
    return {"value": done / el, "unit": "keys/s", "cores": 1, "kind": "oracle", "cpu_model": cpu_model(),
            "sample": f"first {sample} keys of the {n_total}-key {dist} {key_type} workload, "
                      f"oracle.sort.oracle_sort (np.sort of T codes) repeated {done // sample}x in {el:.1f} s"}


def cpu_parallel_baseline(pristine, n_total: int, key_type: str, count: int):
    """GNU parallel mode's sort (__gnu_parallel::sort, all host cores) on the first `count` keys of the
    workload (copied from the GPU-generated input); the paper's CPU library baseline family."""
    import torch

    from baseline import het
    count = int(min(count, pristine.numel()))
    host = torch.empty(count, dtype=pristine.dtype, pin_memory=True)
    src = pristine[:count].cpu()
    kt = {"u32": 0, "u64": 1, "f32": 2, "f64": 3}[key_type]
    times = []
    for _ in range(2):
        host.copy_(src)
        t0 = time.perf_counter()
        het.cpu_parallel_sort(host.data_ptr(), count, kt, 0)
        times.append(time.perf_counter() - t0)
    el = min(times)
    threads = het.max_threads()
    return {"value": count / el, "unit": "keys/s", "cores": threads, "kind": "__gnu_parallel::sort",
            "cpu_model": cpu_model(), "seconds": el,
            "sample": f"first {count} keys of the {n_total}-key workload, best of 2, {threads} OpenMP threads"}


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    cb = cpu_baseline(args.n, args.key_type, args.dist, args.seed, max(1.0, args.cpu_seconds / 2))
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


# --- output verification (torch on the GPU; a check of the timed result, not the product path) -------------

_MIX1, _MIX2 = -0x2917014799A6026D, -0x40A7B892E31B1A47  # 0xD6E8FEB86659FD93, 0xBF58476D1CE4E5B9 as int64


def _order_codes(x, kt):
    """int64 values whose signed order is the T order of the keys (reading Q1)."""
    import torch
    if kt in ("u32", "f32"):
        u = x.view(torch.int32).to(torch.int64) & 0xFFFFFFFF
        if kt == "f32":
            u = torch.where(u >= (1 << 31), u ^ 0xFFFFFFFF, u | (1 << 31))
        return u
    u = x.view(torch.int64)
    if kt == "f64":  # negatives: all bits flipped; then the unsigned order = signed order after a sign flip
        return torch.where(u < 0, ~u ^ (-(1 << 63)), u)
    return u ^ (-(1 << 63))


def _fingerprint(codes):
    import torch
    h1 = codes * _MIX1
    h1 = h1 ^ ((h1 >> 29) & ((1 << 35) - 1))
    h2 = (codes + 0x1234567) * _MIX2
    h2 = h2 ^ ((h2 >> 31) & ((1 << 33) - 1))
    return int(h1.sum().item()) % (1 << 64), int(h2.sum().item()) % (1 << 64), int(codes.numel())


def verify_local(out, inp, valid, kt, block=1 << 27):
    """This rank: out[:valid] non-decreasing under T, and the multiset fingerprint of out[:valid] and
    inp[:valid]; first / last codes for the cross-rank boundary check."""
    ok, last, first = True, None, None
    fo, fi = [0, 0, 0], [0, 0, 0]
    for off in range(0, valid, block):
        hi = min(valid, off + block)
        c = _order_codes(out[off:hi], kt)
        ok = ok and bool((c[1:] >= c[:-1]).all().item()) and (last is None or last <= int(c[0].item()))
        first = int(c[0].item()) if first is None else first
        last = int(c[-1].item())
        a = _fingerprint(c)
        b = _fingerprint(_order_codes(inp[off:hi], kt))
        fo = [(fo[0] + a[0]) % (1 << 64), (fo[1] + a[1]) % (1 << 64), fo[2] + a[2]]
        fi = [(fi[0] + b[0]) % (1 << 64), (fi[1] + b[1]) % (1 << 64), fi[2] + b[2]]
    return {"sorted": ok, "first": first, "last": last, "fp_out": fo, "fp_in": fi}


def verify_all(local, dist):
    """Combine the ranks' verify_local results (rank order)."""
    parts = [local]
    if dist is not None:
        parts = [None] * dist.get_world_size()
        dist.all_gather_object(parts, local)
    ok = all(p["sorted"] for p in parts)
    prev = None
    for p in parts:
        if p["first"] is None:
            continue
        ok = ok and (prev is None or prev <= p["first"])
        prev = p["last"]

    def tot(k):
        return [sum(p[k][0] for p in parts) % (1 << 64), sum(p[k][1] for p in parts) % (1 << 64),
                sum(p[k][2] for p in parts)]
    ok = ok and tot("fp_out") == tot("fp_in")
    return {"verified": bool(ok), "method": "every rank's output non-decreasing under T, rank boundaries ordered, "
                                            "and out/in multiset fingerprints (2 x sum of mixed codes) equal"}


# --- interconnect fractions ---------------------------------------------------------------------------------

def nvlink_fractions(stages: dict, K: int, peaks: dict | None, same_device: bool):
    """Per merge stage: busiest mirrored pair's bytes / the stage's exchange time (fused modes: the
    exchange+merge kernel; copy / NCCL modes: pass the transfer-only time as stage_exchange_ms)."""
    rows = []
    for s, (lab, mx, ms) in enumerate(zip(stages["stage_label"], stages["stage_max_x"], stages["stage_exchange_ms"])):
        b = mx * K
        gbs = b / (ms * 1e6) if ms > 0 else None
        row = {"stage": s, "label": lab, "busiest_pair_bytes": b, "exchange_ms": ms, "achieved_gbs": gbs,
               "frac_of_900": (gbs / NVLINK_NOMINAL_GBS) if gbs else None}
        if peaks and peaks.get("p2p_ce_gbs"):
            row["frac_of_measured_ce"] = gbs / peaks["p2p_ce_gbs"] if gbs else None
            row["frac_of_measured_sm"] = gbs / peaks["p2p_sm_gbs"] if gbs and peaks.get("p2p_sm_gbs") else None
        rows.append(row)
    tot_b = sum(r["busiest_pair_bytes"] for r in rows)
    tot_ms = sum(r["exchange_ms"] for r in rows)
    agg = tot_b / (tot_ms * 1e6) if tot_ms > 0 else None
    return {"per_stage": rows, "busiest_pair_bytes_total": tot_b, "exchange_ms_total": tot_ms, "achieved_gbs": agg,
            "frac_of_900": (agg / NVLINK_NOMINAL_GBS) if agg else None,
            "frac_of_measured_ce": (agg / peaks["p2p_ce_gbs"]) if agg and peaks and peaks.get("p2p_ce_gbs") else None,
            "nominal_gbs": NVLINK_NOMINAL_GBS, "measured_peaks": peaks,
            "note": ("ranks share one GPU: the 'pairs' are HBM copies, not NVLink" if same_device else
                     "distinct GPUs: NVLink 5 through NVSwitch")}


def baseline_config_name(n: int, kt: str, dist: str) -> str:
    """Which BASELINE.json config a bench run measures (the N=1 headline is configs[2])."""
    if n == 4_000_000_000 and kt == "u32" and dist == "uniform":
        return "BASELINE.json configs[2], paper Fig.1 shape"
    if n == 2_000_000_000 and kt == "u32" and dist != "uniform":
        return "BASELINE.json configs[3] key distribution"
    if n == 2_000_000_000 and kt in ("u64", "f32"):
        return "BASELINE.json configs[4] key type"
    if n == 1 << 28 and kt == "u32":
        return "BASELINE.json configs[1] size"
    if n == 1 << 20 and kt == "u32":
        return "BASELINE.json configs[0] size"
    return "not a BASELINE.json configuration"


def main():
    args = parse()
    args.n = int(args.n)
    if args.impl == "reference":
        run_reference(args)
        return
    import torch

    import msort_inputs as mi
    import paper_conf_sigmod_maltenbergeritr22_b200 as ms

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus and world == 1 and args.gpus > 1:
        raise SystemExit("--gpus N > 1 runs under torchrun (one process per GPU)")
    # MSORT_BENCH_SAME_GPU=1 maps every rank to cuda:0 (testing the N>1 path on a
    # one-GPU box: CUDA IPC works between processes on one device)
    same_gpu = os.environ.get("MSORT_BENCH_SAME_GPU") == "1"
    if same_gpu:
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
    if g == 1:
        c, off, valid = n, 0, n
    else:
        c, off, valid = ms.msort_plan_chunk(n, g, rank)   # the library's chunking rule (reading Q3)
    dev = torch.device("cuda", local)
    tdt = mi.torch_dtype(kt)

    # --- input: this rank's slice of the global seeded workload, generated on the GPU (the library pads)
    pristine = torch.empty(c, dtype=tdt, device=dev)
    mi.t_generate_into(pristine[:valid], n, kt, args.dist, seed=args.seed, start=off, block=1 << 27)
    work = torch.empty_like(pristine)
    stream = torch.cuda.Stream(device=dev)

    if g == 1:
        ctx = ms.Context(1, c, kt, device_ids=[local])
        sort_dev = lambda: ctx.sort_device([ms.tensor_ptr(work)], n, streams=[stream])  # noqa: E731
    else:
        from paper_conf_sigmod_maltenbergeritr22_b200 import dist as mdist
        ctx = mdist.dist_context(rank, g, local, c, kt)
        sort_dev = lambda: ctx.sort(ms.tensor_ptr(work), n, stream=stream)  # noqa: E731
    if g > 1:
        if args.exchange == 1:
            raise SystemExit("--exchange 1 (swap then merge) is a single-process option")
        ctx.set_option(ms.MSORT_OPT_EXCHANGE, args.exchange)

    def barrier():
        torch.cuda.synchronize()
        if dist:
            dist.barrier()

    def max_over_ranks(x: float) -> float:
        if not dist:
            return x
        tt = torch.tensor([x], dtype=torch.float64)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        return float(tt.item())

    def timed_steps(steps):
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(steps)]
        acc = {"pass_ms": 0.0, "pass_cnt": 0, "hist_ms": 0.0, "launches": 0, "tm": None, "stage_x_ms": None}
        for i in range(steps):
            with torch.cuda.stream(stream):
                work.copy_(pristine)      # restore input: outside the event pair
                ev[i][0].record(stream)
            sort_dev()
            with torch.cuda.stream(stream):
                ev[i][1].record(stream)
            tm = ctx.timings()
            acc["pass_ms"] += tm["pass_ms_sum"]
            acc["pass_cnt"] += tm["passes_run"]
            acc["hist_ms"] += tm["hist_ms"]
            acc["launches"] += tm["kernel_launches"]
            acc["tm"] = tm
        barrier()
        step_ms = [a.elapsed_time(b) for a, b in ev]
        acc["step_ms"] = step_ms
        acc["ms_per_step"] = max_over_ranks(sum(step_ms)) / steps
        return acc

    # warm-up (untimed)
    for _ in range(args.warmup):
        with torch.cuda.stream(stream):
            work.copy_(pristine)
        sort_dev()
    barrier()
    try:
        pp = torch.cuda.get_device_properties(dev)
        pci = f"{pp.pci_domain_id:08X}:{pp.pci_bus_id:02X}:{pp.pci_device_id:02X}.0"
    except Exception:
        pci = None
    with ClockSampler(local, pci) as clk:
        barrier()
        t_wall = time.perf_counter()
        main_run = timed_steps(args.steps)
        wall = time.perf_counter() - t_wall
    ms_per_step = main_run["ms_per_step"]
    value = n / (ms_per_step / 1e3)
    stage_info = main_run["tm"]
    verify = verify_all(verify_local(work, pristine, valid, kt), dist)

    # --- N>1: the other merge phase (NEXT-1 beside Alg.2, or Alg.2 beside NEXT-1), timed the same way
    compare = None
    if g > 1 and not args.no_compare:
        other = 2 if args.exchange == 0 else 0
        try:  # (a failure here must not cost the headline line printed below)
            ctx.set_option(ms.MSORT_OPT_EXCHANGE, other)
            for _ in range(2):
                with torch.cuda.stream(stream):
                    work.copy_(pristine)
                sort_dev()
            barrier()
            r2 = timed_steps(args.steps)
            v2 = verify_all(verify_local(work, pristine, valid, kt), dist)
            at = r2["tm"]
            compare = {"value": n / (r2["ms_per_step"] / 1e3), "unit": "keys/s", "ms_per_step": r2["ms_per_step"],
                       "exchange": EXCHANGE_NAMES[other], "merge_phase_ms": max_over_ranks(at["merge_ms"]),
                       "stage_label": at["stage_label"], "stage_max_x": at["stage_max_x"],
                       "verified": v2["verified"]}
        except Exception as e:
            compare = {"failed": str(e)[:500]}
        ctx.set_option(ms.MSORT_OPT_EXCHANGE, args.exchange)

    # --- N>1 on distinct GPUs: the swap as NCCL send/recv (mode 4, the north star's S5 mechanism)
    nccl_leg = None
    if g > 1 and not args.no_nccl:
        if same_gpu and os.environ.get("MSORT_BENCH_FORCE_NCCL") != "1":  # (=1: exercise the refusal path)
            nccl_leg = {"unavailable": "ranks share one GPU (NCCL refuses two ranks of a communicator on one device)"}
        else:
            err = None
            try:
                with stdout_to_stderr():
                    obj = [ms.msort_nccl_unique_id() if rank == 0 else None]
                    dist.broadcast_object_list(obj, src=0)
                    ctx.nccl_init(obj[0])
            except Exception as e:  # (collective decision below: every rank runs the leg or none does)
                err = str(e)
            okt = torch.tensor([0 if err else 1], dtype=torch.int32)
            dist.all_reduce(okt, op=dist.ReduceOp.MIN)
            if int(okt.item()) == 0:
                nccl_leg = {"unavailable": err or "NCCL init failed on another rank"}
            else:
                try:  # (a failure here must not cost the headline line printed below)
                    ctx.set_option(ms.MSORT_OPT_EXCHANGE, 4)
                    for _ in range(2):
                        with torch.cuda.stream(stream):
                            work.copy_(pristine)
                        sort_dev()
                    barrier()
                    r4 = timed_steps(args.steps)
                    v4 = verify_all(verify_local(work, pristine, valid, kt), dist)
                    t4 = r4["tm"]
                    st4 = {"stage_label": t4["stage_label"], "stage_max_x": t4["stage_max_x"],
                           "stage_exchange_ms": [max_over_ranks(x) for x in t4["stage_swap_ms"]]}
                    nccl_leg = {"value": n / (r4["ms_per_step"] / 1e3), "unit": "keys/s",
                                "ms_per_step": r4["ms_per_step"],
                                "exchange": "Alg.2, swap as grouped ncclSend/ncclRecv per mirrored pair, then local merge",
                                "verified": v4["verified"], "swap_stage_ms": st4["stage_exchange_ms"], "stages": st4}
                except Exception as e:
                    nccl_leg = {"failed": str(e)[:500]}
            ctx.set_option(ms.MSORT_OPT_EXCHANGE, args.exchange)

    # --- interconnect peaks (msort_measure_links; every rank, collective in dist mode)
    peaks = None
    if not args.no_links:
        try:
            pk = ctx.measure_links(min(c * K, 1 << 30), 3)  # (1 GiB per copy: 8 ranks x 2 pinned buffers stay small)
            if dist:  # the slowest rank's rates
                for k in ("p2p_ce_gbs", "p2p_sm_gbs", "h2d_gbs", "d2h_gbs", "bidir_gbs"):
                    tt = torch.tensor([pk[k]], dtype=torch.float64)
                    dist.all_reduce(tt, op=dist.ReduceOp.MIN)
                    pk[k] = float(tt.item())
            pk["same_device"] = bool(same_gpu or pk.get("same_device") == 1)
            peaks = pk
        except ms.MsortError as e:
            peaks = {"error": str(e)}

    # --- roofline of the dominant kernel (onesweep pass)
    peak, peak_src = hbm_peak()
    pass_avg_ms = main_run["pass_ms"] / max(1, main_run["pass_cnt"])
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
                    smem_pipe = {"wavefronts_per_32_keys": pj["smem_wavefronts_per_32_keys"],
                                 "pct_of_peak": pj.get("smem_wavefronts_pct_of_peak_sustained_elapsed"),
                                 "bank_conflicts_per_launch": pj.get("smem_bank_conflicts_per_launch"),
                                 "source": os.path.relpath(prof, ROOT) + " (ncu --set full capture)"}
                    if pj.get("l1_pipe_wavefronts_per_32_keys"):
                        # the pass's binding resource: the SM's L1 data pipe (shared + global wavefronts)
                        smem_pipe["l1_data_pipe"] = {
                            "wavefronts_per_32_keys": pj["l1_pipe_wavefronts_per_32_keys"],
                            "global_wavefronts_per_32_keys": pj.get("l1_pipe_global_wavefronts_per_32_keys"),
                            "pct_busy": pj.get("l1_pipe_pct_of_peak_sustained_elapsed")}
        except Exception:
            traffic = None
    P = K  # passes (8-bit digits)
    radix_bytes = (1 + 2 * P) * K * c
    merging_stages = sum(1 for x in (stage_info["stage_max_x"] if g > 1 else []) if x) if g > 1 else 0
    roof_ms = (radix_bytes + merging_stages * 2 * K * c) / (peak * 1e9) * 1e3
    roofline = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                "frac": (achieved / peak) if achieved else None, "traffic": traffic,
                "kernel": "onesweep_kernel (S3 pass)", "alg_bytes_per_launch": alg_bytes,
                "mean_launch_ms": pass_avg_ms, "peak_source": peak_src, "smem_pipe": smem_pipe,
                "whole_sort_hbm_frac": roof_ms / ms_per_step,
                "whole_sort_model": "(radix (1+2P)K + 2K per merging stage) bytes per GPU / HBM peak / measured step"}

    nvlink = None
    if g > 1:
        st = {k: stage_info[k] for k in ("stage_label", "stage_max_x")}
        st["stage_exchange_ms"] = [max_over_ranks(x) for x in stage_info["stage_exchange_ms"]]
        nvlink = nvlink_fractions(st, K, peaks if peaks and "error" not in peaks else None, same_gpu)
        nvlink["time_basis"] = "fused exchange+merge kernel time per stage (the partner's block is read inside the merge)"
        if nccl_leg and "stages" in nccl_leg:
            nccl_leg["nvlink"] = nvlink_fractions(nccl_leg.pop("stages"), K,
                                                  peaks if peaks and "error" not in peaks else None, same_gpu)
            nccl_leg["nvlink"]["time_basis"] = "ncclSend/ncclRecv group time per stage (transfer only)"

    # --- end to end through the public host API
    e2e = None
    if not args.no_e2e and args.e2e_steps > 0:
        host = torch.empty(valid, dtype=tdt, pin_memory=True)
        host_pristine = pristine[:valid].cpu()
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
                ctx.sort_host(ms.tensor_ptr(host), n)
                el = max_over_ranks(time.perf_counter() - t0)
                if i > 0:
                    times[v].append(el)
                    et = ctx.timings()
                    phases[v] = {"h2d": max_over_ranks(et["h2d_ms"]), "sort": max_over_ranks(et["sort_ms"]),
                                 "merge": max_over_ranks(et["merge_ms"]), "d2h": max_over_ranks(et["d2h_ms"])}
        main_v = variants[0]
        tm = sum(times[main_v]) / len(times[main_v])
        ph = phases[main_v]
        e2e = {"value": n / tm, "unit": "keys/s", "h2d_bytes_per_step": n * K,
               "d2h_bytes_per_step": n * K, "ms_per_step": 1e3 * tm, "phases_ms": ph,
               "steps": len(times[main_v])}
        # PCIe: this rank's bytes over its H2D / D2H phase vs the measured parallel peaks
        pcie = {"h2d_gbs": valid * K / (ph["h2d"] * 1e6) if ph["h2d"] > 0 else None,
                "d2h_gbs": valid * K / (ph["d2h"] * 1e6) if ph["d2h"] > 0 else None,
                "serial_bound_ms": None}
        if peaks and "error" not in peaks:
            pcie["peak_h2d_gbs"], pcie["peak_d2h_gbs"] = peaks["h2d_gbs"], peaks["d2h_gbs"]
            pcie["frac_h2d"] = pcie["h2d_gbs"] / peaks["h2d_gbs"] if pcie["h2d_gbs"] else None
            pcie["frac_d2h"] = pcie["d2h_gbs"] / peaks["d2h_gbs"] if pcie["d2h_gbs"] else None
            # the e2e time can't beat moving the bytes in and then out at the measured rates
            pcie["serial_bound_ms"] = valid * K / (peaks["h2d_gbs"] * 1e6) + valid * K / (peaks["d2h_gbs"] * 1e6)
            pcie["e2e_frac_of_serial_bound"] = pcie["serial_bound_ms"] / (1e3 * tm)
        e2e["pcie"] = pcie
        if g == 1:
            e2e["path"] = "pipelined (4 H2D pieces sorted as they land, sliced final merge overlapped with D2H)"
            ts = sum(times[0]) / len(times[0])
            e2e["sequential"] = {"value": n / ts, "ms_per_step": 1e3 * ts, "phases_ms": phases[0]}
        del host, host_pristine

    cpu = None
    if rank == 0 and g == 1 and not args.no_cpu:
        cpu = cpu_baseline(n, kt, args.dist, args.seed, args.cpu_seconds)
        try:
            cpu["parallel"] = cpu_parallel_baseline(pristine[:valid], n, kt, int(args.cpu_parallel_keys))
        except Exception as e:  # (the HET/CPU helper library could not be built here)
            cpu["parallel"] = {"error": str(e)}

    het = None
    if args.het and g == 1:
        from baseline import het as hetmod
        ngpu = torch.cuda.device_count() if args.het_gpus <= 0 else min(args.het_gpus, torch.cuda.device_count())
        hs = hetmod.HetSort(n, kt, chunks=args.het_chunks, devices=list(range(ngpu)))
        hk = torch.empty(n, dtype=tdt, pin_memory=True)
        src = pristine[:n].cpu()
        hk.copy_(src)
        hs.run(hk)                                    # warm-up (OpenMP start)
        hk.copy_(src)
        info = hs.run(hk)
        het = {"value": n / info["total_s"], "unit": "keys/s", "kind": "HET sort (paper §5.3): libmsort radix per "
               f"chunk on {info['gpus']} GPU(s) + D2H + CPU multiway merge (libstdc++ parallel, "
               f"{info['threads']} threads); buffers pre-allocated", "chunks": info["chunks"], "gpus": info["gpus"],
               "gpu_sort_and_copies_s": info["gpu_sort_and_copies_s"], "cpu_merge_s": info["cpu_merge_s"]}
        del hk, src, hs

    het_ooc = None
    if args.het_ooc_chunk and g == 1:
        from baseline import het as hetmod
        ngpu = torch.cuda.device_count() if args.het_gpus <= 0 else min(args.het_gpus, torch.cuda.device_count())
        hk = torch.empty(n, dtype=tdt, pin_memory=True)
        ho = torch.empty(n, dtype=tdt, pin_memory=True)
        src = pristine[:n].cpu()
        ck = int(args.het_ooc_chunk)
        hk.copy_(src)
        hetmod.het_ooc_sort(hk, kt, ck, list(range(ngpu)), ho)     # warm-up (OpenMP start, allocations)
        hk.copy_(src)
        info = hetmod.het_ooc_sort(hk, kt, ck, list(range(ngpu)), ho)
        ok = bool(torch.equal(ho[:min(n, 1 << 20)].view(torch.uint8), work[:min(n, 1 << 20)].cpu().view(torch.uint8)))
        het_ooc = {"value": n / info["total_s"], "unit": "keys/s",
                   "kind": f"out-of-core HET (paper §5.3 2n-approach, NEXT-4) on {ngpu} GPU(s): chunks of {ck} keys, "
                           f"two chunk buffers per GPU ({2 * ck * K / 2**30:.1f} GiB), CPU multiway merge "
                           f"({info['threads']} threads)",
                   "chunks": info["chunks"], "chunk_groups": info["chunk_groups"],
                   "gpu_phase_s": info["gpu_phase_s"], "cpu_merge_s": info["merge_s"],
                   "prefix_matches_device_sort": ok}
        del hk, ho, src

    merge_phase_ms = max_over_ranks(stage_info["merge_ms"]) if stage_info else None
    if rank == 0:
        out = {
            "metric": "keys/sec", "value": value, "unit": "keys/s", "n_gpus": g, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": kt, "data": "synthetic",
            "config": {"workload": f"{n} {args.dist} {kt} keys ({baseline_config_name(n, kt, args.dist)}), "
                                   f"device-resident P2P sort on {g} GPU(s)",
                       "n": n, "keys_per_gpu": c, "key_type": kt, "distribution": args.dist, "seed": args.seed,
                       "parallelism": f"p2p{g}", "l2": "inputs 16 GB >> 126 MB L2 (no flush needed)",
                       "exchange": EXCHANGE_NAMES[args.exchange] if g > 1 else "none (1 GPU)",
                       "ranks_share_one_gpu": same_gpu},
            "verified": verify["verified"], "verify_method": verify["method"],
            "roofline": roofline, "cpu_baseline": cpu, "e2e": e2e, "gpu_launches": main_run["launches"],
            "clocks": clk.summary(), "wall_s_timed_region": wall,
            "step_ms": {"min": min(main_run["step_ms"]), "max": max(main_run["step_ms"]),
                        "median": sorted(main_run["step_ms"])[len(main_run["step_ms"]) // 2],
                        "mean_this_rank": sum(main_run["step_ms"]) / len(main_run["step_ms"])},
            "phases_ms": {"hist": main_run["hist_ms"] / args.steps,
                          "onesweep_passes": main_run["pass_ms"] / args.steps,
                          "merge_phase": merge_phase_ms},
            "stages": {k: stage_info[k] for k in ("stage_label", "stage_pivot", "stage_max_x", "stage_ms",
                                                  "stage_exchange_ms", "stage_pivot_ms")} if stage_info and g > 1 else None,
            "nvlink": nvlink, "links": peaks, "nccl_swap": nccl_leg,
            "paper_context": PAPER_CONTEXT,
            "het_baseline": het, "het_out_of_core": het_ooc,
            ("next1" if args.exchange == 0 else "alg2"): compare,
        }
        print(json.dumps(out))
    if dist:
        dist.barrier()
        dist.destroy_process_group()
    if not verify["verified"]:
        sys.exit(3)


if __name__ == "__main__":
    main()
