"""bench.py's reference arm (the oracle on a bounded sample, this tier's `--impl reference`)
runs on CPU: one JSON line with the contract's keys, and under torchrun (N > 1) only rank 0
prints while the other ranks exit 0 without work (task contract, ④)."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
KEYS = {"impl", "metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
        "scaling", "vs_baseline", "dtype", "data", "config", "cpu_baseline", "e2e"}


def _lines(out):
    return [json.loads(x) for x in out.splitlines() if x.startswith("{")]


def test_reference_arm_one_process():
    r = subprocess.run([sys.executable, "bench.py", "--impl", "reference", "--keys", "2e5", "--steps", "2",
                        "--warmup", "1"], cwd=ROOT, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = _lines(r.stdout)
    assert len(lines) == 1
    d = lines[0]
    assert KEYS <= set(d), KEYS - set(d)
    assert d["impl"] == "reference" and d["metric"] == "keys/sec" and d["value"] > 0
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["d2h_bytes_per_step"] == 0
    assert d["e2e"]["value"] == d["value"] and d["e2e"]["unit"] == d["unit"]


def test_reference_arm_under_torchrun_prints_once():
    env = dict(os.environ, OMP_NUM_THREADS="1")
    r = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
                        "--master-addr", "127.0.0.1", "--master-port", "29561", "bench.py", "--impl", "reference",
                        "--gpus", "2", "--keys", "2e5", "--steps", "1", "--warmup", "1"],
                       cwd=ROOT, capture_output=True, text=True, timeout=600, env=env)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = _lines(r.stdout)
    assert len(lines) == 1 and lines[0]["impl"] == "reference" and lines[0]["n_gpus"] == 2


def _bench():
    import importlib.util
    spec = importlib.util.spec_from_file_location("bench_mod", os.path.join(ROOT, "bench.py"))
    b = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(b)
    return b


def test_nvlink_fraction_fields():
    """N > 1 lines carry the §8(d) S5 fractions: per Alg.2 stage the busiest mirrored pair's bytes over
    the stage's exchange time, against 900 GB/s and against the in-run measured mirrored-pair peak."""
    b = _bench()
    st = {"stage_label": [2, 4, 2], "stage_max_x": [100, 0, 50], "stage_exchange_ms": [0.001, 0.0, 0.002]}
    peaks = {"p2p_ce_gbs": 700.0, "p2p_sm_gbs": 800.0}
    r = b.nvlink_fractions(st, 4, peaks, False)
    assert {"per_stage", "achieved_gbs", "frac_of_900", "frac_of_measured_ce", "nominal_gbs", "measured_peaks",
            "note"} <= set(r)
    s0 = r["per_stage"][0]
    assert s0["busiest_pair_bytes"] == 400 and abs(s0["achieved_gbs"] - 400 / 1e3) < 1e-12
    assert abs(s0["frac_of_900"] - s0["achieved_gbs"] / 900) < 1e-12
    assert abs(s0["frac_of_measured_ce"] - s0["achieved_gbs"] / 700) < 1e-12
    assert r["per_stage"][1]["achieved_gbs"] is None          # a stage that moved nothing
    assert "NVLink" in r["note"] and "HBM" in b.nvlink_fractions(st, 4, peaks, True)["note"]


def test_output_verification_helpers():
    """bench.py verifies the timed output: sorted under T and a permutation of the input."""
    import numpy as np
    import torch
    import msort_inputs as mi
    from oracle import sort as osort
    b = _bench()
    for kt in ("u32", "u64", "f32", "f64"):
        a = mi.np_generate(5000, kt, "uniform", seed=3)
        inp = torch.from_numpy(a.copy())
        s = osort.oracle_sort(a, kt)
        good = torch.from_numpy(s.copy())
        r = b.verify_local(good, inp, len(a), kt, block=1024)
        assert b.verify_all(r, None)["verified"], kt
        x = s.copy()
        x[[10, 20]] = x[[20, 10]]                               # unsorted
        assert not b.verify_all(b.verify_local(torch.from_numpy(x), inp, len(a), kt, block=1024), None)["verified"], kt
        y = s.copy()
        y[-1] = y[-2]                                           # sorted, but not a permutation
        assert not b.verify_all(b.verify_local(torch.from_numpy(y), inp, len(a), kt, block=1024), None)["verified"], kt


def test_workload_names_the_baseline_config():
    """bench.py's `config.workload` names the BASELINE.json config it measures (the N=1 headline is configs[2])."""
    import importlib.util
    spec = importlib.util.spec_from_file_location("_bench", os.path.join(ROOT, "bench.py"))
    b = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(b)
    assert "configs[2]" in b.baseline_config_name(4_000_000_000, "u32", "uniform")
    assert "configs[4]" in b.baseline_config_name(2_000_000_000, "u64", "uniform")
    assert "configs[4]" in b.baseline_config_name(2_000_000_000, "f32", "uniform")
    assert "configs[3]" in b.baseline_config_name(2_000_000_000, "u32", "zipf")
    assert "configs[1]" in b.baseline_config_name(1 << 28, "u32", "uniform")
    assert "configs[0]" in b.baseline_config_name(1 << 20, "u32", "uniform")
    assert "not a BASELINE" in b.baseline_config_name(12345, "u32", "uniform")
