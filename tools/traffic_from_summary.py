"""Write profiles/onesweep_traffic[_<kt>].json from an ncu_summary.py text (one onesweep launch).
usage: traffic_from_summary.py SUMMARY.txt KEY_TYPE KEYS_PER_LAUNCH SOURCE_NOTE OUT.json"""
import json, re, sys
txt, kt, n, note, out = sys.argv[1], sys.argv[2], float(sys.argv[3]), sys.argv[4], sys.argv[5]
t = open(txt).read()
g = lambda k: float(re.search(re.escape(k) + r"\s+([0-9.]+)", t).group(1))
K = 8 if kt in ("u64", "f64") else 4
rd, wr = g("dram__bytes_read.sum") * 1e9, g("dram__bytes_write.sum") * 1e9
a, l, s = (g("l1tex__data_pipe_lsu_wavefronts_mem_shared_op_" + o + ".sum") for o in ("atom", "ld", "st"))
j = {"source": note, "keys_per_launch": int(n), "dram_bytes_read": rd, "dram_bytes_write": wr,
     "dram_bytes_per_launch": rd + wr, "algorithmic_bytes_per_launch": 2 * K * n, "key_type": kt,
     "smem_wavefronts_per_launch": a + l + s, "smem_wavefronts_per_32_keys": round((a + l + s) / (n / 32), 2),
     "smem_wavefronts_pct_of_peak_sustained_elapsed": g("l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed"),
     "smem_bank_conflicts_per_launch": g("l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum"),
     "gpu_time_ms_cold": g("gpu__time_duration.sum")}
try:  # the whole L1 data pipe (shared + global/local wavefronts), when the summary carries it
    sms = g("device__attribute_multiprocessor_count")
    sh = g("SM_A.TriageCompute.l1tex__data_pipe_lsu_wavefronts_mem_shared.avg") * sms
    lg = g("SM_A.TriageCompute.l1tex__data_pipe_lsu_wavefronts_mem_lgds.avg") * sms
    j["l1_pipe_wavefronts_per_32_keys"] = round((sh + lg) / (n / 32), 2)
    j["l1_pipe_global_wavefronts_per_32_keys"] = round(lg / (n / 32), 2)
    j["l1_pipe_pct_of_peak_sustained_elapsed"] = g("l1tex__data_pipe_lsu_wavefronts.sum.pct_of_peak_sustained_elapsed")
except AttributeError:
    pass
json.dump(j, open(out, "w"), indent=1)
print(out, round(j["dram_bytes_per_launch"] / j["algorithmic_bytes_per_launch"], 4), j["smem_wavefronts_per_32_keys"], j["gpu_time_ms_cold"])
