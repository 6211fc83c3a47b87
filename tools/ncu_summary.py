"""Summarise an ncu report: key metrics + top stall lines (run here, no GPU)."""
import csv, io, subprocess, sys
rep = sys.argv[1]
KEYS = ['gpu__time_duration.sum', 'dram__bytes_read.sum', 'dram__bytes_write.sum', 'dram__throughput.avg.pct_of_peak_sustained_elapsed',
        'sm__inst_executed_pipe_adu.avg.pct_of_peak_sustained_active', 'sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active',
        'sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active', 'sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active',
        'smsp__issue_active.avg.pct_of_peak_sustained_active', 'l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed',
        'l1tex__data_pipe_lsu_wavefronts_mem_shared_op_atom.sum', 'l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum',
        'l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum', 'l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum',
        'sm__warps_active.avg.pct_of_peak_sustained_active', 'smsp__inst_executed.sum', 'launch__registers_per_thread',
        'launch__occupancy_limit_registers', 'launch__occupancy_limit_shared_mem', 'sm__throughput.avg.pct_of_peak_sustained_elapsed',
        'lts__t_bytes.sum', 'l1tex__data_pipe_lsu_wavefronts_mem_shared_op_atom.sum.pct_of_peak_sustained_elapsed',
        'l1tex__data_pipe_lsu_wavefronts.sum.pct_of_peak_sustained_elapsed',
        'SM_A.TriageCompute.l1tex__data_pipe_lsu_wavefronts_mem_shared.avg',
        'SM_A.TriageCompute.l1tex__data_pipe_lsu_wavefronts_mem_lgds.avg', 'device__attribute_multiprocessor_count']
raw = subprocess.run(['ncu', '-i', rep, '--page', 'raw', '--csv'], capture_output=True, text=True).stdout
r = list(csv.reader(io.StringIO(raw)))
hdr, units, vals = r[0], r[1], r[2]
for k in KEYS:
    if k in hdr:
        i = hdr.index(k)
        print(f"{k:90s} {vals[i]:>16s} {units[i]}")
src = subprocess.run(['ncu', '-i', rep, '--page', 'source', '--csv', '--print-source', 'sass'], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(src)))
h = rows[1]; data = rows[2:]
i_s = h.index("Warp Stall Sampling (All Samples)")
tot = sum(int(x[i_s]) for x in data if x[i_s].isdigit())
print("stall samples", tot)
n = int(sys.argv[2]) if len(sys.argv) > 2 else 25
for x in sorted(data, key=lambda x: -int(x[i_s]) if x[i_s].isdigit() else 0)[:n]:
    print(f"{int(x[i_s]):7d} {x[0][-5:]} {x[1][:100]}")
# warp-state breakdown (cycles per issued instruction by stall reason)
st = [(hdr[i], vals[i]) for i in range(len(hdr)) if hdr[i].startswith('smsp__average_warps_issue_stalled_')
      and hdr[i].endswith('_per_issue_active.ratio')]
st = sorted(((float(v.replace(',', '')) if v.replace(',', '').replace('.', '').isdigit() else 0.0, k) for k, v in st), reverse=True)
print("warp stalls (per issue):", ", ".join(f"{k[len('smsp__average_warps_issue_stalled_'):-len('_per_issue_active.ratio')]}={v:.2f}" for v, k in st[:8]))
