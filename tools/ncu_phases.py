"""Split an ncu SASS source page into BAR.SYNC-delimited phases and sum warp
stall samples per phase (with the top stall reasons); run here, no GPU.
usage: ncu_phases.py report.ncu-rep [kernel-substring]"""
import csv, io, subprocess, sys
rep = sys.argv[1]
cmd = ['ncu', '-i', rep, '--page', 'source', '--csv', '--print-source', 'sass']
if len(sys.argv) > 2:
    cmd += ['--kernel-name', 'regex:' + sys.argv[2]]
rows = list(csv.reader(io.StringIO(subprocess.run(cmd, capture_output=True, text=True).stdout)))
k = next(i for i, r in enumerate(rows) if r and r[0] == 'Address')
h = rows[k]
data = [r for r in rows[k + 1:] if len(r) == len(h)]
i_all = h.index('Warp Stall Sampling (All Samples)')
reasons = [j for j, c in enumerate(h) if c.startswith('stall_') or c.startswith('smsp__pcsamp_warps_issue_stalled')]
tot = sum(int(r[i_all] or 0) for r in data)
phases, cur, first = [], [], None
for r in data:
    cur.append(r)
    if 'BAR.SYNC' in r[1] or 'BAR.RED' in r[1] or 'EXIT' in r[1]:
        phases.append(cur); cur = []
if cur: phases.append(cur)
for n, ph in enumerate(phases):
    s = sum(int(r[i_all] or 0) for r in ph)
    if s * 100 < tot: continue
    rs = {}
    for r in ph:
        for j in reasons:
            try: rs[h[j]] = rs.get(h[j], 0) + int(float(r[j] or 0))
            except ValueError: pass
    top = sorted(rs.items(), key=lambda x: -x[1])[:4]
    print(f"phase {n:2d} [{ph[0][0][-5:]}..{ph[-1][0][-5:]}] {len(ph):4d} instr  {s*100/tot:5.1f}%  " +
          " ".join(f"{a.replace('smsp__pcsamp_warps_issue_stalled_','')}={b*100/tot:.1f}" for a, b in top))
    for r in sorted(ph, key=lambda r: -int(r[i_all] or 0))[:3]:
        print(f"        {int(r[i_all] or 0)*100/tot:5.1f}% {r[0][-5:]} {r[1].strip()[:80]}")
