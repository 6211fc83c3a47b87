"""Condense a tools/gpu_abn.sh log: build, key type, distribution, mean pass ms, histogram ms, sort ms."""
import json, sys
for line in open(sys.argv[1]):
    nm, _, js = line.partition(" ")
    try:
        d = json.loads(js)
        print(nm, d["kt"], d["dist"], round(d["pass_ms"], 3), round(d["hist_ms"], 3), round(d["sort_ms"], 2))
    except Exception:
        print(line.rstrip()[:200])
