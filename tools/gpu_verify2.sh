#!/bin/bash
# re-entry check: restored tree, full GPU suite + bench line
exec > gpurun_out/verify2.log 2>&1
python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')"
timeout 1800 python -m pytest tests -m gpu -q -x --timeout 400 2>&1 | tail -4
timeout 900 python bench.py --steps 10 --warmup 3 --cpu-seconds 10 > gpurun_out/bench_v2.json 2> gpurun_out/bench_v2.err
tail -c 300 gpurun_out/bench_v2.err
cat gpurun_out/bench_v2.json
