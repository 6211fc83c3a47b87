#!/bin/bash
# after the count-at-end onesweep default (4-byte keys): GPU suite, bench line, launch list, ncu of the pass
exec > gpurun_out/verify3.log 2>&1
python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')"
timeout 1800 python -m pytest tests -m gpu -q -x --timeout 400 2>&1 | tail -3
timeout 900 python bench.py --steps 10 --warmup 3 --cpu-seconds 10 > gpurun_out/bench_v3.json 2> gpurun_out/bench_v3.err
tail -c 300 gpurun_out/bench_v3.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_v3.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:onesweep -s 6 -c 1 -o gpurun_out/os_v3 python tools/prof_radix.py 4e9 u32 2 > /dev/null 2>&1
timeout 600 python bench.py --key-type f32 --keys 2e9 --steps 5 --warmup 3 --het > gpurun_out/bench_c5_f32_v3.json 2>/dev/null
timeout 600 ncu --set full --clock-control none --import-source on -k regex:onesweep -s 2 -c 1 -o gpurun_out/os_f32_v3 python tools/prof_radix.py 2e9 f32 2 > /dev/null 2>&1
python tools/ncu_summary.py gpurun_out/os_v3.ncu-rep 12 > gpurun_out/os_v3_summary.txt 2>&1
python tools/ncu_summary.py gpurun_out/os_f32_v3.ncu-rep 12 > gpurun_out/os_f32_v3_summary.txt 2>&1
rm -f gpurun_out/*.ncu-rep   # (gpurun brings back at most 64 MiB)
echo done
