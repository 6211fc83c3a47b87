# re-entry check: full GPU suite + smoke + default bench line + launch list
timeout 1500 python -m pytest tests -m gpu -q -x --timeout 400 2>&1 | tail -15 > gpurun_out/pytest_gpu.txt
tail -15 gpurun_out/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()"
timeout 900 python bench.py --steps 5 --warmup 3 --cpu-seconds 10 > gpurun_out/bench_c3.json 2> gpurun_out/bench_c3.err
head -c 800 gpurun_out/bench_c3.json
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c3.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu > /dev/null 2>&1
