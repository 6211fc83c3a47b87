# full GPU suite + smoke + default bench line (after kernel changes)
timeout 1500 python -m pytest tests -m gpu -q -x --timeout 400 2>&1 | tail -15 > gpurun_out/pytest_gpu.txt
tail -15 gpurun_out/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()"
timeout 900 python bench.py --steps 5 --warmup 3 --cpu-seconds 5 > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err
cat gpurun_out/bench_c2.json | head -c 600
