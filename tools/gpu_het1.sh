timeout 600 python -m pytest tests/test_gpu_het.py tests/test_gpu_parity.py -q -x --timeout 300 2>&1 | tail -3
timeout 900 python bench.py --steps 3 --warmup 3 --keys 1e9 --no-cpu --e2e-steps 1 --het 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d[\"value\"], d[\"e2e\"][\"value\"], d[\"het_baseline\"])"
