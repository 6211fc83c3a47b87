timeout 900 python -m pytest tests -m gpu -q -x --timeout 600 2>&1 | tail -3
python -c "import paper_conf_sigmod_maltenbergeritr22_b200 as m; print(\"rank mode\", m.msort_rank_mode(0))"
for cfg in 0 1 2; do MSORT_OS_CFG=$cfg timeout 300 python tools/time_radix.py 2e9 u32 uniform 3 | cut -c1-330; done
timeout 300 python tools/time_radix.py 2e9 u32 zipf 3 | cut -c1-330
timeout 300 python tools/time_radix.py 1e9 u64 uniform 3 | cut -c1-330
timeout 300 python tools/time_radix.py 2e9 f32 uniform 3 | cut -c1-330
