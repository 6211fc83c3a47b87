exec > gpurun_out/final2.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q -x --timeout 900 2>&1 | tail -3
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')"
