timeout 900 python -m pytest tests/test_gpu_fullsize.py -q --timeout 800 -k "268435456" 2>&1 | grep -E "passed|failed|Error|assert" | head
timeout 900 python -m pytest tests/test_gpu_fullsize.py -q --timeout 800 -k "268435456 or 4e9" 2>&1 | grep -E "passed|failed|Error|assert" | head
