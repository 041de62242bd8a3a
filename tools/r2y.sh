timeout 900 python -m pytest tests/test_parity_gpu.py -q -x -k "host" 2>&1 | tail -1
