timeout 900 python -m pytest tests/test_parity_gpu.py -q -x -k "C3 or part or fanout or C5" 2>&1 | tail -1
