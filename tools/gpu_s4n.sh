timeout 900 python -m pytest tests/test_gpu_gauss.py -x -q 2>&1 | tail -5
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
