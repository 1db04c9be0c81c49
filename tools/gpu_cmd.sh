timeout 1200 python -m pytest tests/test_gpu_klss.py -x -q 2>&1 | tail -25
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_ops.py -x -q 2>&1 | tail -3
