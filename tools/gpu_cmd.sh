timeout 900 python -m pytest tests/test_gpu_boot.py -x -q 2>&1 | tail -15
