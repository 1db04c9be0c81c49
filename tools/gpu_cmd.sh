timeout 600 python -m pytest tests/test_gpu_ops.py -x -q 2>&1 | tail -3
bash tools/gpu_ab.sh
