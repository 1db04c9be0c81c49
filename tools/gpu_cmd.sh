timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_ops.py tests/test_gpu_sharded.py -x -q 2>&1 | tail -3
bash tools/gpu_ab.sh
