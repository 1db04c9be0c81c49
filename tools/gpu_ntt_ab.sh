# first check of the tensor-core NTT: parity of both implementations, NTT micro-benchmark, main parity suite
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 900 python -m pytest tests/test_gpu_ntt_impl.py -x -q 2>&1 | tail -15
timeout 300 python tools/ntt_bench.py 108 50 tc fp64 2>&1 | tail -12
timeout 300 python tools/ntt_bench.py 36 50 tc fp64 2>&1 | tail -12
timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q 2>&1 | tail -5
