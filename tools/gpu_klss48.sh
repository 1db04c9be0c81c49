# KLSS at WordSize_T = 48: parity, then the Set-C KLSS vs Hybrid timing block
set -x
timeout 1200 python -m pytest tests/test_gpu_klss.py -q -x 2>&1 | tail -15
timeout 600 python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-e2e --no-hoisted --no-boot --no-apps --no-latency --batch-hrot 0 > gpurun_out/klss48.json 2> gpurun_out/klss48.err
tail -3 gpurun_out/klss48.err
python -c "
import json; d=json.load(open('gpurun_out/klss48.json')); print(json.dumps(d['klss_vs_hybrid_setc'], indent=1))"
