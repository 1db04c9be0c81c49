set -x
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_extremal.py tests/test_gpu_ops.py -m gpu -q -x 2>&1 | tail -3
Q="--steps 2000 --warmup 10 --no-cpu-baseline --no-e2e --no-hoisted --no-klss --no-boot --no-apps --no-latency --batch-hrot 0"
for v in 0 1 0 1; do
  NEO_KEYIP_CFG=$v timeout 300 python bench.py $Q > gpurun_out/kcfg_$v.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/kcfg_$v.json')); print('cfg $v', round(d['value'],1), round(d['ms_per_step'],4), d['breakdown']['keyip'])"
done
