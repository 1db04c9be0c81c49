# fused ModUp row pass + KeyIP: parity, then A/B against the separate KeyIP launch
set -x
timeout 1500 python -m pytest tests -m gpu -q -x 2>&1 | tail -5
Q="--steps 2000 --warmup 10 --no-cpu-baseline --no-e2e --no-hoisted --no-klss --no-boot --no-apps --no-latency --batch-hrot 0"
for v in 1 0 1 0; do
  NEO_KIP=$v timeout 300 python bench.py $Q > gpurun_out/kip_$v.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/kip_$v.json')); print('NEO_KIP=$v', round(d['value'],1), round(d['ms_per_step'],4))"
done
for cfg in 1 2; do
  NEO_KIP_CFG=$cfg timeout 300 python bench.py $Q > gpurun_out/kipcfg_$cfg.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/kipcfg_$cfg.json')); print('NEO_KIP_CFG=$cfg', round(d['value'],1), round(d['ms_per_step'],4))"
done
timeout 300 python tools/step_launches.py > gpurun_out/step_launches.txt 2>&1; cat gpurun_out/step_launches.txt
