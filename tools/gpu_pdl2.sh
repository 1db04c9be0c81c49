set -x
NEO_PDL=2 timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x 2>&1 | tail -2
Q="--steps 2000 --warmup 10 --no-cpu-baseline --no-e2e --no-hoisted --no-klss --no-boot --no-apps --no-latency --batch-hrot 0"
for v in 0 2 0 2 1; do
  NEO_PDL=$v timeout 300 python bench.py $Q > gpurun_out/pdl_$v.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/pdl_$v.json')); print('pdl $v', round(d['value'],1), round(d['ms_per_step'],4), d['breakdown']['bconv'])"
done
