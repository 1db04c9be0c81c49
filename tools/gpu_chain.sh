set -x
Q="--steps 2000 --warmup 10 --no-cpu-baseline --no-e2e --no-hoisted --no-klss --no-boot --no-apps --no-latency --batch-hrot 0"
for c in 1 8 16 1 8 16 32; do
  timeout 300 python bench.py $Q --chain-steps $c > gpurun_out/chain_$c.json 2>gpurun_out/chain_$c.err
  python -c "import json; d=json.load(open('gpurun_out/chain_$c.json')); print('chain $c', round(d['value'],1), round(d['ms_per_step'],4), d['gpu_launches'])" || tail -3 gpurun_out/chain_$c.err
done
