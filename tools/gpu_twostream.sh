# two-stream hoisted rotations / giant-step sums: parity, bootstrap timing A/B
set -x
timeout 1500 python -m pytest tests -m gpu -q -x 2>&1 | tail -3
for v in 1 0 1 0; do
  NEO_TWO_STREAM=$v timeout 300 python tools/boot_full_profile.py 2>&1 | head -4
done
Q="--steps 200 --warmup 5 --no-cpu-baseline --no-e2e --no-klss --no-latency --batch-hrot 0"
for v in 1 0; do
  NEO_TWO_STREAM=$v timeout 600 python bench.py $Q > gpurun_out/ts_$v.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/ts_$v.json')); b=d['bootstrap']; print('two=$v', round(d['value'],1), 'boot', b['ms_per_bootstrap'], b['ms_eager'], 'sparse', b['sparse_8_slots']['ms_per_bootstrap'], 'hoisted', d['hoisted_rotations'], 'apps', {k: v.get('ms_per_iteration', v.get('ms_per_layer', v.get('ms'))) for k, v in d['apps'].items() if isinstance(v, dict)})"
done
