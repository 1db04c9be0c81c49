set -x
timeout 1500 python -m pytest tests -m gpu -q -x 2>&1 | tail -4
for b in 1 8; do timeout 300 python tools/klss_profile.py $b 48; done
Q="--steps 2000 --warmup 10 --no-cpu-baseline --no-e2e --no-hoisted --no-boot --no-apps --no-latency --batch-hrot 0"
timeout 300 python bench.py $Q > gpurun_out/b12.json 2>/dev/null
python -c "import json; d=json.load(open('gpurun_out/b12.json')); print(round(d['value'],1), round(d['ms_per_step'],4)); print(json.dumps(d['klss_vs_hybrid_setc']))"
