# EvalMod with batched powers / Taylor terms: bootstrap parity and timing
set -x
timeout 1500 python -m pytest tests/test_gpu_boot.py tests/test_gpu_sharded_boot.py -m gpu -q -x 2>&1 | tail -3
timeout 300 python tools/boot_full_profile.py 2>&1 | head -4
Q="--steps 200 --warmup 5 --no-cpu-baseline --no-e2e --no-klss --no-latency --batch-hrot 0 --no-apps --no-hoisted"
timeout 600 python bench.py $Q > gpurun_out/em.json 2>/dev/null
python -c "import json; d=json.load(open('gpurun_out/em.json')); b=d['bootstrap']; print(round(d['value'],1), 'boot', b['ms_per_bootstrap'], b['ms_eager'], 'sparse', b['sparse_8_slots']['ms_per_bootstrap'], 'sharded', b['limb_sharded']['ms_per_bootstrap'])"
