# 8-column column-pass tiles for launches of under two waves: parity and A/B
set -x
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_extremal.py tests/test_gpu_ops.py tests/test_gpu_klss.py tests/test_gpu_ntt_impl.py -m gpu -q -x 2>&1 | tail -2
Q="--steps 2000 --warmup 10 --no-cpu-baseline --no-e2e --no-hoisted --no-klss --no-boot --no-apps --no-latency --batch-hrot 0"
for v in 1 0 1 0; do
  NEO_NTT_C8=$v timeout 300 python bench.py $Q > gpurun_out/c8_$v.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/c8_$v.json')); b=d['breakdown']; print('c8=$v', round(d['value'],1), round(d['ms_per_step'],4), 'ntt', b['ntt']['ms_per_step'], 'single', d['single_stream_profiled_ms_per_step'])"
done
NEO_NTT_C8=1 timeout 300 python tools/step_launches.py 2>&1 | tail -30
