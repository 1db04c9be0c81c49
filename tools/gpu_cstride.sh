# compile-time NTT strides: parity + A/B numbers (baseline of the previous build: 4224 KS/s, NTT 0.419 ms single-stream)
set -x
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_ntt_impl.py tests/test_gpu_extremal.py -m gpu -q -x 2>&1 | tail -2
timeout 300 python tools/ntt_bench.py 2>&1 | tail -4
Q="--steps 2000 --warmup 10 --no-cpu-baseline --no-e2e --no-hoisted --no-klss --no-boot --no-apps --no-latency --batch-hrot 256"
for v in 1 2; do
  timeout 300 python bench.py $Q > gpurun_out/cs_$v.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/cs_$v.json')); b=d['breakdown']; print('run $v', round(d['value'],1), round(d['ms_per_step'],4), 'ntt', b['ntt']['ms_per_step'], 'single', d['single_stream_profiled_ms_per_step'], 'B256', round(d['batch_hrot']['value']))"
done
