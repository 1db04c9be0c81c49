set -x
timeout 1800 python -m pytest tests/test_gpu_parity.py tests/test_gpu_extremal.py tests/test_gpu_ops.py -m gpu -q -x 2>&1 | tail -2
Q="--steps 2000 --warmup 10 --no-cpu-baseline --no-e2e --no-hoisted --no-boot --no-apps --no-latency --batch-hrot 256"
for v in 1 0 1 0; do
  NEO_TENSOR2=$v timeout 300 python bench.py $Q > gpurun_out/t2_$v.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/t2_$v.json')); b=d['breakdown']; print('tensor2=$v', round(d['value'],1), round(d['ms_per_step'],4), 'ntt', b['ntt']['ms_per_step'], 'tensor', b['tensor']['ms_per_step'], 'keyip', b['keyip']['ms_per_step'], 'single', d['single_stream_profiled_ms_per_step'], 'B256', round(d['batch_hrot']['value']), 'klss48', d['klss_vs_hybrid_setc']['klss_t48_B1']['ms_per_call'])"
done
