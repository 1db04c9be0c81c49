set -x
timeout 300 python tools/bconv_trace.py 2>&1 | tail -12
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_klss.py tests/test_gpu_extremal.py tests/test_gpu_sharded_native.py -m gpu -q -x 2>&1 | tail -2
Q="--steps 2000 --warmup 10 --no-cpu-baseline --no-e2e --no-hoisted --no-boot --no-apps --no-latency --batch-hrot 0"
for v in 1 2; do
  timeout 300 python bench.py $Q > gpurun_out/bl_$v.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/bl_$v.json')); b=d['breakdown']; print('run $v', round(d['value'],1), round(d['ms_per_step'],4), 'bconv', b['bconv'], 'single', d['single_stream_profiled_ms_per_step'], 'klss48', d['klss_vs_hybrid_setc']['klss_t48_B1'])"
done
