# fused ModUp row pass + KeyIP, one launch per digit round: parity, A/B
set -x
NEO_KIP=1 timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_ops.py tests/test_gpu_extremal.py tests/test_gpu_boot.py -m gpu -q -x -k "not set_b" 2>&1 | tail -3
Q="--steps 2000 --warmup 10 --no-cpu-baseline --no-e2e --no-hoisted --no-klss --no-boot --no-apps --no-latency --batch-hrot 0"
for v in 1 0 1 0; do
  NEO_KIP=$v timeout 300 python bench.py $Q > gpurun_out/kip2_$v.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/kip2_$v.json')); b=d['breakdown']; print('NEO_KIP=$v', round(d['value'],1), round(d['ms_per_step'],4), 'single', d['single_stream_profiled_ms_per_step'], 'keyip', b['keyip']['ms_per_step'], 'ntt', b['ntt']['ms_per_step'])"
done
NEO_KIP=1 timeout 300 python tools/step_launches.py > gpurun_out/step_launches_kip.txt 2>&1; cat gpurun_out/step_launches_kip.txt
