set -x
Q="--steps 2000 --warmup 10 --no-cpu-baseline --no-e2e --no-hoisted --no-klss --no-boot --no-apps --no-latency --batch-hrot 0"
for v in 0 56 40 0 56 28; do
  NEO_NTT_SPLIT=$v timeout 300 python bench.py $Q > gpurun_out/sp_$v.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/sp_$v.json')); b=d['breakdown']; print('split $v', round(d['value'],1), round(d['ms_per_step'],4), 'ntt', b['ntt']['ms_per_step'], 'single', d['single_stream_profiled_ms_per_step'])"
done
NEO_NTT_SPLIT=56 timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -k "setb" 2>&1 | tail -2
