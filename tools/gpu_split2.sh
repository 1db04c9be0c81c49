set -x
Q="--steps 20 --warmup 3 --no-cpu-baseline --no-e2e --no-hoisted --no-klss --no-boot --no-apps --no-latency --batch-hrot 256"
for v in 0 216 432 0 864; do
  NEO_NTT_SPLIT=$v timeout 300 python bench.py $Q > gpurun_out/spb_$v.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/spb_$v.json')); b=d['batch_hrot']; print('split $v', round(b['value'],1), [(x['batch_per_gpu'], round(x['value'])) for x in b['sweep']])"
done
NEO_NTT_SPLIT=216 timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -k "chunk or batch" 2>&1 | tail -2
