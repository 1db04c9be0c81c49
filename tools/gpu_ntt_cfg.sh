# compare NTT pipeline/occupancy variants (NEO_NTT_CFG) on the bench step
timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -k "ntt or keyswitch_setb" 2>&1 | tail -2
for c in 0 1 2; do
  NEO_NTT_CFG=$c timeout 300 python bench.py --steps 200 --warmup 10 --no-cpu-baseline --no-e2e > gpurun_out/bench_cfg$c.json 2>/dev/null
  python -c "
import json; d=json.load(open('gpurun_out/bench_cfg$c.json')); b=d['breakdown']
print('cfg $c', round(d['value'],1), 'ntt_col', b['ntt_col']['ms_per_step'], 'ntt_row', b['ntt_row']['ms_per_step'])"
done
