for c in 2 3 0 1; do
  NEO_NTT_CFG=$c timeout 300 python bench.py --steps 200 --warmup 10 --no-cpu-baseline --no-e2e --no-hoisted > gpurun_out/bc.json 2>/dev/null
  python -c "
import json; d=json.load(open('gpurun_out/bc.json')); b=d['breakdown']
print('cfg $c', round(d['value'],1), 'ms', round(d['ms_per_step'],4), 'col', b['ntt_col']['ms_per_step'], 'row', b['ntt_row']['ms_per_step'])"
done
