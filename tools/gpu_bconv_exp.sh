for e in 63 256 511; do
  NEO_BCONV_EXP=$e timeout 300 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-e2e > gpurun_out/bx.json 2>/dev/null
  python -c "
import json; d=json.load(open('gpurun_out/bx.json')); b=d['breakdown']
print('exp $e', 'bconv', b['bconv']['ms_per_step'])"
done
