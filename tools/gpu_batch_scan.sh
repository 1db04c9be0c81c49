for B in 1 2 4 8; do
  timeout 600 python bench.py --steps 40 --warmup 3 --batch $B --no-cpu-baseline --no-e2e > gpurun_out/bb.json 2>/dev/null
  python -c "
import json; d=json.load(open('gpurun_out/bb.json')); b=d['breakdown']
print('B=$B', 'KS/s', round(d['value'],1), 'ms/step', round(d['ms_per_step'],3), ' '.join(f'{k}={v[\"ms_per_step\"]/$B:.4f}' for k,v in b.items()))"
done
