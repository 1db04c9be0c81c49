# quick loop: GPU parity tests then a short bench
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -15
timeout 600 python bench.py --steps 200 --warmup 10 --no-cpu-baseline > gpurun_out/bench.json 2> gpurun_out/bench.err
tail -c 2000 gpurun_out/bench.err
python -c "
import json; d=json.load(open('gpurun_out/bench.json'))
print('value', round(d['value'],1), d['unit'], 'ms/step', round(d['ms_per_step'],4), 'e2e', d['e2e'] and round(d['e2e']['value'],1))
print('roofline', d['roofline']['kernel'], round(d['roofline']['achieved'],1), round(d['roofline']['frac'],3), 'clocks', d['clocks'])
for k,v in d['breakdown'].items(): print(' ', k.ljust(18), v)
"
