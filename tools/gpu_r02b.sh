# r02 session 2: baseline of the restored code: GPU tests, bench, per-launch step breakdown
set -x
timeout 1500 python -m pytest tests -m gpu -q -x 2>&1 | tail -5
timeout 600 python bench.py --steps 1000 --warmup 10 --no-cpu-baseline --no-boot --no-apps > gpurun_out/bench.json 2> gpurun_out/bench.err
tail -c 1500 gpurun_out/bench.err
python -c "
import json; d=json.load(open('gpurun_out/bench.json'))
print('value', round(d['value'],1), d['unit'], 'ms/step', round(d['ms_per_step'],4))
print('roofline', d['roofline'])
for k,v in d['breakdown'].items(): print(' ', k.ljust(18), v)
"
timeout 300 python tools/step_launches.py > gpurun_out/step_launches.txt 2>&1; cat gpurun_out/step_launches.txt
