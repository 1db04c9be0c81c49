timeout 600 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
for p in 1 0; do
 for g in 1 0; do
  NEO_PDL=$p timeout 300 python bench.py --steps 200 --warmup 10 --no-cpu-baseline --no-e2e --graph $g > gpurun_out/bp.json 2>/dev/null
  python -c "
import json; d=json.load(open('gpurun_out/bp.json'))
print('pdl $p graph $g', round(d['value'],1), 'ms/step', round(d['ms_per_step'],4))"
 done
done
NEO_PDL=1 timeout 300 python bench.py --steps 200 --warmup 10 --no-cpu-baseline --no-e2e --streams 1 > gpurun_out/bp.json 2>/dev/null
python -c "
import json; d=json.load(open('gpurun_out/bp.json'))
print('pdl 1 graph 1 streams 1', round(d['value'],1), 'ms/step', round(d['ms_per_step'],4))"
NEO_PDL=0 timeout 300 python bench.py --steps 200 --warmup 10 --no-cpu-baseline --no-e2e --streams 1 > gpurun_out/bp.json 2>/dev/null
python -c "
import json; d=json.load(open('gpurun_out/bp.json'))
print('pdl 0 graph 1 streams 1', round(d['value'],1), 'ms/step', round(d['ms_per_step'],4))"
