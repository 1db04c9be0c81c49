# bench variants: graph on/off, streams 1/2
for cfg in "--graph 1 --streams 2" "--graph 0 --streams 2" "--graph 1 --streams 1"; do
  timeout 300 python bench.py --steps 200 --warmup 10 --no-cpu-baseline --no-e2e $cfg > gpurun_out/bv.json 2> gpurun_out/bv.err || tail -20 gpurun_out/bv.err
  python -c "
import json; d=json.load(open('gpurun_out/bv.json'))
print('$cfg', round(d['value'],1), 'ms/step', round(d['ms_per_step'],4), '1-stream profiled', round(d['single_stream_profiled_ms_per_step'],4), 'launches', d['gpu_launches'])"
done
