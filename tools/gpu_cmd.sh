NEO_NTT_TWF=1 timeout 600 python -m pytest tests/test_gpu_parity.py -x -q 2>&1 | tail -1
for T in 0 1 0 1; do
NEO_NTT_TWF=$T timeout 300 python tools/ntt_bench.py 108 50
NEO_NTT_TWF=$T timeout 600 python bench.py --steps 200 --warmup 5 --no-cpu-baseline --no-e2e --no-hoisted --batch-hrot 0 --no-klss > gpurun_out/bb.json 2>/dev/null
python -c "
import json; d=json.load(open('gpurun_out/bb.json'))
print('twf $T', round(d['value'],1), 'KS/s ms/step', round(d['ms_per_step'],4), '1s', round(d['single_stream_profiled_ms_per_step'],4), 'col', d['breakdown']['ntt_col']['ms_per_step'])"
done
for C in 2 1 0; do
NEO_NTT_CFG=$C timeout 600 python bench.py --steps 200 --warmup 5 --no-cpu-baseline --no-e2e --no-hoisted --batch-hrot 0 --no-klss > gpurun_out/bb.json 2>/dev/null
python -c "
import json; d=json.load(open('gpurun_out/bb.json'))
print('cfg $C', round(d['value'],1), 'KS/s ms/step', round(d['ms_per_step'],4), '1s', round(d['single_stream_profiled_ms_per_step'],4))"
done
