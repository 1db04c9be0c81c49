# NTT iteration loop: parity of the NTT + key-switch paths, NTT micro-benchmark, short bench
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q 2>&1 | tail -2
timeout 300 python tools/ntt_bench.py 108 50
timeout 300 python tools/ntt_bench.py 36 50
timeout 600 python bench.py --steps 200 --warmup 10 --no-cpu-baseline --no-e2e --no-hoisted > gpurun_out/bi.json 2>/dev/null
python -c "
import json; d=json.load(open('gpurun_out/bi.json')); b=d['breakdown']
print('bench', round(d['value'],1), 'KS/s ms', round(d['ms_per_step'],4), '1-stream', round(d['single_stream_profiled_ms_per_step'],4))
print(' '.join(f'{k}={v[\"ms_per_step\"]:.4f}' for k,v in b.items() if v['ms_per_step']))"
