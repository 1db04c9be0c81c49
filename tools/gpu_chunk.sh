python -m paper_conf_isca_jiaodwfcm0z25_b200.build > /dev/null
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "chunk or hrot or hmult or keyswitch" 2>&1 | tail -3
for c in 0 16 32 64; do
NEO_BATCH_CHUNK=$c timeout 600 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-e2e --no-hoisted --no-klss --no-boot --no-apps > gpurun_out/chunk.json 2> gpurun_out/chunk.err
python -c "
import json; d=json.load(open('gpurun_out/chunk.json')); b=d['batch_hrot']; print('chunk', $c, 'value', round(d['value'],1), 'B256', round(b['value'],1), [(s['batch_per_gpu'], round(s['value'])) for s in b['sweep']])
"
done
