python -m paper_conf_isca_jiaodwfcm0z25_b200.build > /dev/null
timeout 600 python -m pytest tests/test_gpu_wire.py -x -q 2>&1 | tail -5
timeout 900 python bench.py --steps 300 --warmup 5 --no-cpu-baseline --no-hoisted --no-klss --no-boot --no-apps --batch-hrot 0 > gpurun_out/bench_e2e.json 2> gpurun_out/bench_e2e.err
tail -5 gpurun_out/bench_e2e.err
python -c "
import json; d=json.load(open('gpurun_out/bench_e2e.json'))
print('value', d['value'], 'clocks', d['clocks']); print(json.dumps(d['e2e'])); print(json.dumps(d['e2e_u64']))
"
