python -m paper_conf_isca_jiaodwfcm0z25_b200.build > /dev/null
timeout 900 python -m pytest tests/test_gpu_boot.py -x -q 2>&1 | tail -5
timeout 900 python bench.py --steps 200 --warmup 5 --no-cpu-baseline --no-e2e --no-hoisted --no-klss --no-apps --batch-hrot 0 > gpurun_out/bench_boot.json 2> gpurun_out/bench_boot.err
tail -5 gpurun_out/bench_boot.err
python -c "
import json; d=json.load(open('gpurun_out/bench_boot.json'))
print('value', d['value'], 'clocks', d['clocks']); print(json.dumps(d['bootstrap']))
"
