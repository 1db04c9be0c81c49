python -m paper_conf_isca_jiaodwfcm0z25_b200.build > /dev/null
timeout 900 python -m pytest tests/test_gpu_boot.py tests/test_gpu_apps.py -x -q 2>&1 | tail -5
timeout 900 python bench.py --steps 200 --warmup 5 --no-cpu-baseline --no-e2e --no-hoisted --no-klss --batch-hrot 0 > gpurun_out/bench_ba.json 2> gpurun_out/bench_ba.err
tail -5 gpurun_out/bench_ba.err
python -c "
import json; d=json.load(open('gpurun_out/bench_ba.json'))
print('value', d['value'], 'clocks', d['clocks']); print(json.dumps(d['bootstrap'])); a=d['apps']; print(a['helr_iteration']['ms_per_iteration'], a['resnet20_conv_layer']['ms_per_layer'])
"
