python -m paper_conf_isca_jiaodwfcm0z25_b200.build > /dev/null
for f in 0 1 0 1; do
timeout 600 python bench.py --steps 1000 --warmup 10 --fused-rescale $f --no-cpu-baseline --no-e2e --no-hoisted --no-klss --no-boot --no-apps --batch-hrot 0 > gpurun_out/fab.json 2> gpurun_out/fab.err
python -c "
import json; d=json.load(open('gpurun_out/fab.json'))
print('fused', $f, 'value', round(d['value'],1), 'ms', round(d['ms_per_step'],4), '1s', round(d['single_stream_profiled_ms_per_step'],4), d['roofline']['kernel'], round(d['roofline']['frac'],3), 'step', round(d['step_roofline']['frac'],3), d['clocks'])
"
done
