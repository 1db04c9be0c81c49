# A/B of builds of libneo.so (ab/<name>.so for each name in $AB, default "base new"): NTT
# micro-benchmark + short bench each, then the parity suite on ab/new.so (or the last variant)
L=paper_conf_isca_jiaodwfcm0z25_b200/libneo.so
AB=${AB:-"base new"}
for v in $AB; do
  cp ab/$v.so $L
  echo "== $v"
  [ -z "$NO_NTT" ] && timeout 300 python tools/ntt_bench.py 108 50
  timeout 600 python bench.py --steps 200 --warmup 10 --no-cpu-baseline --no-e2e --no-hoisted --batch-hrot 0 --no-klss > gpurun_out/ab_$v.json 2>/dev/null
  python -c "
import json; d=json.load(open('gpurun_out/ab_$v.json')); b=d['breakdown']
print('bench', round(d['value'],1), 'KS/s ms', round(d['ms_per_step'],4), '1-stream', round(d['single_stream_profiled_ms_per_step'],4))
print(' '.join(f'{k}={v[\"ms_per_step\"]:.4f}' for k,v in b.items() if v['ms_per_step']))"
done
cp ab/${AB##* }.so $L
[ -z "$NO_TEST" ] && timeout 600 python -m pytest tests/test_gpu_parity.py -x -q 2>&1 | tail -2
