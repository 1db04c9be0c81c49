# KeyIP key loads as evict-first (ld.global.cs) A/B: swap the library between runs
set -x
Q="--steps 2000 --warmup 10 --no-cpu-baseline --no-e2e --no-hoisted --no-boot --no-apps --no-latency --batch-hrot 256"
for v in cs base cs base; do
  cp ab/libneo_$v.so paper_conf_isca_jiaodwfcm0z25_b200/libneo.so
  timeout 300 python bench.py $Q > gpurun_out/kc_$v.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/kc_$v.json')); b=d['breakdown']; print('$v', round(d['value'],1), round(d['ms_per_step'],4), 'ntt', b['ntt']['ms_per_step'], 'keyip', b['keyip']['ms_per_step'], 'B256', round(d['batch_hrot']['value']), 'klss48', d['klss_vs_hybrid_setc']['klss_t48_B1']['ms_per_call'])"
done
