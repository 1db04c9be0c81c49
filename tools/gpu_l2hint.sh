# NTT intermediate kept in L2 (evict_last stores) and discarded once read: parity, A/B, in-sequence traffic
set -x
timeout 1800 python -m pytest tests -m gpu -q -x 2>&1 | tail -2
Q="--steps 2000 --warmup 10 --no-cpu-baseline --no-e2e --no-hoisted --no-boot --no-apps --no-latency --batch-hrot 256"
for v in 1 0 1 0; do
  NEO_L2HINT=$v timeout 300 python bench.py $Q > gpurun_out/l2_$v.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/l2_$v.json')); b=d['breakdown']; print('l2hint=$v', round(d['value'],1), round(d['ms_per_step'],4), 'ntt', b['ntt']['ms_per_step'], 'keyip', b['keyip']['ms_per_step'], 'single', d['single_stream_profiled_ms_per_step'], 'B256', round(d['batch_hrot']['value']), 'klss48', d['klss_vs_hybrid_setc']['klss_t48_B1']['ms_per_call'])"
done
NCUARGS="--steps 2 --warmup 1 --no-cpu-baseline --no-e2e --no-hoisted --no-klss --no-boot --no-apps --no-latency --batch-hrot 0 --graph 0 --streams 1"
timeout 900 ncu --cache-control none --clock-control none --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum \
   -k regex:"k_ntt_col|k_ntt_row|k_keyip|k_bconv_tc" -s 60 -c 40 --csv --log-file gpurun_out/ncu_warm_l2.csv python bench.py $NCUARGS > /dev/null 2>&1
wc -l gpurun_out/ncu_warm_l2.csv
