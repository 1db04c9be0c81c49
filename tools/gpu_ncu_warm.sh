# DRAM traffic of the NTT passes inside the real step sequence (ncu --cache-control none: the
# caches are not flushed between kernels, so the column pass's intermediate can stay in L2)
set -x
NCUARGS="--steps 2 --warmup 1 --no-cpu-baseline --no-e2e --no-hoisted --no-klss --no-boot --no-apps --no-latency --batch-hrot 0 --graph 0 --streams 1"
timeout 900 ncu --cache-control none --clock-control none --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum \
   -k regex:"k_ntt_col|k_ntt_row|k_keyip|k_bconv_tc" -s 60 -c 40 --csv --log-file gpurun_out/ncu_warm.csv python bench.py $NCUARGS > /dev/null 2>&1
wc -l gpurun_out/ncu_warm.csv
