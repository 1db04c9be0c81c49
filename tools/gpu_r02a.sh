# round-2 check: GPU tests, bench (FP64 default and tensor-core NTT), NTT A/B under ncu
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
timeout 2400 python -m pytest tests -m gpu -q -x 2>&1 | tail -4
timeout 1200 python bench.py > gpurun_out/bench_r02a.json 2> gpurun_out/bench_r02a.err; tail -2 gpurun_out/bench_r02a.err
NEO_NTT=tc timeout 900 python bench.py --steps 500 --no-cpu-baseline --no-e2e --no-hoisted --no-klss --no-boot --no-apps --no-latency --batch-hrot 0 > gpurun_out/bench_r02a_tc.json 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_ntt" -s 12 -c 4 -o gpurun_out/ab_fp64 python tools/ntt_bench.py 108 2 fp64 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_ntt_tc" -s 12 -c 4 -o gpurun_out/ab_tc python tools/ntt_bench.py 108 2 tc > /dev/null 2>&1
ls -la gpurun_out/*.ncu-rep
