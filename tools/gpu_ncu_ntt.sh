# ncu --set full captures of the NTT passes (first 4 launches after skipping 12) + source-level stalls
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_ntt" -s 12 -c 4 -o gpurun_out/prof_ntt python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e --graph 0 --streams 1 --no-hoisted --batch-hrot 0 --no-klss > gpurun_out/ncu_ntt.log 2>&1
tail -2 gpurun_out/ncu_ntt.log
