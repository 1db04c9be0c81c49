# ncu --set full capture of the ModUp tensor-core BConv (one launch) + source-level stalls
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_bconv_tc_g" -s 4 -c 1 -o gpurun_out/prof_bconv python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e --graph 0 --streams 1 > gpurun_out/ncu_bconv.log 2>&1
tail -3 gpurun_out/ncu_bconv.log
