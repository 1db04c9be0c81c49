set -x
nvidia-smi --query-gpu=clocks.sm,clocks.max.sm --format=csv
timeout 600 python bench.py --steps 200 --warmup 10 > gpurun_out/bench1.json 2> gpurun_out/bench1.err
tail -c 3000 gpurun_out/bench1.err
cat gpurun_out/bench1.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches1.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > /dev/null 2>&1
wc -l gpurun_out/launches1.csv
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_ntt_col -s 20 -c 2 -o gpurun_out/prof_ntt_col python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/ncu_full1.log 2>&1
tail -5 gpurun_out/ncu_full1.log
