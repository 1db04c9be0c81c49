# ncu launch list (durations only) of a single-stream, non-graph bench step
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e --no-hoisted --graph 0 --streams 1 > /dev/null 2>&1
wc -l gpurun_out/launches.csv
