# Round-2 final evidence: GPU tests, smoke, full bench line, ncu launch list and full captures of
# the top kernels (compute-sanitizer is closed on this pool)
set -x
timeout 1800 python -m pytest tests -m gpu -q 2>&1 | tail -3
timeout 300 python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -2
timeout 1500 python bench.py > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err; tail -3 gpurun_out/bench_full.err
python -c "import json; d=json.load(open('gpurun_out/bench_full.json')); print(d['value'], d['ms_per_step'], d['clocks'])"
NCUARGS="--steps 2 --warmup 1 --no-cpu-baseline --no-e2e --no-hoisted --no-klss --no-boot --no-apps --no-latency --batch-hrot 0 --graph 0 --streams 1"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
    python bench.py $NCUARGS > /dev/null 2>&1
wc -l gpurun_out/launches.csv
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_ntt_col|k_ntt_row|k_bconv_tc|k_keyip|k_hmr_cl|k_tensor|k_automorph" -s 40 -c 12 \
    -o gpurun_out/prof_top python bench.py $NCUARGS > gpurun_out/ncu_top.log 2>&1
tail -2 gpurun_out/ncu_top.log
timeout 600 python tools/klss_profile.py 1 48 > gpurun_out/klss_profile.txt 2>&1; cat gpurun_out/klss_profile.txt | head -40
timeout 300 python tools/step_launches.py > gpurun_out/step_launches.txt 2>&1; tail -30 gpurun_out/step_launches.txt
