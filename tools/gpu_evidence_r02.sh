# Round-2 evidence of the current code: GPU tests, smoke, full bench line, ncu launch list and
# full captures of the top kernels, compute-sanitizer over the tiny tests (incl. KLSS-48 and the
# opt-in fused KeyIP path)
set -x
timeout 1500 python -m pytest tests -m gpu -q 2>&1 | tail -3
timeout 300 python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -2
timeout 1200 python bench.py > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err; tail -3 gpurun_out/bench_full.err
python -c "import json; d=json.load(open('gpurun_out/bench_full.json')); print(d['value'], d['ms_per_step'], d['clocks'])"
NCUARGS="--steps 2 --warmup 1 --no-cpu-baseline --no-e2e --no-hoisted --no-klss --no-boot --no-apps --no-latency --batch-hrot 0 --graph 0 --streams 1"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
    python bench.py $NCUARGS > /dev/null 2>&1
wc -l gpurun_out/launches.csv
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_ntt_col|k_ntt_row|k_bconv_tc|k_keyip|k_hmr_cl|k_tensor|k_automorph" -s 40 -c 12 \
    -o gpurun_out/prof_top python bench.py $NCUARGS > gpurun_out/ncu_top.log 2>&1
tail -2 gpurun_out/ncu_top.log
SEL='tiny and not setb'
for tool in memcheck racecheck synccheck; do
  timeout 1500 /usr/local/cuda/bin/compute-sanitizer --tool $tool --error-exitcode 9 --print-limit 20 \
     python -m pytest tests/test_gpu_parity.py tests/test_gpu_wire.py tests/test_gpu_apps.py tests/test_gpu_klss.py -q -x \
     -k "$SEL or wire or pmult_acc or helr or conv or chunk or hrot_sum or tiny48" > gpurun_out/san_$tool.log 2>&1
  echo "$tool rc=$?"; grep -E "ERROR SUMMARY|passed|failed" gpurun_out/san_$tool.log | tail -3
done
NEO_KIP=1 timeout 1500 /usr/local/cuda/bin/compute-sanitizer --tool memcheck --error-exitcode 9 --print-limit 20 \
   python -m pytest tests/test_gpu_parity.py -q -x -k "tiny and not setb" > gpurun_out/san_kip_memcheck.log 2>&1
echo "kip memcheck rc=$?"; grep -E "ERROR SUMMARY|passed|failed" gpurun_out/san_kip_memcheck.log | tail -3
