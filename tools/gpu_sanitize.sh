# compute-sanitizer over the N = 2^12 GPU tests: parity, element-wise / wire / apps
SEL='tiny and not setb'
for tool in memcheck racecheck synccheck; do
  timeout 1500 /usr/local/cuda/bin/compute-sanitizer --tool $tool --error-exitcode 9 --print-limit 20 \
     python -m pytest tests/test_gpu_parity.py tests/test_gpu_wire.py tests/test_gpu_apps.py -q -x \
     -k "$SEL or wire or pmult_acc or helr or conv or chunk or hrot_sum" > gpurun_out/san_$tool.log 2>&1
  echo "$tool rc=$?"; grep -E "ERROR SUMMARY|passed|failed" gpurun_out/san_$tool.log | tail -3
done
