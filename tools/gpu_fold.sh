# hmr merge + fold fusion: full GPU suite, KIP parity (opt-in path), bench, launches
set -x
timeout 1500 python -m pytest tests -m gpu -q -x 2>&1 | tail -5
NEO_KIP=1 timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_ops.py -m gpu -q -x 2>&1 | tail -3
Q="--steps 2000 --warmup 10 --no-cpu-baseline --no-e2e --no-hoisted --no-klss --no-boot --no-apps --no-latency --batch-hrot 0"
for v in 1 2; do
  timeout 300 python bench.py $Q > gpurun_out/fold_$v.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/fold_$v.json')); print('run $v', round(d['value'],1), round(d['ms_per_step'],4))"
done
timeout 300 python tools/step_launches.py > gpurun_out/step_launches.txt 2>&1; cat gpurun_out/step_launches.txt
