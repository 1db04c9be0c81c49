bash tools/gpu_ab.sh 2>&1 | grep -E "==|bench"
bash tools/gpu_ab.sh 2>&1 | grep -E "==|bench"
timeout 900 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-e2e --no-hoisted > gpurun_out/bench_batch.json 2> gpurun_out/bench_batch.err
tail -3 gpurun_out/bench_batch.err
python -c "
import json; d=json.load(open('gpurun_out/bench_batch.json')); print(round(d['value'],1), json.dumps(d['batch_hrot']))"
