timeout 900 python -m pytest tests/test_gpu_boot.py -x -q 2>&1 | tail -3
timeout 900 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-e2e --no-hoisted --batch-hrot 0 --no-klss > gpurun_out/bench_boot.json 2> gpurun_out/bench_boot.err
tail -3 gpurun_out/bench_boot.err
python -c "
import json; d=json.load(open('gpurun_out/bench_boot.json')); print(round(d['value'],1), json.dumps(d['bootstrap']))"
