timeout 900 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-e2e --no-hoisted --batch-hrot 0 > gpurun_out/bench_klss.json 2> gpurun_out/bench_klss.err
tail -3 gpurun_out/bench_klss.err
python -c "
import json; d=json.load(open('gpurun_out/bench_klss.json')); print(round(d['value'],1), json.dumps(d['klss_vs_hybrid_setc'], indent=1))"
