# functional check of the N > 1 bench paths: 2 ranks on one GPU over gloo (not a measurement)
set -x
NEO_BENCH_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 \
   bench.py --gpus 2 --steps 20 --warmup 3 --no-cpu-baseline --batch-hrot 16 > gpurun_out/dist2.json 2> gpurun_out/dist2.err
echo rc=$?
tail -20 gpurun_out/dist2.err
python -c "import json; d=json.load(open('gpurun_out/dist2.json')); print(d['value'], d['n_gpus'], d.get('limb_sharded_keyswitch_native'), d.get('limb_sharded_keyswitch'), d['bootstrap'].get('limb_sharded') if d.get('bootstrap') else None, d['e2e'] and d['e2e']['value'])"
