"""Time one limb-sharded key-switch (1 rank, Set-B l=35) against neo_keyswitch, and the host
time of its orchestration (CPU wall between launches)."""
import os
import sys
import time

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_isca_jiaodwfcm0z25_b200 import neo  # noqa: E402
from paper_conf_isca_jiaodwfcm0z25_b200.sharded import NeoOps, ShardPlan, limb_sharded_keyswitch  # noqa: E402

N, NQ, NP, DNUM, L = 1 << 16, 36, 12, 3, 35
ctx = neo.Context(16, NQ, NP, DNUM)
rnd = lambda *s: torch.randint(0, 1 << 35, s, dtype=torch.int64, device="cuda").view(torch.uint64)
key = neo.EvalKey(ctx, rnd(DNUM, 2, NQ + NP, N))
d = rnd(1, L + 1, N)
ops = NeoOps(ctx)
plan = ShardPlan(L, NQ, NP, ctx.alpha, 1, 0, strided=True)
for _ in range(3):
    limb_sharded_keyswitch(ops, plan, d, key)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
t0 = time.perf_counter()
e0.record()
for _ in range(10):
    limb_sharded_keyswitch(ops, plan, d, key)
e1.record()
t1 = time.perf_counter()
torch.cuda.synchronize()
print(f"sharded KS (1 rank): {e0.elapsed_time(e1) / 10:.3f} ms/KS device, host issue {1e3 * (t1 - t0) / 10:.3f} ms/KS")
ws = ctx.workspace(neo.NEO_OP_KEYSWITCH, L, 1)
o0, o1 = rnd(1, L + 1, N), rnd(1, L + 1, N)
for _ in range(3):
    neo.neo_keyswitch(ctx, key, d, L, o0, o1, 1, ws)
e0.record()
for _ in range(10):
    neo.neo_keyswitch(ctx, key, d, L, o0, o1, 1, ws)
e1.record()
torch.cuda.synchronize()
print(f"neo_keyswitch: {e0.elapsed_time(e1) / 10:.3f} ms/KS")

if os.environ.get("NEO_CPROFILE"):
    import cProfile
    import pstats
    pr = cProfile.Profile()
    pr.enable()
    for _ in range(10):
        limb_sharded_keyswitch(ops, plan, d, key)
    torch.cuda.synchronize()
    pr.disable()
    pstats.Stats(pr).sort_stats("tottime").print_stats(14)
