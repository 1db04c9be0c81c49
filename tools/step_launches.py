"""Per-launch device time of one bench step on ONE stream (HMULT+Rescale fused, then HROTATE, Set-B
l=35, B=1), event-timed per launch: where the step's time goes, launch by launch.
usage: python tools/step_launches.py [fp64|tc]"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_isca_jiaodwfcm0z25_b200 import neo  # noqa: E402

ctx = neo.Context(16, 36, 12, 3)
if len(sys.argv) > 1 and sys.argv[1] == "tc":
    ctx.ntt_select(neo.NEO_NTT_TC)
N, L, Lq = ctx.N, 35, 36
g = torch.Generator(device="cuda")
g.manual_seed(3)
rnd = lambda *s: torch.randint(0, 1 << 35, s, dtype=torch.int64, device="cuda", generator=g).view(torch.uint64)
relin, rot = neo.EvalKey(ctx, rnd(3, 2, 48, N)), neo.EvalKey(ctx, rnd(3, 2, 48, N))
a, b, c = rnd(1, 2, Lq, N), rnd(1, 2, Lq, N), rnd(1, 2, Lq, N)
rs, hr = rnd(1, 2, L, N), torch.empty_like(a)
wsn = max(ctx.workspace_size(op, L, 1) for op in (neo.NEO_OP_HROT, neo.NEO_OP_HMULT_RESCALE))
ws = torch.empty(wsn // 8, dtype=torch.uint64, device="cuda")


def step():
    neo.neo_hmult_rescale(ctx, relin, a, b, L, rs, 1, ws)
    neo.neo_hrot(ctx, rot, 5, c, L, hr, 1, ws)


for _ in range(5):
    step()
torch.cuda.synchronize()
acc = {}
reps = 20
for r in range(reps):
    neo.neo_profile_enable(True)
    step()
    tl = neo.neo_profile_timeline()
    neo.neo_profile_enable(False)
    for i, (k, s, e) in enumerate(tl):
        acc.setdefault(i, [k, 0.0])[1] += (e - s) * 1e3 / reps
tot = sum(v for _, v in acc.values())
for i, (k, us) in acc.items():
    print(f"{i:3d} {k:18s} {us:8.1f} us")
print(f"sum {tot:.1f} us")
