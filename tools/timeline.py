"""Launch timeline of one bench step (2 streams, no graph): which kernels overlap.
usage: python tools/timeline.py"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_isca_jiaodwfcm0z25_b200 import neo  # noqa: E402

ctx = neo.Context(16, 36, 12, 3)
N, L, Lq = ctx.N, 35, 36
g = torch.Generator(device="cuda")
g.manual_seed(3)
rnd = lambda *s: torch.randint(0, 1 << 35, s, dtype=torch.int64, device="cuda", generator=g).view(torch.uint64)
relin, rot = neo.EvalKey(ctx, rnd(3, 2, 48, N)), neo.EvalKey(ctx, rnd(3, 2, 48, N))
a, b, c = rnd(1, 2, Lq, N), rnd(1, 2, Lq, N), rnd(1, 2, Lq, N)
hm, rs, hr = torch.empty_like(a), rnd(1, 2, L, N), torch.empty_like(a)
wsn = max(ctx.workspace_size(op, L, 1) for op in (1, 2, 3))
ws1 = torch.empty(wsn // 8, dtype=torch.uint64, device="cuda")
ws2 = torch.empty_like(ws1)
side = torch.cuda.Stream()
main = torch.cuda.current_stream()
def step():
    ev = torch.cuda.Event()
    ev.record(main)
    side.wait_event(ev)
    neo.neo_hrot(ctx, rot, 5, c, L, hr, 1, ws2, stream=side)
    neo.neo_hmult(ctx, relin, a, b, L, hm, 1, ws1, stream=main)
    neo.neo_rescale(ctx, hm, L, rs, 1, ws1, stream=main)
    ev2 = torch.cuda.Event()
    ev2.record(side)
    main.wait_event(ev2)
for _ in range(5):
    step()
torch.cuda.synchronize()
neo.neo_profile_enable(True)
step()
tl = neo.neo_profile_timeline()
neo.neo_profile_enable(False)
# issue order: hrot launches first (side stream), then hmult + rescale (main)
for i, (k, s, e) in enumerate(tl):
    print(f"{i:3d} {k:18s} {s * 1e3:8.1f} {e * 1e3:8.1f} {1e3 * (e - s):7.1f}")
print("step span us", 1e3 * (max(e for _, _, e in tl) - min(s for _, s, _ in tl)))
