"""Per-launch breakdown of one Set-C key-switch (level 35), KLSS vs Hybrid (neo_profile events).
usage: python tools/klss_profile.py [batch] [word_bits_t]   (default 1, 48)"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_isca_jiaodwfcm0z25_b200 import neo  # noqa: E402

B = int(sys.argv[1]) if len(sys.argv) > 1 else 1
WT = int(sys.argv[2]) if len(sys.argv) > 2 else 48
ctx = neo.Context(16, 36, 4, 9, alpha_t=5, word_bits_t=WT)
N, L = ctx.N, 35
g = torch.Generator(device="cuda")
g.manual_seed(1)
rnd = lambda *s: torch.randint(0, 1 << 35, s, dtype=torch.int64, device="cuda", generator=g).view(torch.uint64)
keys = {"klss": neo.EvalKey(ctx, rnd(2, 8, 9, ctx.alpha_p, N), klss=True), "hybrid": neo.EvalKey(ctx, rnd(9, 2, 40, N))}
d = rnd(B, L + 1, N)
o0, o1 = torch.empty_like(d), torch.empty_like(d)
ws = ctx.workspace(neo.NEO_OP_KEYSWITCH, L, B)
reps = 10
print(f"Set-C l=35 B={B} WordSize_T={WT} alpha'={ctx.alpha_p}")
for name, k in keys.items():
    for _ in range(3):
        neo.neo_keyswitch(ctx, k, d, L, o0, o1, B, ws)
    torch.cuda.synchronize()
    acc = {}
    for _ in range(reps):
        neo.neo_profile_enable(True)
        neo.neo_keyswitch(ctx, k, d, L, o0, o1, B, ws)
        tl = neo.neo_profile_timeline()
        neo.neo_profile_enable(False)
        for i, (kind, s, e) in enumerate(tl):
            acc.setdefault(i, [kind, 0.0])[1] += (e - s) * 1e3 / reps
    tot = sum(v for _, v in acc.values())
    print(f"{name}: {len(acc)} launches, {tot:.1f} us")
    for i, (kind, us) in acc.items():
        print(f"  {i:3d} {kind:18s} {us:8.1f} us")
