"""Per-kernel-kind breakdown of one Set-C key-switch, KLSS vs Hybrid (neo_profile events).
usage: python tools/klss_profile.py [batch]"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_isca_jiaodwfcm0z25_b200 import neo  # noqa: E402

B = int(sys.argv[1]) if len(sys.argv) > 1 else 1
ctx = neo.Context(16, 36, 4, 9, alpha_t=5)
N, L = ctx.N, 35
g = torch.Generator(device="cuda")
g.manual_seed(1)
rnd = lambda *s: torch.randint(0, 1 << 35, s, dtype=torch.int64, device="cuda", generator=g).view(torch.uint64)
keys = {"klss": neo.EvalKey(ctx, rnd(2, 8, 9, ctx.alpha_p, N), klss=True), "hybrid": neo.EvalKey(ctx, rnd(9, 2, 40, N))}
d = rnd(B, L + 1, N)
o0, o1 = torch.empty_like(d), torch.empty_like(d)
ws = ctx.workspace(neo.NEO_OP_KEYSWITCH, L, B)
for name, k in keys.items():
    for _ in range(3):
        neo.neo_keyswitch(ctx, k, d, L, o0, o1, B, ws)
    torch.cuda.synchronize()
    neo.neo_profile_enable(True)
    for _ in range(10):
        neo.neo_keyswitch(ctx, k, d, L, o0, o1, B, ws)
    pr = neo.neo_profile_read()
    neo.neo_profile_enable(False)
    tot = sum(v[0] for v in pr.values()) / 10
    print(name, f"B={B} total {tot:.4f} ms/KS:", " ".join(f"{kk}={v[0] / 10:.4f}({v[1] // 10})" for kk, v in pr.items() if v[1]))
