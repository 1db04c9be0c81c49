"""Per-phase timing of the Set-B bootstrapping (CUDA events between the phases of
Bootstrapper.run, replicated here) and per-kernel-kind totals (neo_profile)."""
import math
import sys
import os

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_isca_jiaodwfcm0z25_b200 import neo, boot as gboot  # noqa: E402

N, NQ, NP, DNUM, L = 1 << 16, 36, 12, 3, 35
nb, rb = 8, 12
ctx = neo.Context(16, NQ, NP, DNUM)
gen = torch.Generator(device="cuda")
gen.manual_seed(7)
rnd = lambda *s: torch.randint(0, 1 << 35, s, dtype=torch.int64, device="cuda", generator=gen).view(torch.uint64)
evk = rnd(DNUM, 2, NQ + NP, N)
keys = {"relin": neo.EvalKey(ctx, evk)}
for g in gboot.rotations(N, nb):
    keys[g] = neo.EvalKey(ctx, evk)
for g in gboot.hoisted_rotations(N, nb):
    keys[("h", g)] = neo.EvalKey(ctx, evk, hoisted_galois=g)
consts = {k: rnd(l + 1, N) for k, l in gboot.const_levels(L, nb, rb).items()}
bt = gboot.Bootstrapper(ctx, nb, rb, keys, consts)
ct0 = rnd(1, 2, 1, N)

marks = []
orig = {name: getattr(bt, name) for name in ("rot", "hmul", "rescale", "pmul", "add", "sub", "padd", "drop")}
cur = ["other"]
acc = {}


def wrap(name):
    f = orig[name]

    def g(*a, **k):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        r = f(*a, **k)
        e1.record()
        marks.append((name, a[0].shape[0] if hasattr(a[0], "shape") else 1, e0, e1))
        return r
    return g


for _ in range(2):
    bt.run(ct0)
torch.cuda.synchronize()
for name in orig:
    setattr(bt, name, wrap(name))
t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
t0.record()
bt.run(ct0)
t1.record()
torch.cuda.synchronize()
tot = t0.elapsed_time(t1)
by = {}
for name, B, a, b in marks:
    k = f"{name}(B={B})"
    c, t = by.get(k, (0, 0.0))
    by[k] = (c + 1, t + a.elapsed_time(b))
print(f"total {tot:.3f} ms (wrapped ops {sum(t for _, t in by.values()):.3f})")
for k, (c, t) in sorted(by.items(), key=lambda x: -x[1][1]):
    print(f"  {k:16s} n={c:3d} {t:8.3f} ms  {t / c:.4f} ms/op")
