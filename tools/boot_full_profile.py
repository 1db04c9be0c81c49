"""Phase timing of the Set-B full-slot bootstrap (CUDA events around the phases, eager)."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_isca_jiaodwfcm0z25_b200 import neo, boot as gboot  # noqa: E402

N, NQ, NP, DNUM, L = 1 << 16, 36, 12, 3, 35
nb, rb, fl = N // 2, int(os.environ.get("R", "9")), int(os.environ.get("FL", "4"))
boost, ds_sq = (20, 20), int(os.environ.get("DS", "4"))      # bench.py's configuration (oracle.boot.set_b_full)
ctx = neo.Context(16, NQ, NP, DNUM)
rnd = lambda *s: torch.randint(0, 1 << 35, s, dtype=torch.int64, device="cuda").view(torch.uint64)
evk = rnd(DNUM, 2, NQ + NP, N)
keys = {"relin": neo.EvalKey(ctx, evk)}
for g in gboot.rotations(N, nb, fl):
    keys[g] = neo.EvalKey(ctx, evk)
for g in gboot.hoisted_rotations(N, nb, fl):
    keys[("h", g)] = neo.EvalKey(ctx, evk, hoisted_galois=g)
consts = {k: rnd(l + 1, N) for k, l in gboot.const_levels(L, nb, rb, N, fl, boost, ds_sq).items()}
bt = gboot.Bootstrapper(ctx, nb, rb, keys, consts, fft_levels=fl, boost=boost, ds_sq=ds_sq)
ct0 = rnd(1, 2, 1, N)
for _ in range(2):
    bt.run(ct0)
torch.cuda.synchronize()
marks = {}
orig_lt = bt.lintrans_fft


def lt(ct, lv, inverse, tag):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    r = orig_lt(ct, lv, inverse, tag)
    e1.record()
    marks[tag] = (e0, e1)
    return r


bt.lintrans_fft = lt
t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
t0.record()
bt.run(ct0)
t1.record()
torch.cuda.synchronize()
tot = t0.elapsed_time(t1)
print(f"total {tot:.2f} ms (eager)")
neo.neo_profile_enable(True)
bt.run(ct0)
pr = neo.neo_profile_read()
neo.neo_profile_enable(False)
print("per kind (ms, launches):", {k: (round(v[0], 3), v[1]) for k, v in pr.items() if v[1]})
for k, (a, b) in marks.items():
    print(f"  {k}: {a.elapsed_time(b):.2f} ms")
print(f"  rest (ModRaise, conj split, EvalMod, combine): {tot - sum(a.elapsed_time(b) for a, b in marks.values()):.2f} ms")
for lvl in (True, False):
    print("plan", [(h, b1, len(ms)) for h, b1, ms in gboot.fft_plan(N, fl, lvl)])
