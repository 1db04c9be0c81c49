"""Micro-benchmark of the NTT passes at Set-B (N = 2^16): neo_ntt / neo_intt over n limbs
(default 108, the ModUp launch shape), per-pass device time from neo_profile, and the
FP64-op and byte rates they imply.  usage: python tools/ntt_bench.py [n_limbs] [reps] [tc|fp64 ...]"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synth  # noqa: E402
from paper_conf_isca_jiaodwfcm0z25_b200 import neo  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 108
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 50
impls = sys.argv[3:] or ["tc", "fp64"]
ctx = neo.Context(16, 36, 12, 3)
N = ctx.N
ids = [i % 48 for i in range(n)]
x = torch.from_numpy(synth.uniform_residues(5, [ctx.moduli[i] for i in ids], N)).cuda()
ws = torch.empty(n * N, dtype=torch.uint64, device="cuda")
for impl in impls:
  ctx.ntt_select(neo.NEO_NTT_TC if impl == "tc" else neo.NEO_NTT_FP64)
  print("==", impl)
  for _ in range(3):
    neo.neo_ntt(ctx, x, ids, 1, ws)
    neo.neo_intt(ctx, x, ids, 1, ws)
  torch.cuda.synchronize()
  neo.neo_profile_enable(True)
  for _ in range(reps):
    neo.neo_ntt(ctx, x, ids, 1, ws)
    neo.neo_intt(ctx, x, ids, 1, ws)
  prof = neo.neo_profile_read()
  neo.neo_profile_enable(False)
  limb = N * 8
  tot = 0.0
  for k in ("ntt_col", "ntt_row"):
    ms, cnt = prof[k]
    us = ms * 1e3 / cnt
    tot += us
    print(f"{k}: {us:.2f} us/launch ({cnt} launches, {n} limbs) = {us / n * 1e3:.1f} ns/limb, "
          f"{2 * n * limb / us / 1e3:.0f} GB/s algorithmic")
  print(f"fwd+inv per limb: {tot / n * 1e3:.1f} ns ({tot / 2 / n * 1e3:.1f} ns per limb transform)")
