"""Time neo_bconv (tensor-core path) vs batch to separate fixed and per-tile costs."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_isca_jiaodwfcm0z25_b200 import neo
ctx = neo.Context(16, 36, 12, 3)
N = ctx.N
src = list(range(12)); dst = list(range(12, 48))
for B in (1, 2, 4, 8, 16):
    x = torch.randint(0, 2**35, (B, 12, N), dtype=torch.int64, device="cuda").view(torch.uint64)
    out = torch.empty((B, 36, N), dtype=torch.uint64, device="cuda")
    for _ in range(3):
        neo.neo_bconv(ctx, x, src, out, dst, B)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    R = 20
    e0.record()
    for _ in range(R):
        neo.neo_bconv(ctx, x, src, out, dst, B)
    e1.record(); torch.cuda.synchronize()
    us = e0.elapsed_time(e1) / R * 1e3
    tiles = B * N // 128
    gb = B * 48 * N * 8 / 1e9
    print(f"B={B:2d} tiles={tiles:5d} {us:8.1f} us  {gb/us*1e6/1e3:6.2f} TB/s  per-tile-per-SM {us/(tiles/148):.2f} us")
