"""Experiment: the bench step (HMULT+Rescale on one stream || HROTATE on another, Set-B l=35,
B=1, CUDA graph) with each chain's NTT implementation chosen separately (two contexts), to see
whether running the FP64 NTT on one chain and the tcgen05 NTT on the other overlaps better.
usage: python tools/mix_ntt.py"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_isca_jiaodwfcm0z25_b200 import neo  # noqa: E402

N, L, Lq = 1 << 16, 35, 36
g = torch.Generator(device="cuda")
g.manual_seed(3)
rnd = lambda *s: torch.randint(0, 1 << 35, s, dtype=torch.int64, device="cuda", generator=g).view(torch.uint64)
ca, cb = neo.Context(16, 36, 12, 3), neo.Context(16, 36, 12, 3)
relin, rot = neo.EvalKey(ca, rnd(3, 2, 48, N)), neo.EvalKey(cb, rnd(3, 2, 48, N))
a, b, c = rnd(1, 2, Lq, N), rnd(1, 2, Lq, N), rnd(1, 2, Lq, N)
rs, hr = rnd(1, 2, L, N), torch.empty_like(a)
wa = ca.workspace(neo.NEO_OP_HMULT_RESCALE, L, 1)
wb = cb.workspace(neo.NEO_OP_HROT, L, 1)
side = torch.cuda.Stream()
e0, e1 = torch.cuda.Event(), torch.cuda.Event()


def step():
    main = torch.cuda.current_stream()
    e0.record(main)
    side.wait_event(e0)
    neo.neo_hrot(cb, rot, 5, c, L, hr, 1, wb, stream=side)
    neo.neo_hmult_rescale(ca, relin, a, b, L, rs, 1, wa, stream=main)
    e1.record(side)
    main.wait_event(e1)


for ia, ib in ((0, 0), (0, 1), (1, 0), (1, 1), (0, 0)):
    ca.ntt_select(ia)
    cb.ntt_select(ib)
    for _ in range(5):
        step()
    torch.cuda.synchronize()
    gr = torch.cuda.CUDAGraph()
    with torch.cuda.graph(gr):
        step()
    for _ in range(20):
        gr.replay()
    torch.cuda.synchronize()
    t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t0.record()
    for _ in range(1000):
        gr.replay()
    t1.record()
    torch.cuda.synchronize()
    ms = t0.elapsed_time(t1) / 1000
    print(f"HMULT+Rescale NTT={'tc' if ia else 'fp64'}  HROT NTT={'tc' if ib else 'fp64'}: {ms:.4f} ms/step, {2 / ms * 1e3:.0f} KS/s")
