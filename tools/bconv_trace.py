"""Dump the tensor-core BConv pipeline trace of CTA 0 (NEO_BCONV_DBG=1) for one Set-B key-switch.

Rows 0..59: per tile [producer in, A ready, MMA start, MMA committed, epilogue part-0 start,
last part end] (clock64); row 60: cycles spent waiting per barrier (TMA in_empty, producer
in_full, producer empty_a, epilogue set-0 tmem_full, MMA full_a, MMA tmem_empty) and the end
stamps of epilogue warp 4 / producer thread 0."""
import os
import sys

os.environ["NEO_BCONV_DBG"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_isca_jiaodwfcm0z25_b200 import neo  # noqa: E402

ctx = neo.Context(16, 36, 12, 3)
N = ctx.N
evk = neo.EvalKey(ctx, torch.from_numpy(bench.rand_evk(ctx.moduli, 5, N)).cuda())
d = torch.from_numpy(bench.rand_limbs(ctx.q, 7, N)[None]).cuda()
o0 = torch.empty_like(d)
o1 = torch.empty_like(d)
ws = ctx.workspace(neo.NEO_OP_KEYSWITCH, 35, 1)
for _ in range(3):
    neo.neo_keyswitch(ctx, evk, d, 35, o0, o1, 1, ws)
torch.cuda.synchronize()
tr = neo.neo_debug_bconv_trace()
assert tr is not None, "tracing is off (NEO_BCONV_DBG)"
names = ["prod_in", "prod_A", "mma_go", "mma_done", "epi_start", "epi_end"]
for which, w in (("ModUp", 0), ("ModDown", 1)):
    a = np.array(tr[w], dtype=np.int64)
    t0 = a[0, 0]
    n = int((a[:60, 0] > 0).sum())
    print(which, "tiles traced:", n)
    rel = a[:n, :6] - a[:n, :1]
    print("  mean per tile (cycles rel. to prod_in):", {names[k]: int(np.mean(rel[:, k])) for k in range(6)})
    print("  tile period (prod_in diff):", int(np.mean(np.diff(a[:n, 0]))), "epi_end diff:", int(np.mean(np.diff(a[:n, 5]))))
    span = int(max(a[60, 6], a[60, 7]) - t0)
    print(f"  waiting cycles (span from tile 0 {span}):", {"tma in_empty": int(a[60, 0]), "prod in_full": int(a[60, 1]),
          "prod empty_a": int(a[60, 2]), "epi tfull (set 0)": int(a[60, 3]), "mma full_a": int(a[60, 4]),
          "mma tempty": int(a[60, 5])})
    st = a[61, :4]                                   # setup stamps of CTA 0: entry, TMEM allocated, set up, past PDL wait
    if st[0]:
        print(f"  setup (cycles from kernel entry): TMEM alloc {int(st[1] - st[0])}, tables / barriers / B "
              f"{int(st[2] - st[1])}, PDL wait {int(st[3] - st[2])}, to tile 0 input {int(t0 - st[3])}, "
              f"last epilogue end {int(max(a[60, 6], a[60, 7]) - st[0])}")
