"""Dump the BConv pipeline trace of CTA 0 (NEO_BCONV_DBG=1): one ModUp (3 digits) at Set-B."""
import ctypes, os, sys
os.environ["NEO_BCONV_DBG"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_isca_jiaodwfcm0z25_b200 import neo
import bench
ctx = neo.Context(16, 36, 12, 3)
N = ctx.N
evk = neo.EvalKey(ctx, torch.from_numpy(bench.rand_evk(ctx.moduli, 5, N)).cuda())
d = torch.from_numpy(bench.rand_limbs(ctx.q, 7, N)[None]).cuda()
o0 = torch.empty_like(d); o1 = torch.empty_like(d)
ws = ctx.workspace(neo.NEO_OP_KEYSWITCH, 35, 1)
for _ in range(3):
    neo.neo_keyswitch(ctx, evk, d, 35, o0, o1, 1, ws)
torch.cuda.synchronize()
tr = neo.neo_debug_bconv_trace()
assert tr is not None, "tracing is off (NEO_BCONV_DBG)"
names = ["prod_start", "prod_fullA", "mma_go", "mma_done", "epi_start", "epi_end"]
for which, off in (("ModUp", 0), ("ModDown", 512)):
    a = np.array(tr[off // 512], dtype=np.int64)
    t0 = a[0, 0]
    n = int((a[:62, 0] > 0).sum())
    print(which, "tiles traced:", n)
    for i in range(min(n, 4)):
        print(i, " ".join(f"{names[k]}={a[i,k]-t0:7d}" for k in range(6)))
    rel = a[:n, :6] - a[:n, :1]
    print("mean per tile (cycles rel. to prod_start):", {names[k]: int(np.mean(rel[:, k])) for k in range(6)})
    print("tile period (prod_start diff):", int(np.mean(np.diff(a[:n, 0]))), "epi_end diff:", int(np.mean(np.diff(a[:n, 5]))))
    c = a[62]
    print("clock64 CTA0 rel. to entry: setup done", int(c[1] - c[0]), "pdl", int(c[2] - c[0]), "tile0 prod_start", int(t0 - c[0]),
          "prefill stage0/1/2 issued", [int(c[4 + k] - c[0]) for k in range(3)], "last epi_end", int(a[n - 1, 5] - c[0]), "exit", int(c[3] - c[0]))
    g = a[63]
    print("setup ns CTA0 [entry, setup done, pdl done, exit]:", [int(g[k] - g[0]) for k in range(4)],
          "| last CTA start skew", int(g[4] - g[0]), [int(g[4 + k] - g[4]) for k in range(4)])
