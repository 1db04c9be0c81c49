"""int8 tensor-core peak of this B200: the tcgen05 kind::i8 micro-benchmark (tools/microbench/
i8peak.cu: the NTT / BConv kernels' own MMA path, operands in shared memory, no HBM traffic)
cross-checked with torch._int_mm (cuBLASLt int8 GEMM, s8 x s8 -> s32) on large square
matrices.  Writes profiles/int8_peak.json (bench.py reports the tensor-core kernels' int8
fraction against it).  usage: python tools/i8peak.py [out.json]"""
import json
import os
import subprocess
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
out_path = sys.argv[1] if len(sys.argv) > 1 else os.path.join(ROOT, "profiles", "int8_peak.json")
src = os.path.join(ROOT, "tools", "microbench", "i8peak.cu")
exe = "/tmp/neo_i8peak"
subprocess.check_call(["/usr/local/cuda/bin/nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-o", exe, src])
tc = json.loads(subprocess.check_output([exe]).decode())

res = []
for n in (4096, 8192, 16384):
    a = torch.randint(-128, 127, (n, n), dtype=torch.int8, device="cuda")
    b = torch.randint(-128, 127, (n, n), dtype=torch.int8, device="cuda")
    for _ in range(3):
        torch._int_mm(a, b)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    reps = 20
    e0.record()
    for _ in range(reps):
        torch._int_mm(a, b)
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / reps
    res.append({"M": n, "N": n, "K": n, "ms": round(ms, 4), "tops": round(2 * n ** 3 / (ms * 1e-3) / 1e12, 1)})
out = {"tcgen05_i8_smem": tc, "torch_int_mm": res,
       "note": "tcgen05 figures are the tensor pipe alone (operands resident in shared memory); "
               "torch._int_mm is cuBLASLt end to end (HBM operands). Nominal dense int8: 4.5 POPS."}
print(json.dumps(out))
os.makedirs(os.path.dirname(out_path), exist_ok=True)
with open(out_path, "w") as f:
    json.dump(out, f, indent=1)
