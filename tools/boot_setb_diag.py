"""Diagnostic: stage-by-stage accuracy of the Set-B full-slot bootstrap on the GPU (CoeffToSlot
output against the exact bit-reversed coefficients of the ModRaised plaintext; the final
output against the input), decoding sampled slots with the oracle (test infrastructure)."""
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import synth  # noqa: E402
from oracle import boot, ckks  # noqa: E402
from paper_conf_isca_jiaodwfcm0z25_b200 import boot as gboot, neo  # noqa: E402

boost = tuple(int(x) for x in (sys.argv[1:3] if len(sys.argv) > 2 else (20, 20)))
h = int(sys.argv[3]) if len(sys.argv) > 3 else 192
r = int(sys.argv[4]) if len(sys.argv) > 4 else 12
bp = boot.BootParams(ckks.set_b(), n=32768, r=r, h=h, fft_levels=4, boost=boost)
prm = bp.prm
N = prm.N
t0 = time.time()
s = ckks.secret(prm, 61, bp.h)
keys_np = boot.boot_keys(bp, s, 700)
lv_out, scale_out, consts = boot.dry_run(bp)
print(f"keys + consts {time.time() - t0:.0f} s", flush=True)
z = synth.complex_slots(63, N // 2)
delta = 2.0 ** 31
ct0 = ckks.encrypt(prm, ckks.encode_fft(N, z, delta), s, 0, 65)
ctx = neo.Context(prm.log_n, prm.num_q, prm.num_p, prm.dnum)
dev = lambda a: torch.from_numpy(np.ascontiguousarray(a, dtype=np.uint64)).cuda()
keys = {k: neo.EvalKey(ctx, dev(v)) for k, v in keys_np.items()}
for g in gboot.hoisted_rotations(N, bp.n, bp.fft_levels):
    keys[("h", g)] = neo.EvalKey(ctx, dev(keys_np[g]), hoisted_galois=g)
b = gboot.Bootstrapper(ctx, bp.n, bp.r, keys, {k: dev(v) for k, v in consts.items()}, fft_levels=bp.fft_levels,
                       boost=bp.boost)
js = np.random.default_rng(7).choice(N // 2, 128, replace=False)


def dec_coeffs(ct, level):
    return ckks.crt_centered(prm, ckks.decrypt_residues(prm, ct, s, level), list(range(level + 1)))


def slots(m, scale, sel):
    mf = np.array([float(v) for v in m])
    e = np.array([pow(5, int(j), 2 * N) for j in sel], dtype=np.int64)
    k = np.arange(N, dtype=np.int64)
    return np.array([np.exp(1j * np.pi * ((ej * k) % (2 * N)) / N) @ mf for ej in e]) / scale


L = bp.top
x = dev(ct0[None])
raised = b.modraise(x, L)
p = dec_coeffs(raised.cpu().numpy()[0], L)
q0 = prm.q[0]
t = np.array([float(v) / q0 for v in p])
n = N // 2
brev = np.array([int(format(i, f"0{int(np.log2(n))}b")[::-1], 2) for i in range(n)])
want_w = t[:n][brev] + 1j * t[n:][brev]
print(f"ModRaise: |t| max {np.max(np.abs(t)):.3e}, |I| max {np.max(np.abs(np.round(t))):.0f}", flush=True)
ct = raised
sc = float(q0)
if boost[0]:
    ct = b.pmul(ct, "boost_cts", L)
    sc *= float(1 << boost[0])
cts, lv = b.lintrans_fft(ct, L, True, "cts")
torch.cuda.synchronize()
got_w = slots(dec_coeffs(cts.cpu().numpy()[0], lv), sc, js)
print(f"CoeffToSlot (level {lv}): max |w - exact| {np.max(np.abs(got_w - want_w[js])):.3e} "
      f"(|w| max {np.max(np.abs(want_w[js])):.3e})", flush=True)
out, glv = b.run(x)
torch.cuda.synchronize()
zz = slots(dec_coeffs(out.cpu().numpy()[0], glv), scale_out * delta / q0, js)
print(f"bootstrap (level {glv}): max slot error {np.max(np.abs(zz - z[js])):.3e}", flush=True)
