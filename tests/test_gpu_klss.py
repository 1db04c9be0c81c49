"""GPU parity of the KLSS key-switch (L155-180, readings K1-K6) through the
C-ABI against the CPU oracle (oracle/klss.py), bit-exact on every residue: the tiny KLSS set
(N = 2^12) at several levels and batches, and Set-C (N = 2^16, dnum = 9, alpha~ = 5) at l = 35 in
the launch configuration bench.py times, with T primes of 36 bits (10 of them) and of 48 bits
(WordSize_T = 48 as Table 4 prints it, L511: 8 of them; reading K6)."""
import numpy as np
import pytest
import torch

import synth
from oracle import ckks, klss

pytestmark = pytest.mark.gpu

neo = pytest.importorskip("paper_conf_isca_jiaodwfcm0z25_b200.neo")

_CACHE = {}


def setup(name):
    if name not in _CACHE:
        kp = {"tiny": klss.tiny, "setc": klss.set_c_t36, "tiny48": klss.tiny48, "setc48": klss.set_c}[name]()
        b = kp.base
        ctx = neo.Context(b.log_n, b.num_q, b.num_p, b.dnum, alpha_t=kp.alpha_t, word_bits_t=kp.word_bits_t)
        evk = np.stack([np.stack([synth.uniform_residues(600 + 2 * j + c, b.moduli, b.N) for c in range(2)])
                        for j in range(b.dnum)])
        ek = klss.klss_key(kp, evk)
        key = neo.EvalKey(ctx, dev(ek), klss=True)
        _CACHE[name] = (kp, ctx, evk, ek, key)
    return _CACHE[name]


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.uint64)).cuda()


def host(t):
    torch.cuda.synchronize()
    return t.cpu().numpy()


@pytest.mark.parametrize("name", ["tiny", "setc", "tiny48", "setc48"])
def test_klss_params_match_oracle(name):
    kp, ctx, *_ = setup(name)
    assert ctx.q == kp.base.q and ctx.p == kp.base.p
    assert ctx.alpha_t == kp.alpha_t and ctx.alpha_p == kp.alpha_p and ctx.t == kp.t


@pytest.mark.parametrize("name,level,batch", [("tiny", 5, 2), ("tiny", 3, 1), ("tiny", 0, 1), ("setc", 35, 1),
                                              ("tiny", 5, 34),      # 34: two chunks on two streams
                                              ("tiny48", 5, 2), ("tiny48", 3, 1), ("tiny48", 0, 1),
                                              ("setc48", 35, 2), ("setc48", 20, 1), ("setc48", 3, 1)])
def test_klss_keyswitch(name, level, batch):
    kp, ctx, evk, ek, key = setup(name)
    b = kp.base
    d = np.stack([synth.uniform_residues(700 + 3 * bb + level, b.q[:level + 1], b.N) for bb in range(batch)])
    o0 = torch.empty((batch, level + 1, b.N), dtype=torch.uint64, device="cuda")
    o1 = torch.empty_like(o0)
    ws = ctx.workspace(neo.NEO_OP_KEYSWITCH, level, batch)
    neo.neo_keyswitch(ctx, key, dev(d), level, o0, o1, batch, ws)
    g0, g1 = host(o0), host(o1)
    for bb in range(batch):
        w0, w1 = klss.keyswitch(kp, d[bb], level, ek)
        assert np.array_equal(g0[bb], w0) and np.array_equal(g1[bb], w1)


@pytest.mark.parametrize("name,level", [("tiny", 5), ("setc", 35), ("tiny48", 5), ("setc48", 35)])
def test_klss_hmult_hrot(name, level):
    kp, ctx, evk, ek, key = setup(name)
    b = kp.base
    ids = list(range(level + 1))
    cts = [np.stack([synth.uniform_residues(800 + 2 * k + c, [b.moduli[i] for i in ids], b.N) for c in range(2)])
           for k in range(3)]
    out = torch.empty((1, 2, level + 1, b.N), dtype=torch.uint64, device="cuda")
    neo.neo_hmult(ctx, key, dev(cts[0][None]), dev(cts[1][None]), level, out, 1,
                  ctx.workspace(neo.NEO_OP_HMULT, level, 1))
    assert np.array_equal(host(out)[0], klss.hmult(kp, cts[0], cts[1], level, ek))
    g = 5
    neo.neo_hrot(ctx, key, g, dev(cts[2][None]), level, out, 1, ctx.workspace(neo.NEO_OP_HROT, level, 1))
    assert np.array_equal(host(out)[0], klss.hrot(kp, cts[2], g, level, ek))


def test_klss_key_rejected_without_t_primes():
    kp, ctx, evk, ek, key = setup("tiny")
    b = kp.base
    plain = neo.Context(b.log_n, b.num_q, b.num_p, b.dnum)
    with pytest.raises(neo.NeoError):
        neo.EvalKey(plain, dev(ek), klss=True)


@pytest.mark.parametrize("name,level", [("tiny48", 5), ("setc48", 35)])
def test_klss48_extremal(name, level):
    """WordSize_T = 48 at its extremes: every key word t_k - 1 and every input residue q_i - 1
    (the largest 64-bit IP products, BConv byte planes and T-basis NTT magnitudes), and zeros."""
    kp, ctx, evk, ek, key = setup(name)
    b = kp.base
    ek_max = np.empty_like(ek)
    for k, t in enumerate(kp.t):
        ek_max[:, :, :, k, :] = t - 1
    kmax = neo.EvalKey(ctx, dev(ek_max), klss=True)
    for fill in ("max", "zero"):
        d = np.stack([np.full(b.N, (q - 1) if fill == "max" else 0, dtype=np.uint64) for q in b.q[:level + 1]])
        o0 = torch.empty((1, level + 1, b.N), dtype=torch.uint64, device="cuda")
        o1 = torch.empty_like(o0)
        neo.neo_keyswitch(ctx, kmax, dev(d[None]), level, o0, o1, 1, ctx.workspace(neo.NEO_OP_KEYSWITCH, level, 1))
        w0, w1 = klss.keyswitch(kp, d, level, ek_max)
        assert np.array_equal(host(o0)[0], w0) and np.array_equal(host(o1)[0], w1)
