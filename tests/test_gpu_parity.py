"""GPU parity: every stage of the CUDA path (through the C-ABI) against the CPU oracle,
element by element and bit-exact on every residue (integer work: SURVEY §8(c) Z23).

Inputs are seeded (synth); expected values come only from oracle/.  Sizes: the tiny config
(N=2^12) with ragged shapes and batches, and Set-B (N=2^16, 36+12 limbs, dnum=3) in the
launch configuration bench.py times."""
import numpy as np
import pytest
import torch

import synth
from oracle import ckks

pytestmark = pytest.mark.gpu

neo = pytest.importorskip("paper_conf_isca_jiaodwfcm0z25_b200.neo")

_CTX = {}
_PRM = {}


def ctx_of(name):
    if name not in _CTX:
        prm = {"tiny": ckks.tiny, "tiny3": ckks.tiny_dnum3, "setb": ckks.set_b}[name]()
        _PRM[name] = prm
        _CTX[name] = neo.Context(prm.log_n, prm.num_q, prm.num_p, prm.dnum)
    return _CTX[name], _PRM[name]


def dev(a: np.ndarray) -> torch.Tensor:
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.uint64)).cuda()


def host(t: torch.Tensor) -> np.ndarray:
    torch.cuda.synchronize()
    return t.cpu().numpy()


def rand_poly(prm, ids, seed):
    return synth.uniform_residues(seed, [prm.moduli[i] for i in ids], prm.N)


def rand_ct(prm, level, seed):
    ids = list(range(level + 1))
    return np.stack([rand_poly(prm, ids, seed), rand_poly(prm, ids, seed + 1)])


def rand_evk(prm, seed):
    ids = list(range(prm.num_q + prm.num_p))
    return np.stack([np.stack([rand_poly(prm, ids, seed + 2 * j + c) for c in range(2)])
                     for j in range(prm.dnum)])


@pytest.mark.parametrize("name", ["tiny", "tiny3", "setb"])
def test_params_match_oracle(name):
    ctx, prm = ctx_of(name)
    assert ctx.q == prm.q and ctx.p == prm.p and ctx.psi == prm.psi


@pytest.mark.parametrize("name,batch", [("tiny", 3), ("setb", 1)])
def test_ntt_intt(name, batch):
    ctx, prm = ctx_of(name)
    ids = list(range(prm.num_q + prm.num_p))
    x = np.stack([rand_poly(prm, ids, 100 + b) for b in range(batch)])
    t = dev(x)
    ws = torch.empty(t.numel(), dtype=torch.uint64, device="cuda")
    neo.neo_ntt(ctx, t, ids, batch, ws)
    got = host(t)
    for b in range(batch):
        assert np.array_equal(got[b], ckks.ntt(prm, x[b], ids))
    neo.neo_intt(ctx, t, ids, batch, ws)
    assert np.array_equal(host(t), x)


def test_intt_matches_oracle_ragged_ids():
    ctx, prm = ctx_of("tiny")
    ids = [3, 0, 2]                      # arbitrary order, P limb first
    x = rand_poly(prm, ids, 7)[None]
    t = dev(x)
    ws = torch.empty_like(t)
    neo.neo_intt(ctx, t, ids, 1, ws)
    assert np.array_equal(host(t)[0], ckks.intt(prm, x[0], ids))


@pytest.mark.parametrize("name,src,dst,batch", [
    ("tiny", [0, 1, 2], [3], 2),                          # ModUp of the whole digit (dnum = 1)
    ("tiny", [3], [0, 1, 2], 1),                          # ModDown shape
    ("setb", list(range(12)), list(range(12, 48)), 1),    # Set-B ModUp digit 0
    ("setb", list(range(36, 48)), list(range(36)), 2),    # Set-B ModDown
    ("setb", [5, 17, 40, 2, 33], [0, 47, 9, 21, 3, 11, 30], 1),   # ragged
])
def test_bconv(name, src, dst, batch):
    ctx, prm = ctx_of(name)
    x = np.stack([rand_poly(prm, src, 200 + b) for b in range(batch)])
    out = torch.empty((batch, len(dst), prm.N), dtype=torch.uint64, device="cuda")
    neo.neo_bconv(ctx, dev(x), src, out, dst, batch)
    got = host(out)
    for b in range(batch):
        assert np.array_equal(got[b], ckks.bconv(prm, x[b], src, dst))


@pytest.mark.parametrize("name,level,batch", [("tiny", 2, 2), ("setb", 35, 1)])
def test_tensor(name, level, batch):
    ctx, prm = ctx_of(name)
    a = np.stack([rand_ct(prm, level, 300 + 4 * b) for b in range(batch)])
    b_ = np.stack([rand_ct(prm, level, 302 + 4 * b) for b in range(batch)])
    d = torch.empty((batch, 3, level + 1, prm.N), dtype=torch.uint64, device="cuda")
    neo.neo_tensor(ctx, dev(a), dev(b_), level, d, batch)
    got = host(d)
    for bb in range(batch):
        want = ckks.tensor(prm, a[bb], b_[bb], level)
        for k in range(3):
            assert np.array_equal(got[bb, k], want[k])


@pytest.mark.parametrize("g", [5, 25, 8191, 3])
def test_automorphism(g):
    ctx, prm = ctx_of("tiny")
    x = np.stack([rand_poly(prm, [0, 1, 2, 3], 400 + b) for b in range(2)])
    out = torch.empty_like(dev(x))
    neo.neo_automorphism(ctx, dev(x), 4, g, out, 2)
    assert np.array_equal(host(out), ckks.automorphism_ntt(x, g))


def _ks(name, level, batch, seed):
    ctx, prm = ctx_of(name)
    evk_np = rand_evk(prm, seed)
    evk = neo.EvalKey(ctx, dev(evk_np))
    d = np.stack([rand_poly(prm, list(range(level + 1)), seed + 50 + b) for b in range(batch)])
    o0 = torch.empty((batch, level + 1, prm.N), dtype=torch.uint64, device="cuda")
    o1 = torch.empty_like(o0)
    ws = ctx.workspace(neo.NEO_OP_KEYSWITCH, level, batch)
    neo.neo_keyswitch(ctx, evk, dev(d), level, o0, o1, batch, ws)
    g0, g1 = host(o0), host(o1)
    for b in range(batch):
        k0, k1 = ckks.keyswitch(prm, d[b], level, evk_np)
        assert np.array_equal(g0[b], k0)
        assert np.array_equal(g1[b], k1)


@pytest.mark.parametrize("name,level,batch", [
    ("tiny", 2, 2), ("tiny", 0, 1), ("tiny3", 2, 1), ("tiny3", 1, 3),
])
def test_keyswitch_tiny(name, level, batch):
    _ks(name, level, batch, 500 + level)


@pytest.mark.parametrize("level", [35, 13, 0])
def test_keyswitch_setb(level):
    """Set-B: full level (3 full digits), a partial last digit (l = 13), and level 0."""
    _ks("setb", level, 1, 600 + level)


def test_keyswitch_setb_batch2():
    _ks("setb", 35, 2, 700)


@pytest.mark.parametrize("name,level,batch", [("tiny", 2, 2), ("setb", 35, 1)])
def test_hmult(name, level, batch):
    ctx, prm = ctx_of(name)
    evk_np = rand_evk(prm, 800)
    relin = neo.EvalKey(ctx, dev(evk_np))
    a = np.stack([rand_ct(prm, level, 810 + 4 * b) for b in range(batch)])
    b_ = np.stack([rand_ct(prm, level, 812 + 4 * b) for b in range(batch)])
    out = torch.empty((batch, 2, level + 1, prm.N), dtype=torch.uint64, device="cuda")
    ws = ctx.workspace(neo.NEO_OP_HMULT, level, batch)
    neo.neo_hmult(ctx, relin, dev(a), dev(b_), level, out, batch, ws)
    got = host(out)
    for bb in range(batch):
        assert np.array_equal(got[bb], ckks.hmult(prm, a[bb], b_[bb], level, evk_np))


@pytest.mark.parametrize("name,level,batch,r", [("tiny", 2, 2, 1), ("setb", 35, 1, 1), ("setb", 20, 1, 7),
                                                ("tiny", 2, 1, 0), ("tiny", 1, 2, "conj"), ("setb", 35, 1, "conj")])
def test_hrot(name, level, batch, r):
    """r = 0 is the identity Galois element g = 1 (Z11's special case); "conj" is g = 2N - 1."""
    ctx, prm = ctx_of(name)
    g = 2 * prm.N - 1 if r == "conj" else pow(5, r, 2 * prm.N)
    evk_np = rand_evk(prm, 900)
    rk = neo.EvalKey(ctx, dev(evk_np))
    ct = np.stack([rand_ct(prm, level, 910 + 2 * b) for b in range(batch)])
    out = torch.empty((batch, 2, level + 1, prm.N), dtype=torch.uint64, device="cuda")
    ws = ctx.workspace(neo.NEO_OP_HROT, level, batch)
    neo.neo_hrot(ctx, rk, g, dev(ct), level, out, batch, ws)
    got = host(out)
    for bb in range(batch):
        assert np.array_equal(got[bb], ckks.hrot(prm, ct[bb], g, level, evk_np))


@pytest.mark.parametrize("name,level,batch", [("tiny", 2, 2), ("tiny", 1, 1), ("setb", 35, 1)])
def test_rescale(name, level, batch):
    ctx, prm = ctx_of(name)
    ct = np.stack([rand_ct(prm, level, 1000 + 2 * b) for b in range(batch)])
    out = torch.empty((batch, 2, level, prm.N), dtype=torch.uint64, device="cuda")
    ws = ctx.workspace(neo.NEO_OP_RESCALE, level, batch)
    neo.neo_rescale(ctx, dev(ct), level, out, batch, ws)
    got = host(out)
    for bb in range(batch):
        assert np.array_equal(got[bb], ckks.rescale(prm, ct[bb], level))


def test_hmult_rescale_decrypts():
    """Real encryptions (tiny, dnum=3): GPU HMULT + Rescale decodes to z_a z_b within 1e-6
    at Delta = 2^40 and equals the oracle bit for bit."""
    ctx, prm = ctx_of("tiny3")
    delta = 2.0 ** 40
    s = ckks.secret(prm, 11, 192)
    za, zb = synth.complex_slots(101, prm.N // 2), synth.complex_slots(102, prm.N // 2)
    cta = ckks.encrypt(prm, ckks.encode(prm.N, za, delta), s, 2, 201)
    ctb = ckks.encrypt(prm, ckks.encode(prm.N, zb, delta), s, 2, 202)
    relin_np = ckks.relin_key(prm, s, 301)
    relin = neo.EvalKey(ctx, dev(relin_np))
    out = torch.empty((1, 2, 3, prm.N), dtype=torch.uint64, device="cuda")
    neo.neo_hmult(ctx, relin, dev(cta[None]), dev(ctb[None]), 2, out, 1, ctx.workspace(neo.NEO_OP_HMULT, 2, 1))
    res = torch.empty((1, 2, 2, prm.N), dtype=torch.uint64, device="cuda")
    neo.neo_rescale(ctx, out, 2, res, 1, ctx.workspace(neo.NEO_OP_RESCALE, 2, 1))
    got = host(res)[0]
    want = ckks.rescale(prm, ckks.hmult(prm, cta, ctb, 2, relin_np), 2)
    assert np.array_equal(got, want)
    m = ckks.crt_centered(prm, ckks.decrypt_residues(prm, got, s, 1), [0, 1])
    z = ckks.decode(prm.N, m, delta * delta / prm.q[2])
    assert np.max(np.abs(z - za * zb)) < 1e-6


def test_invalid_arguments_fail_loudly():
    ctx, prm = ctx_of("tiny")
    t = torch.zeros((1, 3, prm.N), dtype=torch.uint64, device="cuda")
    ws = torch.empty_like(t)
    with pytest.raises(neo.NeoError):
        neo.neo_ntt(ctx, t, [0, 1, 99], 1, ws)
    with pytest.raises(neo.NeoError):
        neo.neo_automorphism(ctx, t, 3, 4, t.clone(), 1)        # even Galois element
    evk = neo.EvalKey(ctx, dev(rand_evk(prm, 1)))
    with pytest.raises(neo.NeoError):
        neo.neo_keyswitch(ctx, evk, t, 5, t, t, 1, ws)          # level out of range
    with pytest.raises(neo.NeoError):
        neo.neo_keyswitch(ctx, evk, t[:, :3], 2, t.clone(), t.clone(), 1, ws)   # workspace too small


@pytest.mark.parametrize("name,level,batch,rs", [("tiny", 2, 2, (1, 2, 7)), ("setb", 35, 1, (1, 4))])
def test_hrot_hoisted(name, level, batch, rs):
    ctx, prm = ctx_of(name)
    gs = [pow(5, r, 2 * prm.N) for r in rs]
    keys_np = [rand_evk(prm, 950 + 10 * r) for r in rs]
    keys = [neo.EvalKey(ctx, dev(k), hoisted_galois=g) for k, g in zip(keys_np, gs)]
    ct = np.stack([rand_ct(prm, level, 970 + 2 * b) for b in range(batch)])
    out = torch.empty((len(rs), batch, 2, level + 1, prm.N), dtype=torch.uint64, device="cuda")
    ws = ctx.workspace(neo.NEO_OP_HROT_HOISTED, level, batch)
    neo.neo_hrot_hoisted(ctx, keys, dev(ct), level, out, batch, ws)
    got = host(out)
    for bb in range(batch):
        want = ckks.hrot_hoisted(prm, ct[bb], gs, level, keys_np)
        for r in range(len(rs)):
            assert np.array_equal(got[r, bb], want[r])


@pytest.mark.parametrize("name,level,batch", [("tiny", 2, 2), ("tiny", 1, 1), ("tiny3", 2, 3), ("setb", 35, 1),
                                              ("setb", 20, 2), ("setb", 1, 1)])
def test_hmult_rescale_fused(name, level, batch):
    """neo_hmult_rescale == Rescale(HMULT) of the oracle, bit for bit (the fused ModDown tail)."""
    ctx, prm = ctx_of(name)
    evk_np = rand_evk(prm, 1100)
    relin = neo.EvalKey(ctx, dev(evk_np))
    a = np.stack([rand_ct(prm, level, 1110 + 4 * b) for b in range(batch)])
    b_ = np.stack([rand_ct(prm, level, 1112 + 4 * b) for b in range(batch)])
    out = torch.empty((batch, 2, level, prm.N), dtype=torch.uint64, device="cuda")
    ws = ctx.workspace(neo.NEO_OP_HMULT_RESCALE, level, batch)
    neo.neo_hmult_rescale(ctx, relin, dev(a), dev(b_), level, out, batch, ws)
    got = host(out)
    for bb in range(batch):
        assert np.array_equal(got[bb], ckks.rescale(prm, ckks.hmult(prm, a[bb], b_[bb], level, evk_np), level))


def test_hmult_rescale_fused_rejects():
    ctx, prm = ctx_of("tiny")
    relin = neo.EvalKey(ctx, dev(rand_evk(prm, 1200)))
    ct = dev(rand_ct(prm, 2, 1210)[None])
    ws = ctx.workspace(neo.NEO_OP_HMULT_RESCALE, 2, 1)
    with pytest.raises(neo.NeoError):           # level 0 cannot be rescaled
        neo.neo_hmult_rescale(ctx, relin, ct[:, :, :1].contiguous(), ct[:, :, :1].contiguous(), 0,
                              torch.empty((1, 2, 1, prm.N), dtype=torch.uint64, device="cuda"), 1, ws)
    with pytest.raises(neo.NeoError):           # workspace too small
        neo.neo_hmult_rescale(ctx, relin, ct, ct, 2, torch.empty((1, 2, 2, prm.N), dtype=torch.uint64, device="cuda"),
                              1, ws[: ws.numel() // 2])


@pytest.mark.parametrize("op", ["hrot", "hmult_rescale", "keyswitch"])
def test_batch_larger_than_chunk(op):
    """Batches above the library's chunk (32 ciphertexts) run as several chunks alternating
    over two streams: every ciphertext still equals the oracle's; the workspace is two chunks'."""
    ctx, prm = ctx_of("tiny")
    level, batch = 2, 35
    evk_np = rand_evk(prm, 1300)
    key = neo.EvalKey(ctx, dev(evk_np))
    code = {"hrot": neo.NEO_OP_HROT, "hmult_rescale": neo.NEO_OP_HMULT_RESCALE, "keyswitch": neo.NEO_OP_KEYSWITCH}[op]
    assert ctx.workspace_size(code, level, batch) == 2 * ctx.workspace_size(code, level, 32)   # two chunks in flight
    ws = ctx.workspace(code, level, batch)
    a = np.stack([rand_ct(prm, level, 1310 + 4 * b) for b in range(batch)])
    g = pow(5, 3, 2 * prm.N)
    if op == "hrot":
        out = torch.empty((batch, 2, level + 1, prm.N), dtype=torch.uint64, device="cuda")
        neo.neo_hrot(ctx, key, g, dev(a), level, out, batch, ws)
        want = [ckks.hrot(prm, a[b], g, level, evk_np) for b in range(batch)]
    elif op == "hmult_rescale":
        b_ = np.stack([rand_ct(prm, level, 1312 + 4 * b) for b in range(batch)])
        out = torch.empty((batch, 2, level, prm.N), dtype=torch.uint64, device="cuda")
        neo.neo_hmult_rescale(ctx, key, dev(a), dev(b_), level, out, batch, ws)
        want = [ckks.rescale(prm, ckks.hmult(prm, a[b], b_[b], level, evk_np), level) for b in range(batch)]
    else:
        d = np.ascontiguousarray(a[:, 0])
        o0 = torch.empty((batch, level + 1, prm.N), dtype=torch.uint64, device="cuda")
        o1 = torch.empty_like(o0)
        neo.neo_keyswitch(ctx, key, dev(d), level, o0, o1, batch, ws)
        out = torch.stack([o0, o1], dim=1)
        want = [np.stack(ckks.keyswitch(prm, d[b], level, evk_np)) for b in range(batch)]
    got = host(out)
    for bb in range(batch):
        assert np.array_equal(got[bb], want[bb]), bb


@pytest.mark.parametrize("name,level,n", [("tiny", 2, 1), ("tiny3", 2, 3), ("setb", 35, 3), ("setb", 20, 2)])
def test_hrot_sum(name, level, n):
    """neo_hrot_sum (rotations summed with one ModDown) equals the oracle's hrot_sum bit for bit;
    with one term it is HROTATE itself."""
    from oracle import boot as oboot
    ctx, prm = ctx_of(name)
    gs = [pow(5, r, 2 * prm.N) for r in (1, 4, 9)[:n]]
    evks = [rand_evk(prm, 1400 + 10 * k) for k in range(n)]
    keys = [neo.EvalKey(ctx, dev(e)) for e in evks]
    cts = [rand_ct(prm, level, 1450 + 4 * k) for k in range(n)]
    out = torch.empty((1, 2, level + 1, prm.N), dtype=torch.uint64, device="cuda")
    ws = ctx.workspace(neo.NEO_OP_HROT_SUM, level, 1)
    neo.neo_hrot_sum(ctx, keys, gs, [dev(c[None]) for c in cts], level, out, 1, ws)
    got = host(out)[0]
    assert np.array_equal(got, oboot.hrot_sum(prm, cts, gs, level, evks))
    if n == 1:
        assert np.array_equal(got, ckks.hrot(prm, cts[0], gs[0], level, evks[0]))


def test_batch_chunks_setb_sampled():
    """Set-B HROTATE over 33 ciphertexts (chunks of 32 + 1 on two streams, the configuration
    bench.py's batch_hrot times): sampled ciphertexts from both chunks equal the oracle."""
    ctx, prm = ctx_of("setb")
    level, batch = 35, 33
    evk_np = rand_evk(prm, 1500)
    key = neo.EvalKey(ctx, dev(evk_np))
    g = pow(5, 1, 2 * prm.N)
    a = np.stack([rand_ct(prm, level, 1510 + 2 * b) for b in range(batch)])
    out = torch.empty((batch, 2, level + 1, prm.N), dtype=torch.uint64, device="cuda")
    neo.neo_hrot(ctx, key, g, dev(a), level, out, batch, ctx.workspace(neo.NEO_OP_HROT, level, batch))
    got = host(out)
    for bb in (0, 31, 32):
        assert np.array_equal(got[bb], ckks.hrot(prm, a[bb], g, level, evk_np)), bb


def test_pmult_acc_setb():
    """neo_pmult_acc at Set-B l = 35 (9 terms, the conv layer's inner sum) equals PMULT + HADD."""
    ctx, prm = ctx_of("setb")
    level, k = 35, 9
    cts = [rand_ct(prm, level, 1600 + 2 * i) for i in range(k)]
    pts = [rand_poly(prm, list(range(level + 1)), 1700 + i) for i in range(k)]
    out = torch.empty((1, 2, level + 1, prm.N), dtype=torch.uint64, device="cuda")
    neo.neo_pmult_acc(ctx, [dev(c[None]) for c in cts], [dev(p) for p in pts], level, out, 1, pt_shared=True)
    want = None
    for c, p in zip(cts, pts):
        t = ckks.pmult(prm, c, p, level)
        want = t if want is None else ckks.hadd(prm, want, t, level)
    assert np.array_equal(host(out)[0], want)


# The library's environment-selected variants are read once per process, so each runs the parity
# tests above in a fresh interpreter: NEO_TWO_STREAM=0 (hoisted rotations / giant-step sums on one
# stream) and NEO_KIP=1 (KeyIP fused into the ModUp NTT's row pass, opt-in).
@pytest.mark.parametrize("env,sel", [("NEO_TWO_STREAM=0", "hoisted or hrot_sum"),
                                     ("NEO_KIP=1", "keyswitch or hmult or hrot")])
def test_env_variants_bit_exact(env, sel):
    import os
    import subprocess
    import sys
    k, v = env.split("=")
    r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-m", "gpu", "-k",
                        f"({sel}) and not env_variants", __file__],
                       env=dict(os.environ, **{k: v}), capture_output=True, text=True, timeout=1200)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-2000:]
