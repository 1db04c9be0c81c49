"""GPU parity of both NTT implementations (neo_ntt_select): the tcgen05 form (both radix-16
DFT stages of every 256-point pass as int8 tensor-core GEMMs, Neo's matrix-multiplication NTT,
PAPER L438-450 / Fig. 9) and the FP64 CUDA-core butterflies.  Every transform is compared
element by element with the oracle (bit-exact: exact modular arithmetic),
on uniform residues and on inputs that drive the lazy-reduction bounds to their extremes
(all q-1, zeros, alternating 0 / q-1, a single spike), and inside the key-switching
operations that use every fused variant (lazy BConv input, per-row ModUp scale, the Galois
read of HROTATE, the ModDown tail, the fused Rescale)."""
import numpy as np
import pytest
import torch

import synth
from oracle import ckks

pytestmark = pytest.mark.gpu

neo = pytest.importorskip("paper_conf_isca_jiaodwfcm0z25_b200.neo")

IMPLS = {"tc": 1, "fp64": 0}
_C = {}


def setb(impl):
    if impl not in _C:
        prm = _C.get("prm") or ckks.set_b()
        _C["prm"] = prm
        ctx = neo.Context(prm.log_n, prm.num_q, prm.num_p, prm.dnum)
        ctx.ntt_select(IMPLS[impl])
        assert ctx.ntt_impl == IMPLS[impl]
        _C[impl] = ctx
    return _C[impl], _C["prm"]


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.uint64)).cuda()


def host(t):
    torch.cuda.synchronize()
    return t.cpu().numpy()


def rand_poly(prm, ids, seed):
    return synth.uniform_residues(seed, [prm.moduli[i] for i in ids], prm.N)


def extremal(prm, ids, kind):
    q = np.array([prm.moduli[i] for i in ids], dtype=np.uint64)[:, None]
    N = prm.N
    if kind == "zeros":
        return np.zeros((len(ids), N), dtype=np.uint64)
    if kind == "qm1":
        return np.broadcast_to(q - np.uint64(1), (len(ids), N)).copy()
    if kind == "alt":
        x = np.zeros((len(ids), N), dtype=np.uint64)
        x[:, 1::2] = (q - np.uint64(1))
        return x
    if kind == "spike":
        x = np.zeros((len(ids), N), dtype=np.uint64)
        x[:, N - 1] = (q - np.uint64(1))[:, 0]
        x[:, 0] = np.uint64(1)
        return x
    raise ValueError(kind)


@pytest.mark.parametrize("impl", ["tc", "fp64"])
def test_ntt_intt_setb_all_limbs_batch2(impl):
    ctx, prm = setb(impl)
    ids = list(range(prm.num_q + prm.num_p))
    x = np.stack([rand_poly(prm, ids, 900 + b) for b in range(2)])
    t = dev(x)
    ws = torch.empty(t.numel(), dtype=torch.uint64, device="cuda")
    neo.neo_ntt(ctx, t, ids, 2, ws)
    got = host(t)
    for b in range(2):
        assert np.array_equal(got[b], ckks.ntt(prm, x[b], ids))
    neo.neo_intt(ctx, t, ids, 2, ws)
    assert np.array_equal(host(t), x)


@pytest.mark.parametrize("impl", ["tc", "fp64"])
@pytest.mark.parametrize("kind", ["zeros", "qm1", "alt", "spike"])
def test_ntt_intt_setb_extremal(impl, kind):
    ctx, prm = setb(impl)
    ids = [0, 11, 35, 36, 47, 20]
    x = extremal(prm, ids, kind)
    t = dev(x[None])
    ws = torch.empty(t.numel(), dtype=torch.uint64, device="cuda")
    neo.neo_ntt(ctx, t, ids, 1, ws)
    fwd = host(t)[0]
    assert np.array_equal(fwd, ckks.ntt(prm, x, ids))
    neo.neo_intt(ctx, t, ids, 1, ws)
    assert np.array_equal(host(t)[0], x)
    # the inverse of an extremal NTT-domain input as well
    t2 = dev(x[None])
    neo.neo_intt(ctx, t2, ids, 1, ws)
    assert np.array_equal(host(t2)[0], ckks.intt(prm, x, ids))


def test_impls_agree_on_many_limbs():
    """108 limb rows in one launch (the ModUp NTT shape), ragged limb ids, both directions."""
    ctx_t, prm = setb("tc")
    ctx_f, _ = setb("fp64")
    ids = [(7 * i + 3) % 48 for i in range(108)]
    x = rand_poly(prm, ids, 1234)[None]
    a, b = dev(x), dev(x)
    ws = torch.empty(a.numel(), dtype=torch.uint64, device="cuda")
    neo.neo_ntt(ctx_t, a, ids, 1, ws)
    neo.neo_ntt(ctx_f, b, ids, 1, ws)
    assert torch.equal(a, b)
    sample = [0, 57, 107]
    want = ckks.ntt(prm, x[0][sample], [ids[i] for i in sample])
    assert np.array_equal(host(a)[0][sample], want)
    neo.neo_intt(ctx_t, a, ids, 1, ws)
    assert np.array_equal(host(a), x)


def rand_ct(prm, level, seed):
    ids = list(range(level + 1))
    return np.stack([rand_poly(prm, ids, seed), rand_poly(prm, ids, seed + 1)])


def rand_evk(prm, seed):
    ids = list(range(prm.num_q + prm.num_p))
    return np.stack([np.stack([rand_poly(prm, ids, seed + 2 * j + c) for c in range(2)])
                     for j in range(prm.dnum)])


_EVK = {}


def evk_of(impl):
    ctx, prm = setb(impl)
    if "np" not in _EVK:
        _EVK["np"] = rand_evk(prm, 4100)
    if impl not in _EVK:
        _EVK[impl] = neo.EvalKey(ctx, dev(_EVK["np"]))
    return _EVK[impl], _EVK["np"]


@pytest.mark.parametrize("impl", ["tc", "fp64"])
def test_hrot_and_hmult_rescale_setb(impl):
    """HROTATE (Galois read fused into the INTT row pass, ModDown tail with sigma(c0)) and the
    fused HMULT + Rescale (ModDown tail with the q_l^-1 post-multiply) at Set-B l = 35."""
    ctx, prm = setb(impl)
    key, evk_np = evk_of(impl)
    level = 35
    a, b = rand_ct(prm, level, 4200), rand_ct(prm, level, 4202)
    rot = torch.empty((1, 2, level + 1, prm.N), dtype=torch.uint64, device="cuda")
    neo.neo_hrot(ctx, key, 5, dev(a[None]), level, rot, 1, ctx.workspace(neo.NEO_OP_HROT, level, 1))
    hmr = torch.empty((1, 2, level, prm.N), dtype=torch.uint64, device="cuda")
    neo.neo_hmult_rescale(ctx, key, dev(a[None]), dev(b[None]), level, hmr, 1,
                          ctx.workspace(neo.NEO_OP_HMULT_RESCALE, level, 1))
    assert np.array_equal(host(rot)[0], ckks.hrot(prm, a, 5, level, evk_np))
    want = ckks.rescale(prm, ckks.hmult(prm, a, b, level, evk_np), level)
    assert np.array_equal(host(hmr)[0], want)


@pytest.mark.parametrize("impl", ["tc", "fp64"])
def test_keyswitch_setb_partial_digit_batch2(impl):
    ctx, prm = setb(impl)
    key, evk_np = evk_of(impl)
    level = 20
    d = np.stack([rand_poly(prm, list(range(level + 1)), 4300 + b) for b in range(2)])
    o0 = torch.empty((2, level + 1, prm.N), dtype=torch.uint64, device="cuda")
    o1 = torch.empty_like(o0)
    neo.neo_keyswitch(ctx, key, dev(d), level, o0, o1, 2, ctx.workspace(neo.NEO_OP_KEYSWITCH, level, 2))
    g0, g1 = host(o0), host(o1)
    for b in range(2):
        k0, k1 = ckks.keyswitch(prm, d[b], level, evk_np)
        assert np.array_equal(g0[b], k0) and np.array_equal(g1[b], k1)


def test_select_rejects():
    ctx, _ = setb("tc")
    with pytest.raises(neo.NeoError):
        ctx.ntt_select(7)
    prm = ckks.tiny()
    small = neo.Context(prm.log_n, prm.num_q, prm.num_p, prm.dnum)
    assert small.ntt_impl == 0                      # N = 2^12: FP64 only
    with pytest.raises(neo.NeoError):
        small.ntt_select(1)
