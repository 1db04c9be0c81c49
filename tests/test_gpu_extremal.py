"""GPU parity at Set-B on inputs that drive the lazy-reduction bounds to their extremes.

The kernels keep residues lazy between steps (FP64 |x| < 2^45 in the NTT passes, the BConv
epilogue's V < 2^51, the tensor-core NTT's byte planes, 128-bit KeyIP accumulation); uniform
random residues rarely reach those bounds, so every stage is also checked, element by element
against the oracle, on all-(q-1), all-zero, alternating 0 / q-1 and single-spike inputs (the
NTT/INTT themselves: tests/test_gpu_ntt_impl.py).  Keys are all-(q-1) for the KeyIP products
(the largest 36x36-bit product sums a KeyIP can see)."""
import numpy as np
import pytest
import torch

from oracle import ckks

pytestmark = pytest.mark.gpu

neo = pytest.importorskip("paper_conf_isca_jiaodwfcm0z25_b200.neo")

KINDS = ["qm1", "zeros", "alt", "spike"]
_C = {}


def setb():
    if "ctx" not in _C:
        prm = ckks.set_b()
        _C["prm"] = prm
        _C["ctx"] = neo.Context(prm.log_n, prm.num_q, prm.num_p, prm.dnum)
    return _C["ctx"], _C["prm"]


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.uint64)).cuda()


def host(t):
    torch.cuda.synchronize()
    return t.cpu().numpy()


def extremal(prm, ids, kind, phase=0):
    q = np.array([prm.moduli[i] for i in ids], dtype=np.uint64)[:, None]
    x = np.zeros((len(ids), prm.N), dtype=np.uint64)
    if kind == "qm1":
        x[:] = q - np.uint64(1)
    elif kind == "alt":
        x[:, (1 + phase) % 2::2] = (q - np.uint64(1))
    elif kind == "spike":
        x[:, (prm.N - 1 - phase) % prm.N] = (q - np.uint64(1))[:, 0]
    return x


def ct_of(prm, level, kind, phase=0):
    ids = list(range(level + 1))
    return np.stack([extremal(prm, ids, kind, phase), extremal(prm, ids, kind, phase + 1)])


def key_qm1(prm):
    ids = list(range(prm.num_q + prm.num_p))
    one = extremal(prm, ids, "qm1")
    return np.stack([np.stack([one, one]) for _ in range(prm.dnum)])


@pytest.mark.parametrize("kind", KINDS)
@pytest.mark.parametrize("src,dst", [(list(range(12)), list(range(12, 48))),     # ModUp digit 0
                                     (list(range(36, 48)), list(range(36)))])    # ModDown
def test_bconv_extremal(kind, src, dst):
    ctx, prm = setb()
    x = extremal(prm, src, kind)
    out = torch.empty((1, len(dst), prm.N), dtype=torch.uint64, device="cuda")
    neo.neo_bconv(ctx, dev(x[None]), src, out, dst, 1)
    assert np.array_equal(host(out)[0], ckks.bconv(prm, x, src, dst))


@pytest.mark.parametrize("kind", KINDS)
def test_tensor_extremal(kind):
    ctx, prm = setb()
    level = 35
    a, b = ct_of(prm, level, kind), ct_of(prm, level, kind, 1)
    d = torch.empty((1, 3, level + 1, prm.N), dtype=torch.uint64, device="cuda")
    neo.neo_tensor(ctx, dev(a[None]), dev(b[None]), level, d, 1)
    got, want = host(d)[0], ckks.tensor(prm, a, b, level)
    for k in range(3):
        assert np.array_equal(got[k], want[k])


@pytest.mark.parametrize("kind", ["qm1", "alt", "spike"])
def test_keyswitch_extremal_input_and_key(kind):
    """KeyIP at its largest products (input and key all q-1 or patterned), the BConv and NTT
    stages of the same key-switch on extremal coefficient data."""
    ctx, prm = setb()
    level = 35
    evk_np = key_qm1(prm)
    key = neo.EvalKey(ctx, dev(evk_np))
    d = extremal(prm, list(range(level + 1)), kind)
    o0 = torch.empty((1, level + 1, prm.N), dtype=torch.uint64, device="cuda")
    o1 = torch.empty_like(o0)
    neo.neo_keyswitch(ctx, key, dev(d[None]), level, o0, o1, 1, ctx.workspace(neo.NEO_OP_KEYSWITCH, level, 1))
    k0, k1 = ckks.keyswitch(prm, d, level, evk_np)
    assert np.array_equal(host(o0)[0], k0)
    assert np.array_equal(host(o1)[0], k1)


@pytest.mark.parametrize("kind", KINDS)
def test_rescale_extremal(kind):
    ctx, prm = setb()
    level = 35
    ct = ct_of(prm, level, kind)
    out = torch.empty((1, 2, level, prm.N), dtype=torch.uint64, device="cuda")
    neo.neo_rescale(ctx, dev(ct[None]), level, out, 1, ctx.workspace(neo.NEO_OP_RESCALE, level, 1))
    assert np.array_equal(host(out)[0], ckks.rescale(prm, ct, level))


@pytest.mark.parametrize("kind", ["qm1", "alt"])
def test_hmult_rescale_extremal(kind):
    """The fused HMULT + Rescale (fold kernel, ModDown tail with q_l^-1) on extremal
    ciphertexts and an all-(q-1) relinearisation key."""
    ctx, prm = setb()
    level = 35
    evk_np = key_qm1(prm)
    key = neo.EvalKey(ctx, dev(evk_np))
    a, b = ct_of(prm, level, kind), ct_of(prm, level, kind, 1)
    out = torch.empty((1, 2, level, prm.N), dtype=torch.uint64, device="cuda")
    neo.neo_hmult_rescale(ctx, key, dev(a[None]), dev(b[None]), level, out, 1,
                          ctx.workspace(neo.NEO_OP_HMULT_RESCALE, level, 1))
    want = ckks.rescale(prm, ckks.hmult(prm, a, b, level, evk_np), level)
    assert np.array_equal(host(out)[0], want)
