"""GPU parity of the ops without key-switching (PMULT, HADD, PADD: L133-135) and of Double
Rescale (L138, L151) through the C-ABI against the CPU oracle, bit-exact on every residue."""
import numpy as np
import pytest
import torch

import synth
from oracle import ckks

pytestmark = pytest.mark.gpu

neo = pytest.importorskip("paper_conf_isca_jiaodwfcm0z25_b200.neo")

_CTX = {}


def ctx_of(name):
    if name not in _CTX:
        prm = {"tiny": ckks.tiny, "tiny3": ckks.tiny_dnum3, "setb": ckks.set_b}[name]()
        _CTX[name] = (neo.Context(prm.log_n, prm.num_q, prm.num_p, prm.dnum), prm)
    return _CTX[name]


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.uint64)).cuda()


def host(t):
    torch.cuda.synchronize()
    return t.cpu().numpy()


def rand_ct(prm, level, seed):
    ids = list(range(level + 1))
    return np.stack([synth.uniform_residues(seed + c, [prm.moduli[i] for i in ids], prm.N) for c in range(2)])


@pytest.mark.parametrize("name,level,batch", [("tiny", 2, 3), ("tiny", 0, 1), ("setb", 35, 2), ("setb", 20, 1)])
@pytest.mark.parametrize("op", ["pmult", "hadd", "padd"])
def test_elementwise(op, name, level, batch):
    ctx, prm = ctx_of(name)
    a = np.stack([rand_ct(prm, level, 500 + 3 * b) for b in range(batch)])
    if op == "hadd":
        b_ = np.stack([rand_ct(prm, level, 700 + 3 * b) for b in range(batch)])
    else:
        b_ = np.stack([rand_ct(prm, level, 700 + 3 * b)[0] for b in range(batch)])      # plaintexts
    out = torch.empty(a.shape, dtype=torch.uint64, device="cuda")
    getattr(neo, "neo_" + op)(ctx, dev(a), dev(b_), level, out, batch)
    got = host(out)
    fn = getattr(ckks, op)
    for bb in range(batch):
        assert np.array_equal(got[bb], fn(prm, a[bb], b_[bb], level))


@pytest.mark.parametrize("name,level,batch", [("tiny", 2, 2), ("setb", 35, 1), ("setb", 13, 2), ("setb", 2, 1)])
def test_double_rescale(name, level, batch):
    ctx, prm = ctx_of(name)
    ct = np.stack([rand_ct(prm, level, 1100 + 2 * b) for b in range(batch)])
    out = torch.empty((batch, 2, level - 1, prm.N), dtype=torch.uint64, device="cuda")
    ws = ctx.workspace(neo.NEO_OP_DOUBLE_RESCALE, level, batch)
    neo.neo_double_rescale(ctx, dev(ct), level, out, batch, ws)
    got = host(out)
    for bb in range(batch):
        assert np.array_equal(got[bb], ckks.double_rescale(prm, ct[bb], level))


def test_double_rescale_rejects_low_level():
    ctx, prm = ctx_of("tiny")
    t = torch.zeros((1, 2, 2, prm.N), dtype=torch.uint64, device="cuda")
    with pytest.raises(neo.NeoError):
        neo.neo_double_rescale(ctx, t, 1, t.clone(), 1, torch.empty(8 * prm.N, dtype=torch.uint64, device="cuda"))
