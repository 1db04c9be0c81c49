"""GPU parity of the native limb-sharded key-switch (neo_keyswitch_sharded):
every rank's output rows are compared element by element with the oracle's single-device
key-switch (bit-exact).  One rank runs through neo_comm_create (no NCCL needed); several ranks
share the one GPU through neo_comm_create_local, one host thread per rank calling the library
concurrently (the exchanges are device-to-device copies after a host barrier, the same data
flow NCCL's all-gather gives across GPUs)."""
import threading

import numpy as np
import pytest
import torch

import synth
from oracle import ckks

pytestmark = pytest.mark.gpu

neo = pytest.importorskip("paper_conf_isca_jiaodwfcm0z25_b200.neo")

_C = {}


def setup(name):
    if name not in _C:
        prm = {"tiny3": ckks.tiny_dnum3, "setb": ckks.set_b}[name]()
        ctx = neo.Context(prm.log_n, prm.num_q, prm.num_p, prm.dnum)
        ids = list(range(prm.num_q + prm.num_p))
        evk_np = np.stack([np.stack([synth.uniform_residues(900 + 2 * j + c, [prm.moduli[i] for i in ids], prm.N)
                                     for c in range(2)]) for j in range(prm.dnum)])
        key = neo.EvalKey(ctx, torch.from_numpy(evk_np).cuda())
        _C[name] = (prm, ctx, evk_np, key)
    return _C[name]


def run_ranks(ctx, comms, key, d, level, batch):
    """Every rank's share of one key-switch, the ranks on concurrent host threads."""
    outs, errs = {}, []
    bufs = []
    for cm in comms:
        q_ids, _ = cm.limbs(level)
        dl = torch.from_numpy(np.ascontiguousarray(d[:, q_ids])).cuda() if q_ids else None
        o0 = torch.empty((batch, len(q_ids), d.shape[-1]), dtype=torch.uint64, device="cuda") if q_ids else None
        o1 = torch.empty_like(o0) if q_ids else None
        bufs.append((q_ids, dl, o0, o1, cm.workspace(level, batch), torch.cuda.Stream()))
    torch.cuda.synchronize()

    def work(r):
        try:
            q_ids, dl, o0, o1, ws, st = bufs[r]
            neo.neo_keyswitch_sharded(ctx, comms[r], key, dl, level, o0, o1, batch, ws, stream=st)
        except Exception as e:          # noqa: BLE001 -- reported by the main thread
            errs.append(e)

    ths = [threading.Thread(target=work, args=(r,)) for r in range(len(comms))]
    for t in ths:
        t.start()
    for t in ths:
        t.join()
    torch.cuda.synchronize()
    assert not errs, errs
    for r, (q_ids, dl, o0, o1, ws, st) in enumerate(bufs):
        outs[r] = (q_ids, o0.cpu().numpy() if o0 is not None else None, o1.cpu().numpy() if o1 is not None else None)
    return outs


def check(prm, evk_np, d, level, outs):
    seen = []
    for b in range(d.shape[0]):
        k0, k1 = ckks.keyswitch(prm, d[b], level, evk_np)
        for r, (q_ids, g0, g1) in outs.items():
            if q_ids:
                assert np.array_equal(g0[b], k0[q_ids]), (r, b)
                assert np.array_equal(g1[b], k1[q_ids]), (r, b)
                seen += q_ids if b == 0 else []
    assert sorted(seen) == list(range(level + 1))       # the ranks cover every Q limb once


@pytest.mark.timeout(600)
@pytest.mark.parametrize("name,level,batch", [("tiny3", 2, 2), ("setb", 35, 1), ("setb", 13, 2), ("setb", 0, 1)])
def test_one_rank(name, level, batch):
    prm, ctx, evk_np, key = setup(name)
    cm = neo.Comm.create(ctx, bytes(128), 1, 0)
    d = np.stack([synth.uniform_residues(950 + b, prm.q[: level + 1], prm.N) for b in range(batch)])
    check(prm, evk_np, d, level, run_ranks(ctx, [cm], key, d, level, batch))


@pytest.mark.timeout(600)
@pytest.mark.parametrize("name,world,level,batch", [
    ("tiny3", 2, 2, 2), ("tiny3", 3, 1, 1),          # 3 ranks at level 1: rank 2 owns P limbs only
    ("setb", 2, 35, 1), ("setb", 3, 20, 2), ("setb", 4, 35, 1),
])
def test_local_group(name, world, level, batch):
    prm, ctx, evk_np, key = setup(name)
    comms = neo.Comm.create_local(ctx, world)
    d = np.stack([synth.uniform_residues(960 + b, prm.q[: level + 1], prm.N) for b in range(batch)])
    check(prm, evk_np, d, level, run_ranks(ctx, comms, key, d, level, batch))


def test_ownership_and_errors():
    prm, ctx, evk_np, key = setup("tiny3")
    comms = neo.Comm.create_local(ctx, 2)
    assert comms[0].limbs(2) == ([0, 2], [3]) and comms[1].limbs(2) == ([1], [])
    with pytest.raises(neo.NeoError):
        comms[0].limbs(7)
    assert len(neo.Comm.unique_id()) == 128                    # NCCL is loadable (dlopen)
    with pytest.raises(neo.NeoError):                          # batch > 32
        neo.neo_keyswitch_sharded(ctx, comms[0], key, None, 2, None, None, 33, comms[0].workspace(2, 1))
