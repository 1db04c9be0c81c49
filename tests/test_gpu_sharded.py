"""GPU: the limb-sharded key-switch (sharded.py + neo_keyip / neo_moddown_combine / neo_bconv /
neo_ntt through the C-ABI) against the oracle, with 1 rank and with 2 ranks sharing cuda:0
(gloo gathers staged through the host; on an 8-GPU box the same code gathers over NCCL)."""
import os
import socket
import sys

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(rank, world, port, cfg, level, q):
    try:
        _run_inner(rank, world, port, cfg, level, q)
    except Exception as e:                       # report instead of hanging the parent
        import traceback
        q.put((rank, "".join(traceback.format_exception(e))))


def _run_inner(rank, world, port, cfg, level, q):
    sys.path.insert(0, ROOT)
    import synth
    from oracle import ckks
    from paper_conf_isca_jiaodwfcm0z25_b200 import neo
    from paper_conf_isca_jiaodwfcm0z25_b200.sharded import NeoOps, ShardPlan, limb_sharded_keyswitch
    if world > 1:
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)
        prm = ckks.Params(*cfg)
        ctx = neo.Context(prm.log_n, prm.num_q, prm.num_p, prm.dnum)
        evk_np = np.stack([np.stack([synth.uniform_residues(40 + 2 * j + c, prm.moduli, prm.N) for c in range(2)])
                           for j in range(prm.dnum)])
        evk = neo.EvalKey(ctx, torch.from_numpy(evk_np).cuda())
        B = 2
        d = np.stack([synth.uniform_residues(60 + b, prm.q[: level + 1], prm.N) for b in range(B)])
        plan = ShardPlan(level, prm.num_q, prm.num_p, prm.alpha, world, rank)
        d_local = torch.from_numpy(np.ascontiguousarray(d[:, plan.my_q])).cuda()
        k0, k1 = limb_sharded_keyswitch(NeoOps(ctx), plan, d_local, evk)
        torch.cuda.synchronize()
        ok = True
        for b in range(B):
            r0, r1 = ckks.keyswitch(prm, d[b], level, evk_np)
            ok &= np.array_equal(k0.cpu().numpy()[b], r0[plan.my_q]) and np.array_equal(k1.cpu().numpy()[b], r1[plan.my_q])
        q.put((rank, bool(ok)))
    finally:
        if world > 1:
            dist.destroy_process_group()


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.mark.parametrize("world,cfg,level", [(1, (12, 3, 1, 3), 2), (2, (12, 6, 2, 3), 5), (2, (16, 36, 12, 3), 35)])
def test_limb_sharded_keyswitch(world, cfg, level):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=_run, args=(r, world, port, cfg, level, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=240) for _ in procs)
    for p in procs:
        p.join(timeout=60)
    assert all(res[r] is True for r in range(world)), res
