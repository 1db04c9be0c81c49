"""Multi-process (gloo, CPU) tests of the multi-GPU host logic:
data-parallel slicing / max-over-ranks, and the limb-sharded key-switch orchestration with
two all-gathers, run with a test-only oracle backend and compared against the single-process
oracle key-switch bit for bit."""
import os
import socket
import sys

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

from paper_conf_isca_jiaodwfcm0z25_b200.sharded import ShardPlan, dp_slice, limb_blocks  # noqa: E402


def test_dp_slice_and_blocks():
    for total in (1, 7, 256):
        for world in (1, 2, 3, 8):
            covered = []
            for r in range(world):
                s, n = dp_slice(total, world, r)
                covered += list(range(s, s + n))
            assert covered == list(range(total))
    assert limb_blocks(list(range(5)), 2) == [[0, 1, 2], [3, 4]]
    p = ShardPlan(35, 36, 12, 12, 8, 3)
    assert p.my_q == list(range(15, 20)) and p.my_p == [42, 43] and p.beta == 3


class OracleOps:
    """TEST-ONLY backend: the oracle's arithmetic on numpy arrays, gloo all-gathers."""

    def __init__(self, prm):
        from oracle import ckks
        self.c, self.prm = ckks, prm

    take = staticmethod(lambda x, idx: np.ascontiguousarray(x[:, idx]))
    take2 = staticmethod(lambda x, idx: np.ascontiguousarray(x[:, :, idx]))
    cat = staticmethod(lambda xs, axis: np.concatenate(xs, axis=axis))
    stack = staticmethod(lambda xs, axis: np.stack(xs, axis=axis))
    component = staticmethod(lambda x, c: np.ascontiguousarray(x[:, c]))
    empty2 = staticmethod(lambda like, n: np.zeros((like.shape[0], 2, n, like.shape[-1]), dtype=np.uint64))

    def _gather(self, x, sizes, axis):
        if len(sizes) == 1:
            return x
        m = max(sizes)
        shape = list(x.shape)
        shape[axis] = m
        pad = np.zeros(shape, dtype=np.uint64)
        sl = [slice(None)] * len(shape)
        sl[axis] = slice(0, x.shape[axis])
        pad[tuple(sl)] = x
        t = torch.from_numpy(pad.view(np.int64))
        parts = [torch.empty_like(t) for _ in sizes]
        dist.all_gather(parts, t)
        outs = []
        for p, n in zip(parts, sizes):
            a = p.numpy().view(np.uint64)
            sl[axis] = slice(0, n)
            outs.append(a[tuple(sl)])
        return np.ascontiguousarray(np.concatenate(outs, axis=axis))

    def allgather(self, x, sizes):
        return self._gather(x, sizes, 1)

    def allgather2(self, x, sizes):
        return self._gather(x, sizes, 2)

    def intt(self, x, ids):
        return np.stack([self.c.intt(self.prm, x[b], ids) for b in range(x.shape[0])])

    def ntt(self, x, ids):
        return np.stack([self.c.ntt(self.prm, x[b], ids) for b in range(x.shape[0])])

    def intt2(self, x, ids):
        return self.intt(x.reshape(-1, len(ids), x.shape[-1]), ids).reshape(x.shape)

    def ntt2(self, x, ids):
        return self.ntt(x.reshape(-1, len(ids), x.shape[-1]), ids).reshape(x.shape)

    def bconv(self, x, src, dst):
        return np.stack([self.c.bconv(self.prm, x[b], src, dst) for b in range(x.shape[0])])

    def bconv2(self, x, src, dst):
        B = x.shape[0]
        return self.bconv(x.reshape(2 * B, len(src), -1), src, dst).reshape(B, 2, len(dst), -1)

    def keyip(self, dhat, ids, beta, evk):
        B, N = dhat.shape[0], dhat.shape[-1]
        acc = np.zeros((B, 2, len(ids), N), dtype=np.uint64)
        for b in range(B):
            for c in range(2):
                for j in range(beta):
                    prod = self.c.mul(self.prm, dhat[b, j], evk[j, c][ids], ids)
                    acc[b, c] = self.c.add(self.prm, acc[b, c], prod, ids)
        return acc

    def moddown_combine(self, acc, conv, q_ids):
        pinv = [pow(self.prm.P % self.prm.moduli[i], -1, self.prm.moduli[i]) for i in q_ids]
        out = np.empty_like(acc)
        for b in range(acc.shape[0]):
            for c in range(2):
                out[b, c] = self.c.scalar_mul(self.prm, self.c.sub(self.prm, acc[b, c], conv[b, c], q_ids), pinv, q_ids)
        return out


def _worker(rank, world, port, cfg, level, q, strided=False):
    sys.path.insert(0, ROOT)
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import synth
        from oracle import ckks
        from paper_conf_isca_jiaodwfcm0z25_b200.sharded import ShardPlan, limb_sharded_keyswitch, max_over_ranks
        prm = ckks.Params(*cfg)
        ids = list(range(prm.num_q + prm.num_p))
        evk = np.stack([np.stack([synth.uniform_residues(40 + 2 * j + c, prm.moduli, prm.N) for c in range(2)])
                        for j in range(prm.dnum)])
        B = 2
        d = np.stack([synth.uniform_residues(60 + b, prm.q[: level + 1], prm.N) for b in range(B)])
        plan = ShardPlan(level, prm.num_q, prm.num_p, prm.alpha, world, rank, strided=strided)
        ops = OracleOps(prm)
        k0, k1 = limb_sharded_keyswitch(ops, plan, np.ascontiguousarray(d[:, plan.my_q]), evk)
        ok = k0.shape == (B, len(plan.my_q), prm.N) and k1.shape == k0.shape
        for b in range(B):
            r0, r1 = ckks.keyswitch(prm, d[b], level, evk)
            ok &= np.array_equal(k0[b], r0[plan.my_q]) and np.array_equal(k1[b], r1[plan.my_q])
        m = max_over_ranks(float(rank))
        ok &= m == float(world - 1)
        q.put((rank, bool(ok)))
    finally:
        dist.destroy_process_group()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.mark.parametrize("world,cfg,level,strided", [
    (2, (10, 6, 2, 3), 5, False),      # N=2^10, 6 Q + 2 P, dnum 3: both ranks own Q and P limbs
    (3, (10, 6, 2, 3), 4, False),      # rank 2 owns no P limb; partial last digit
    (2, (10, 3, 1, 1), 2, False),      # dnum = 1 (one digit spans both ranks)
    (2, (10, 6, 2, 3), 4, True),       # round-robin ownership (the sharded evaluator's plan)
    (3, (10, 6, 2, 3), 5, True),
    (3, (10, 6, 3, 3), 1, False),      # world > level + 1: rank 2 owns no Q limb, only P limbs
    (4, (10, 6, 4, 3), 1, True),       # round-robin, ranks 2 and 3 own P limbs only
])
def test_limb_sharded_keyswitch_gloo(world, cfg, level, strided):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, cfg, level, q, strided)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=300) for _ in procs)
    for p in procs:
        p.join(timeout=60)
    assert all(res[r] for r in range(world)), res
