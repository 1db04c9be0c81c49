"""Multi-GPU key-switching: one process per GPU, torch.distributed plumbing.

* Data parallel (independent ciphertexts, P1): `dp_slice` partitions a batch; every rank
  runs the single-GPU C-ABI path on its slice and no collective touches the data.
  bench.py uses this for `--gpus N` (weak scaling).
* Limb-sharded key-switch (P2): one key-switch at level l is split by RNS limb.  Each rank
  owns a contiguous block of the Q limbs and of the P limbs of PQ_l.  NTT, KeyIP and the
  ModDown tail are limb-local; only BConv needs other limbs, so the path has exactly two
  exchange steps, both all-gathers of coefficient-form limbs:
      INTT(own Q) -> ALL-GATHER Q -> ModUp BConv (own targets) -> NTT -> KeyIP (own limbs)
      -> INTT(own P) -> ALL-GATHER P -> ModDown BConv (own Q) -> NTT -> (acc - conv) P^-1
  (Table 2, Fig. 5).  The output stays sharded by Q limb.

The orchestration below is host logic only.  Every arithmetic step goes through an `ops`
backend: `NeoOps` runs the CUDA library through its C-ABI on the rank's GPU and gathers
over NCCL.  The CPU tests run the same orchestration with a test-only backend built on the
oracle over gloo (tests/test_dist_gloo.py).
"""
from __future__ import annotations

import torch
import torch.distributed as dist


def dp_slice(total: int, world: int, rank: int) -> tuple[int, int]:
    """Contiguous, balanced slice [start, start+count) of `total` items for `rank`."""
    base, extra = divmod(total, world)
    start = rank * base + min(rank, extra)
    return start, base + (1 if rank < extra else 0)


def limb_blocks(ids: list[int], world: int) -> list[list[int]]:
    """Split a limb-id list into `world` contiguous, balanced blocks (some may be empty)."""
    out = []
    for r in range(world):
        s, n = dp_slice(len(ids), world, r)
        out.append(ids[s:s + n])
    return out


def max_over_ranks(value: float, group=None) -> float:
    """Max of a host float over all ranks (timing is reported as the slowest rank)."""
    if not dist.is_available() or not dist.is_initialized() or dist.get_world_size(group) == 1:
        return float(value)
    backend = dist.get_backend(group)
    dev = torch.device("cuda", torch.cuda.current_device()) if backend == "nccl" else torch.device("cpu")
    t = torch.tensor([float(value)], dtype=torch.float64, device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
    return float(t.item())


def strided_blocks(ids: list[int], world: int) -> list[list[int]]:
    """Round-robin ownership: position k goes to rank k mod world (level drops stay balanced)."""
    return [ids[r::world] for r in range(world)]


class ShardPlan:
    """Limb ownership for a key-switch at `level` (digits of Z8: D_j = [j alpha, ...)).
    strided=False: contiguous blocks; strided=True: round-robin (the limb-sharded evaluator,
    whose ciphertexts lose their top limb at every Rescale)."""

    def __init__(self, level: int, num_q: int, num_p: int, alpha: int, world: int, rank: int,
                 strided: bool = False):
        self.level, self.num_q, self.num_p, self.alpha = level, num_q, num_p, alpha
        self.world, self.rank = world, rank
        self.q_ids = list(range(level + 1))
        self.p_ids = list(range(num_q, num_q + num_p))
        split = strided_blocks if strided else limb_blocks
        self.q_blocks = split(self.q_ids, world)
        self.p_blocks = split(self.p_ids, world)
        # the all-gathers concatenate the blocks rank by rank: positions of the natural order
        cq = [i for b in self.q_blocks for i in b]
        cp = [i for b in self.p_blocks for i in b]
        self.q_perm = None if cq == self.q_ids else [cq.index(i) for i in self.q_ids]
        self.p_perm = None if cp == self.p_ids else [cp.index(i) for i in self.p_ids]
        self.my_q = self.q_blocks[rank]
        self.my_p = self.p_blocks[rank]
        self.mine = self.my_q + self.my_p                 # this rank's limbs of PQ_l
        beta = -(-(level + 1) // alpha)
        self.digits = [list(range(j * alpha, min((j + 1) * alpha, level + 1))) for j in range(beta)]
        self.beta = beta


def limb_sharded_keyswitch(ops, plan: ShardPlan, d_local, evk):
    """One key-switch of the rank's Q limbs `d_local` [B][len(my_q)][N] (NTT form).

    Returns (k0, k1) restricted to this rank's Q limbs, each [B][len(my_q)][N].
    """
    return limb_sharded_moddown(ops, plan, limb_sharded_keyip(ops, plan, d_local, evk))


def limb_sharded_keyip(ops, plan: ShardPlan, d_local, evk):
    """Steps a3-a6 (INTT, exchange #1, ModUp, NTT, KeyIP): the rank's rows of the KeyIP output
    acc [B][2][len(plan.mine)][N] (PQ_l, NTT form)."""
    P = plan
    # a3: INTT of the rank's Q limbs, then exchange #1: every rank gets all Q limbs.  A rank
    # that owns no Q limb (world > level + 1) still joins both exchanges: it owns P limbs the
    # other ranks' ModDown needs, and returns empty outputs.
    y_local = ops.intt(d_local, P.my_q) if P.my_q else d_local
    y_all = ops.allgather(y_local, [len(b) for b in P.q_blocks])          # [B][l+1][N]
    if P.q_perm is not None:
        y_all = ops.take(y_all, P.q_perm)
    # a4/a5: ModUp of every digit onto this rank's own target limbs, then NTT
    dhat_rows = []                                                          # per digit: [B][n_mine][N]
    for dj in P.digits:
        targets = [t for t in P.mine if t not in dj]
        up = ops.ntt(ops.bconv(ops.take(y_all, dj), dj, targets), targets) if targets else None
        # rows of d_hat_j in P.mine order: the digit's own limbs are d_t itself, the rest ModUp's
        # outputs -- one concatenation and one row selection (not one copy per limb)
        n_d = len(P.my_q)
        idx = [P.my_q.index(t) if t in dj else n_d + targets.index(t) for t in P.mine]
        both = ops.cat([d_local, up], axis=1) if up is not None else d_local
        dhat_rows.append(ops.take(both, idx))
    return ops.keyip(ops.stack(dhat_rows, axis=1), P.mine, P.beta, evk)     # a6 -> [B][2][n_mine][N]


def limb_sharded_moddown(ops, plan: ShardPlan, acc):
    """Steps a7-a10 (INTT of P, exchange #2, ModDown BConv, NTT, combine) of a KeyIP output."""
    P = plan
    # a7: INTT of the rank's P limbs of acc, exchange #2: every rank gets all P limbs
    p_pos = [P.mine.index(t) for t in P.my_p]
    acc_p_local = ops.intt2(ops.take2(acc, p_pos), P.my_p) if p_pos else ops.empty2(acc, 0)
    acc_p_all = ops.allgather2(acc_p_local, [len(b) for b in P.p_blocks])  # [B][2][num_p][N]
    if P.p_perm is not None:
        acc_p_all = ops.take2(acc_p_all, P.p_perm)
    # a8/a9: ModDown BConv onto the rank's Q limbs, NTT, a10: combine
    if not P.my_q:
        empty = ops.empty2(acc, 0)
        return ops.component(empty, 0), ops.component(empty, 1)
    conv = ops.ntt2(ops.bconv2(acc_p_all, P.p_ids, P.my_q), P.my_q)
    q_pos = [P.mine.index(t) for t in P.my_q]
    out = ops.moddown_combine(ops.take2(acc, q_pos), conv, P.my_q)          # [B][2][n_q][N]
    return ops.component(out, 0), ops.component(out, 1)


class NeoOps:
    """The CUDA library (C-ABI) as the backend of `limb_sharded_keyswitch`, NCCL gathers."""

    def __init__(self, ctx, group=None, stream=None):
        from . import neo
        # resolve the stream once: torch.cuda.current_stream() per C-ABI call costs ~15 us of host time
        self.neo, self.ctx, self.group = neo, ctx, group
        self.stream = stream if stream is not None else torch.cuda.current_stream()
        self._icache = {}

    # ---- tensor plumbing (torch.uint64 CUDA tensors, moved through int64 views because
    #      torch implements few uint64 CUDA ops; the bits are unchanged)
    def _sel(self, x, idx, dim):
        """Rows idx of x along dim: a slice when idx is a run, else index_select with a cached
        device index (a Python list index would be copied host->device, synchronously, per call)."""
        xi = x.view(torch.int64)
        if idx and list(idx) == list(range(idx[0], idx[0] + len(idx))):
            return xi.narrow(dim, idx[0], len(idx)).contiguous().view(torch.uint64)
        key = (tuple(idx), x.device)
        t = self._icache.get(key)
        if t is None:
            t = torch.tensor(list(idx), dtype=torch.int64, device=x.device)
            self._icache[key] = t
        return xi.index_select(dim, t).view(torch.uint64)

    def take(self, x, idx):
        return self._sel(x, idx, 1)

    def take2(self, x, idx):
        return self._sel(x, idx, 2)

    @staticmethod
    def cat(xs, axis):
        return torch.cat([x.view(torch.int64) for x in xs], dim=axis).contiguous().view(torch.uint64)

    @staticmethod
    def stack(xs, axis):
        return torch.stack([x.view(torch.int64) for x in xs], dim=axis).contiguous().view(torch.uint64)

    @staticmethod
    def component(x, c):
        return x.view(torch.int64)[:, c].contiguous().view(torch.uint64)

    @staticmethod
    def empty2(like, n):
        return torch.empty((like.shape[0], 2, n, like.shape[-1]), dtype=torch.uint64, device=like.device)

    def _gather(self, x, sizes, dim):
        world = len(sizes)
        if world == 1:
            return x
        m = max(sizes)
        shape = list(x.shape)
        shape[dim] = m
        pad = torch.zeros(shape, dtype=torch.int64, device=x.device)
        pad.narrow(dim, 0, x.shape[dim]).copy_(x.view(torch.int64))
        if dist.get_backend(self.group) == "nccl":            # device-to-device over NVLink
            parts = [torch.empty_like(pad) for _ in range(world)]
            dist.all_gather(parts, pad, group=self.group)
        else:                                                  # gloo (tests: several ranks on one GPU)
            host = pad.cpu()
            parts = [torch.empty_like(host) for _ in range(world)]
            dist.all_gather(parts, host, group=self.group)
            parts = [p.to(x.device) for p in parts]
        return torch.cat([p.narrow(dim, 0, n) for p, n in zip(parts, sizes)], dim=dim).contiguous().view(torch.uint64)

    def allgather(self, x, sizes):
        return self._gather(x, sizes, 1)

    def allgather2(self, x, sizes):
        return self._gather(x, sizes, 2)

    # ---- arithmetic through the C-ABI
    def intt(self, x, ids):
        y = x.view(torch.int64).clone().view(torch.uint64)
        self.neo.neo_intt(self.ctx, y, ids, y.shape[0], torch.empty_like(y), self.stream)
        return y

    def ntt(self, x, ids):
        y = x.view(torch.int64).clone().view(torch.uint64)
        self.neo.neo_ntt(self.ctx, y, ids, y.shape[0], torch.empty_like(y), self.stream)
        return y

    def intt2(self, x, ids):
        B = x.shape[0]
        return self.intt(x.reshape(2 * B, len(ids), -1), ids).reshape(x.shape)

    def ntt2(self, x, ids):
        B = x.shape[0]
        return self.ntt(x.reshape(2 * B, len(ids), -1), ids).reshape(x.shape)

    def bconv(self, x, src, dst):
        out = torch.empty((x.shape[0], len(dst), x.shape[-1]), dtype=torch.uint64, device=x.device)
        self.neo.neo_bconv(self.ctx, x, src, out, dst, x.shape[0], self.stream)
        return out

    def bconv2(self, x, src, dst):
        B = x.shape[0]
        return self.bconv(x.reshape(2 * B, len(src), -1), src, dst).reshape(B, 2, len(dst), -1)

    def keyip(self, dhat, ids, beta, evk):
        B = dhat.shape[0]
        acc = torch.empty((B, 2, len(ids), dhat.shape[-1]), dtype=torch.uint64, device=dhat.device)
        self.neo.neo_keyip(self.ctx, evk, dhat, ids, beta, acc, B, self.stream)
        return acc

    def ew(self, op, a, b, ids, out=None, scal=None, src=0, batch=None):
        """neo_ew_limbs on the rows `ids` (a new output unless `out` is given)."""
        if out is None:
            shape = list(a.shape)
            if op == self.neo.NEO_EWL_TENSOR:
                shape[1] = 3
            elif op == self.neo.NEO_EWL_LIFT:
                shape = [a.shape[0], 2, len(ids), a.shape[-1]]
            out = torch.empty(shape, dtype=torch.uint64, device=a.device)
        if ids:
            self.neo.neo_ew_limbs(self.ctx, op, a, b if b is not None else a, ids, out,
                                  a.shape[0] if batch is None else batch, scal=scal, src_limb=src, stream=self.stream)
        return out

    def automorphism(self, x, g):
        """sigma_g on every row of x (any leading shape; rows of N)."""
        out = torch.empty_like(x)
        rows = x.numel() // x.shape[-1]
        if rows:
            self.neo.neo_automorphism(self.ctx, x, rows, g, out, 1, self.stream)
        return out

    def broadcast(self, x, src):
        if not dist.is_initialized() or dist.get_world_size(self.group) == 1:
            return x
        if dist.get_backend(self.group) == "nccl":
            dist.broadcast(x.view(torch.int64), src=src, group=self.group)
            return x
        host = x.view(torch.int64).cpu()
        dist.broadcast(host, src=src, group=self.group)
        return host.to(x.device).view(torch.uint64)

    def moddown_combine(self, acc, conv, q_ids):
        out = torch.empty_like(acc)
        self.neo.neo_moddown_combine(self.ctx, acc, conv, q_ids, out, acc.shape[0], self.stream)
        return out
