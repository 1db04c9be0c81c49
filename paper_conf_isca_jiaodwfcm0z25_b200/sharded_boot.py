"""Limb-sharded CKKS evaluation and bootstrapping (bootstrapping
"with limb-sharded BConv all-gather over 8 B200"; §8(e) P2).

Every rank holds the Q limbs i with i mod world == rank of every ciphertext (round-robin, so
the limb a Rescale drops rotates over the ranks and the shards stay balanced), as a tensor
[B][2][n_own(level)][N] in ascending limb order.  Element-wise work is limb-local
(`neo_ew_limbs`, `neo_automorphism` on the rank's rows); the only exchanges are

* the key-switch's two all-gathers (`sharded.limb_sharded_keyswitch`: coefficient-form Q limbs
  before ModUp, P limbs before ModDown) inside every HMULT / HROTATE, and
* one broadcast of the 2B coefficient rows of the dropped limb per Rescale (its owner runs the
  INTT; every rank reduces it onto its own limbs with a one-input BConv, NTTs and finishes with
  (c_i - r_i) q_l^-1), and of limb 0 for ModRaise.

`ShardedBootstrapper` runs paper_conf_isca_jiaodwfcm0z25_b200.boot's schedule (the same
operations on the same operands, hoisted rotations included) on shards, so the gathered result
is bit-identical to the single-GPU bootstrap and to oracle/boot.py."""
from __future__ import annotations

import torch

from . import neo
from .boot import Bootstrapper
from .sharded import NeoOps, ShardPlan, limb_sharded_keyip, limb_sharded_keyswitch, limb_sharded_moddown


class ShardedBootstrapper(Bootstrapper):
    """keys as for Bootstrapper (full keys on every rank; KeyIP reads the rank's limbs);
    consts: full plaintexts [l+1][N] (each rank keeps its own rows)."""

    def __init__(self, ctx: neo.Context, n: int, r: int, keys: dict, consts: dict, world: int, rank: int,
                 group=None, stream=None, fft_levels: int = 0, boost: tuple = (0, 0), ds_sq: int = 0):
        self.ctx, self.n, self.r, self.keys, self.stream = ctx, n, r, keys, stream
        self.fft_levels = fft_levels
        self.boost = tuple(boost)
        self.ds_sq = ds_sq
        self.N = ctx.N
        self.top = ctx.num_q - 1
        self.world, self.rank = world, rank
        self.ops = NeoOps(ctx, group, stream)
        self._stack = {}
        self.consts = {k: v.view(torch.int64)[self.own(v.shape[0] - 1)].contiguous().view(torch.uint64)
                       for k, v in consts.items()}
        self._qinv = {}

    # ---- ownership
    def own(self, level: int) -> list[int]:
        return list(range(self.rank, level + 1, self.world))

    def owner(self, limb: int) -> int:
        return limb % self.world

    def _ct(self, level, B=1, lead=()):
        return torch.empty((*lead, B, 2, len(self.own(level)), self.N), dtype=torch.uint64, device="cuda")

    def shard(self, ct_full: torch.Tensor, level: int) -> torch.Tensor:
        """This rank's rows of a full ciphertext [B][2][level+1][N]."""
        return ct_full.view(torch.int64)[:, :, self.own(level)].contiguous().view(torch.uint64)

    def double_rescale(self, a, lv):
        """Double Rescale as two sharded Rescales (bit-identical: floor(floor(x/a)/b) = floor(x/ab),
        pinned in test_oracle_ops.py)."""
        return self.rescale(self.rescale(a, lv), lv - 1)

    def _ks(self, d_local, lv, key):
        plan = ShardPlan(lv, self.ctx.num_q, self.ctx.num_p, self.ctx.alpha, self.world, self.rank, strided=True)
        return limb_sharded_keyswitch(self.ops, plan, d_local, key)

    def _ew(self, op, a, b, lv, out=None, scal=None):
        return self.ops.ew(op, a, b, self.own(lv), out=out, scal=scal)

    def _pt_b(self, names, B):
        pt = self._pt(names)
        return pt if pt.dim() == 3 else pt.unsqueeze(0).expand(B, -1, -1).contiguous()

    # ---- element-wise (limb-local)
    def add(self, a, b, lv, out=None):
        return self._ew(neo.NEO_EWL_HADD, a, b, lv, out)

    def sub(self, a, b, lv):
        return self._ew(neo.NEO_EWL_HSUB, a, b, lv)

    def pmul(self, a, name, lv, out=None):
        return self._ew(neo.NEO_EWL_PMULT, a, self._pt_b(name, a.shape[0]), lv, out)

    def padd(self, a, name, lv):
        return self._ew(neo.NEO_EWL_PADD, a, self._pt_b(name, a.shape[0]), lv)

    def drop(self, a, li, lo):
        if li == lo:
            return a
        return a.view(torch.int64)[:, :, : len(self.own(lo))].contiguous().view(torch.uint64)

    # ---- key-switching ops (two all-gathers each)
    def _plus_k(self, c0, k0, k1, lv):
        """(c0 + k0, k1) as one ciphertext shard."""
        pre = torch.stack([c0.view(torch.int64), k1.view(torch.int64)], dim=1).contiguous().view(torch.uint64)
        return self._ew(neo.NEO_EWL_PADD, pre, k0, lv)

    def rot(self, ct, g, lv):
        s = self.ops.automorphism(ct, g)                       # sigma_g on c0 and c1, limb-local
        k0, k1 = self._ks(s[:, 1].contiguous(), lv, self.keys[g])
        return self._plus_k(s[:, 0].contiguous(), k0, k1, lv)

    def hmul(self, a, b, lv):
        d = self._ew(neo.NEO_EWL_TENSOR, a, b, lv)             # [B][3][n][N]
        k0, k1 = self._ks(d[:, 2].contiguous(), lv, self.keys["relin"])
        kk = torch.stack([k0.view(torch.int64), k1.view(torch.int64)], dim=1).contiguous().view(torch.uint64)
        return self._ew(neo.NEO_EWL_HADD, d[:, :2].contiguous(), kk, lv)

    def hmul_rescale(self, a, b, lv):
        return self.rescale(self.hmul(a, b, lv), lv)

    # ---- exchanges of one limb
    def _limb_coeffs(self, ct, limb, lv):
        """Coefficient form of limb `limb` of both components, [B][2][N], on every rank."""
        B = ct.shape[0]
        if self.rank == self.owner(limb):
            pos = self.own(lv).index(limb)
            row = ct.view(torch.int64)[:, :, pos].contiguous().view(torch.uint64).view(2 * B, 1, self.N)
            coef = self.ops.intt(row, [limb]).view(B, 2, self.N)
        else:
            coef = torch.empty((B, 2, self.N), dtype=torch.uint64, device=ct.device)
        return self.ops.broadcast(coef, self.owner(limb))

    def rescale(self, a, lv):
        """(c_i - [c_l]_{q_l} mod q_i) q_l^-1 (L137, Z10) on this rank's limbs i < l."""
        B = a.shape[0]
        coef = self._limb_coeffs(a, lv, lv)
        ids = self.own(lv - 1)
        if not ids:
            return self._ct(lv - 1, B)
        r = self.ops.ntt(self.ops.bconv(coef.view(2 * B, 1, self.N), [lv], ids), ids).view(B, 2, len(ids), self.N)
        if (lv, tuple(ids)) not in self._qinv:                    # the context's constants (C-ABI)
            self._qinv[(lv, tuple(ids))] = neo.neo_query_ql_inv(self.ctx, lv, ids)
        return self._ew(neo.NEO_EWL_SUBMUL, self.drop(a, lv, lv - 1), r, lv - 1, scal=self._qinv[(lv, tuple(ids))])

    def modraise(self, ct0, L):
        """ct0: this rank's shard of the level-0 ciphertext ([1][2][1][N] on limb 0's owner,
        [1][2][0][N] elsewhere) -> its rows of ModRaise at level L."""
        coef = self._limb_coeffs(ct0, 0, 0)
        ids = self.own(L)
        lifted = self.ops.ew(neo.NEO_EWL_LIFT, coef, None, ids, src=0)        # [1][2][n][N] coefficients
        return self.ops.ntt(lifted.view(2, len(ids), self.N), ids).view(1, 2, len(ids), self.N)

    def rot_hoisted(self, ct, gs, lv):
        """Hoisted rotations (BOOT-H) on shards: per g the key-switch of c1 under the hoisted key,
        then sigma_g of (c0 + k0', k1')."""
        out = []
        for g in gs:
            k0, k1 = self._ks(ct[:, 1].contiguous(), lv, self.keys[("h", g)])
            out.append(self.ops.automorphism(self._plus_k(ct[:, 0].contiguous(), k0, k1, lv), g))
        return out

    def rot_sum(self, cts, gs, lv):
        """sum_k HROTATE(cts[k], gs[k]) with one ModDown (BOOT-G): KeyIP outputs summed on the
        rank's PQ_l rows, one sharded ModDown, plus the summed sigma_g(c0)."""
        plan = ShardPlan(lv, self.ctx.num_q, self.ctx.num_p, self.ctx.alpha, self.world, self.rank, strided=True)
        acc = sig = None
        for ct, g in zip(cts, gs):
            sg = self.ops.automorphism(ct, g)
            a = limb_sharded_keyip(self.ops, plan, sg[:, 1].contiguous(), self.keys[g])
            acc = a if acc is None else self.ops.ew(neo.NEO_EWL_HADD, acc, a, plan.mine)
            sig = sg if sig is None else self.add(sig, sg, lv)
        k0, k1 = limb_sharded_moddown(self.ops, plan, acc)
        return self._plus_k(sig[:, 0].contiguous(), k0, k1, lv)

    def pmul_sum(self, cts, names, lv):
        acc = self.pmul(cts[0], names[0], lv)
        for c, nm in zip(cts[1:], names[1:]):
            acc = self.add(acc, self.pmul(c, nm, lv), lv)
        return acc

    def lintrans(self, ct, lv, tag):
        """The diagonal method with hoisted rotations (BOOT-H): for g = 5^d the key-switch of c1
        under the hoisted key sigma_g^-1(rotkey_g), then sigma_g of (c0 + k0', k1')."""
        N, n = self.N, self.n
        acc = self.pmul(ct, f"{tag}_0", lv)
        for d in range(1, n):
            g = pow(5, d, 2 * N)
            k0, k1 = self._ks(ct[:, 1].contiguous(), lv, self.keys[("h", g)])
            rot_d = self.ops.automorphism(self._plus_k(ct[:, 0].contiguous(), k0, k1, lv), g)
            acc = self.add(acc, self.pmul(rot_d, f"{tag}_{d}", lv), lv)
        return self.rescale(acc, lv)
