"""Sparse-slot CKKS bootstrapping on the GPU (PackBootstrap, L529; reading
BOOT in DESIGN.md): an orchestration of the library's own kernels through the C-ABI --
ModRaise, HROTATE (SubSum, the diagonal method, conjugation), PMULT / HADD / HSUB / PADD,
HMULT and Rescale (every HMULT -> Rescale pair as one neo_hmult_rescale call, bit-identical)
-- in the order oracle/boot.py defines (same operations, same operands).

The plaintext constants (CoeffToSlot / SlotToCoeff diagonals, EvalMod's Taylor coefficients,
the monomials +-X^(N/2)) are inputs, like evaluation keys: a dict name -> device tensor
[l+1][N] (NTT form at the level the step runs at).  Their values only matter for correctness
(tests/ produce them with the oracle's encoder); timing is data-independent."""
from __future__ import annotations

import math

import torch

from . import neo

D_TAYLOR = 7


def levels_used(r: int) -> int:
    return 1 + (1 + 3 + 1 + r + 1) + 1


def rotations(N: int, n: int) -> list[int]:
    """Galois elements the run needs: SubSum (n 2^j), the diagonal method (1..n-1), conj (2N-1)."""
    M = N // (2 * n)
    gs = [pow(5, n << j, 2 * N) for j in range(int(math.log2(M)))]
    gs += [pow(5, d, 2 * N) for d in range(1, n)]
    return sorted(set(gs)) + [2 * N - 1]


def const_levels(top: int, n: int, r: int) -> dict:
    """Level of every plaintext constant (the same schedule as run())."""
    lv = {f"cts_{d}": top for d in range(n)}
    l1 = top - 1
    lv["mono_mi"] = l1
    for tag in ("re", "im"):
        lv[f"{tag}theta"] = l1
        y = l1 - 1                                          # y^1 level
        lk = {1: y, 2: y - 1, 3: y - 2, 4: y - 2, 5: y - 3, 6: y - 3, 7: y - 3}
        for k in range(1, D_TAYLOR + 1):
            lv[f"{tag}c{k}"] = lk[k]
        lt = y - 3
        lv[f"{tag}c0"] = lt - 1
        lv[f"{tag}sin"] = lt - 1 - r
    lf = l1 - (1 + 3 + 1 + r + 1)
    lv["mono_i"] = lf
    for d in range(n):
        lv[f"stc_{d}"] = lf
    return lv


def hoisted_rotations(N: int, n: int) -> list[int]:
    """Galois elements of the diagonal method's hoisted rotations (5^d, d = 1 .. n-1)."""
    return [pow(5, d, 2 * N) for d in range(1, n)]


class Bootstrapper:
    """keys: {'relin': EvalKey, g: EvalKey for g in rotations(N, n), ('h', g): hoisted EvalKey
    (neo_evk_create_hoisted) for g in hoisted_rotations(N, n)}; consts: {name: tensor}."""

    def __init__(self, ctx: neo.Context, n: int, r: int, keys: dict, consts: dict, stream=None):
        self.ctx, self.n, self.r, self.keys, self.consts, self.stream = ctx, n, r, keys, consts, stream
        self.N = ctx.N
        self.top = ctx.num_q - 1
        ops = (neo.NEO_OP_HMULT, neo.NEO_OP_HROT, neo.NEO_OP_RESCALE, neo.NEO_OP_MODRAISE, neo.NEO_OP_HROT_HOISTED,
               neo.NEO_OP_HMULT_RESCALE)
        wsn = max(ctx.workspace_size(op, self.top, 2) for op in ops)
        self._stack = {}
        self.ws = torch.empty(wsn // 8, dtype=torch.uint64, device="cuda")

    def _ct(self, level, B=1, lead=()):
        return torch.empty((*lead, B, 2, level + 1, self.N), dtype=torch.uint64, device="cuda")

    # ---- primitive ops (each one C-ABI call)
    # a ciphertext tensor is [B][2][l+1][N]; B = 2 runs EvalMod's real and imaginary halves as
    # one batch (plaintexts: one per batch entry, stacked)
    def rot(self, ct, g, lv):
        B = ct.shape[0]
        out = self._ct(lv, B)
        neo.neo_hrot(self.ctx, self.keys[g], g, ct, lv, out, B, self.ws, self.stream)
        return out

    def add(self, a, b, lv, out=None):
        out = self._ct(lv, a.shape[0]) if out is None else out
        neo.neo_hadd(self.ctx, a, b, lv, out, a.shape[0], self.stream)
        return out

    def sub(self, a, b, lv):
        out = self._ct(lv, a.shape[0])
        neo.neo_hsub(self.ctx, a, b, lv, out, a.shape[0], self.stream)
        return out

    def _pt(self, names):
        return self.consts[names] if isinstance(names, str) else self._stacked(names)

    def _stacked(self, names):
        key = tuple(names)
        if key not in self._stack:
            self._stack[key] = torch.stack([self.consts[k] for k in names]).contiguous()
        return self._stack[key]

    def pmul(self, a, name, lv, out=None):
        out = self._ct(lv, a.shape[0]) if out is None else out
        neo.neo_pmult(self.ctx, a, self._pt(name), lv, out, a.shape[0], self.stream)
        return out

    def padd(self, a, name, lv):
        out = self._ct(lv, a.shape[0])
        neo.neo_padd(self.ctx, a, self._pt(name), lv, out, a.shape[0], self.stream)
        return out

    def rescale(self, a, lv):
        out = self._ct(lv - 1, a.shape[0])
        neo.neo_rescale(self.ctx, a, lv, out, a.shape[0], self.ws, self.stream)
        return out

    def hmul(self, a, b, lv):
        out = self._ct(lv, a.shape[0])
        neo.neo_hmult(self.ctx, self.keys["relin"], a, b, lv, out, a.shape[0], self.ws, self.stream)
        return out

    def hmul_rescale(self, a, b, lv):
        out = self._ct(lv - 1, a.shape[0])
        neo.neo_hmult_rescale(self.ctx, self.keys["relin"], a, b, lv, out, a.shape[0], self.ws, self.stream)
        return out

    def drop(self, a, li, lo):
        if li == lo:
            return a
        out = self._ct(lo, a.shape[0])
        neo.neo_drop_levels(self.ctx, a, li, out, lo, a.shape[0], self.stream)
        return out

    def modraise(self, ct0, L):
        ct = self._ct(L)
        neo.neo_modraise(self.ctx, ct0, L, ct, 1, self.ws, self.stream)
        return ct

    def lintrans(self, ct, lv, tag):           # diagonal method: hoisted rotations + one fused PMULT sum
        N, n = self.N, self.n
        hk = [self.keys[("h", pow(5, d, 2 * N))] for d in range(1, n)]
        rots = self._ct(lv, 1, (n - 1,))
        neo.neo_hrot_hoisted(self.ctx, hk, ct, lv, rots, 1, self.ws, self.stream)
        acc = self._ct(lv)
        neo.neo_pmult_acc(self.ctx, [ct] + [rots[d] for d in range(n - 1)],
                          [self.consts[f"{tag}_{d}"] for d in range(n)], lv, acc, 1, pt_shared=True,
                          stream=self.stream)
        return self.rescale(acc, lv)

    # ---- the run
    def run(self, ct0: torch.Tensor):
        """ct0 [1][2][1][N] (level 0) -> (ct, level)."""
        N, n, L = self.N, self.n, self.top
        M = N // (2 * n)
        ct = self.modraise(ct0, L)
        for j in range(int(math.log2(M))):                             # SubSum
            ct = self.add(ct, self.rot(ct, pow(5, n << j, 2 * N), L), L)
        lintrans = self.lintrans

        ct = lintrans(ct, L, "cts")                                    # CoeffToSlot
        lv = L - 1
        cj = self.rot(ct, 2 * N - 1, lv)
        xs = self._ct(lv, 2)                                            # [x1, x2]: one batch of 2
        self.add(ct, cj, lv, out=xs[0:1])                               # 2 Re(w)
        self.pmul(self.sub(ct, cj, lv), "mono_mi", lv, out=xs[1:2])     # 2 Im(w)

        def evalmod(x, lv, tags):
            y1 = self.rescale(self.pmul(x, [f"{t}theta" for t in tags], lv), lv)
            lv -= 1
            pw = {1: (y1, lv)}

            def mul(a, b):
                (ca, la), (cb, lb) = pw[a], pw[b]
                l0 = min(la, lb)
                pw[a + b] = (self.hmul_rescale(self.drop(ca, la, l0), self.drop(cb, lb, l0), l0), l0 - 1)
            for a, b in ((1, 1), (2, 1), (2, 2), (4, 1), (4, 2), (4, 3)):
                mul(a, b)
            lt = min(l for _, l in pw.values())
            E = None
            for k in range(1, D_TAYLOR + 1):
                ck, lk = pw[k]
                term = self.drop(self.rescale(self.pmul(ck, [f"{t}c{k}" for t in tags], lk), lk), lk - 1, lt - 1)
                E = term if E is None else self.add(E, term, lt - 1)
            lv = lt - 1
            E = self.padd(E, [f"{t}c0" for t in tags], lv)
            for _ in range(self.r):
                E = self.hmul_rescale(E, E, lv)
                lv -= 1
            cE = self.rot(E, 2 * N - 1, lv)
            f = self.rescale(self.pmul(self.sub(E, cE, lv), [f"{t}sin" for t in tags], lv), lv)
            return f, lv - 1

        # EvalMod of the real and imaginary halves as one batch of 2
        f, lv = evalmod(xs, lv, ("re", "im"))
        w = self.add(f[0:1], self.pmul(f[1:2], "mono_i", lv), lv)
        out = lintrans(w, lv, "stc")                                   # SlotToCoeff
        return out, lv - 1
