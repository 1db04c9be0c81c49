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


def levels_used(r: int, fft_levels: int = 0, boost: tuple = (0, 0), ds_sq: int = 0) -> int:
    lt = max(1, fft_levels)
    extra = 1 if (boost[0] or ds_sq) else 0                  # theta's Double Rescale
    if ds_sq:
        extra += 3 + 1 + ds_sq + 2                           # powers, Taylor terms, squarings, the 3-prime one
    return lt + (1 + 3 + 1 + r + 1) + lt + extra


def _sq_primes(i: int, ds_sq: int) -> int:
    """Primes the i-th EvalMod squaring divides by: 2 while at ~q^2, 3 once to return to ~q, then 1."""
    if not ds_sq:
        return 1
    return 2 if i < ds_sq else 3 if i == ds_sq else 1


# ---- full-slot linear transforms (n = N/2): the special FFT's log2(n) butterfly stages, stage
# F_len mixing slots p and p + len/2 (rotation amounts 0, +-len/2), merged into fft_levels
# groups; CoeffToSlot applies the stages from len = n down to 2, SlotToCoeff from 2 up to n.
# Only the rotation structure is computed here (the diagonals are plaintext inputs).

def fft_plan(N: int, fft_levels: int, inverse: bool) -> list[tuple[int, int, list[int]]]:
    """Per level: (h, b1, ms) -- the group's rotation amounts are m h (m in ms, signed mod N/2),
    evaluated baby-step giant-step with m = g b1 + b, b in [0, b1)."""
    n = N // 2
    lenhs = [1 << k for k in range(int(math.log2(n)))]           # F_2 .. F_n: len/2 = 1 .. n/2
    order = lenhs[::-1] if inverse else lenhs
    L = len(order)
    sizes = [L // fft_levels + (1 if i < L % fft_levels else 0) for i in range(fft_levels)]
    plan, k = [], 0
    for sz in sizes:
        amounts = {0}
        for lh in order[k:k + sz]:
            amounts = {((a + e * lh) + n // 2) % n - n // 2 for a in amounts for e in (-1, 0, 1)}
        if sz == 1:                                                # an unmerged stage keeps +-n/2 apart
            amounts = {0, order[k], -order[k]}
        h = min(abs(a) for a in amounts if a)
        ms = sorted(a // h for a in amounts)
        b1 = 1
        while b1 * b1 < len(ms):
            b1 *= 2
        plan.append((h, b1, ms))
        k += sz
    return plan


def fft_rotations(N: int, fft_levels: int) -> tuple[list[int], list[int]]:
    """(hoisted baby-step Galois elements, giant-step Galois elements) of both transforms."""
    n = N // 2
    hoisted, giant = set(), set()
    for inverse in (True, False):
        for h, b1, ms in fft_plan(N, fft_levels, inverse):
            hoisted |= {pow(5, ((m % b1) * h) % n, 2 * N) for m in ms if m % b1}
            giant |= {pow(5, ((m // b1) * b1 * h) % n, 2 * N) for m in ms if m // b1}
    return sorted(hoisted), sorted(giant)


def rotations(N: int, n: int, fft_levels: int = 0) -> list[int]:
    """Galois elements the run needs: SubSum (n 2^j), the linear transforms, conj (2N-1)."""
    M = N // (2 * n)
    gs = [pow(5, n << j, 2 * N) for j in range(int(math.log2(M)))]
    if fft_levels:
        hz, gz = fft_rotations(N, fft_levels)
        gs += hz + gz
    else:
        gs += [pow(5, d, 2 * N) for d in range(1, n)]
    return sorted(set(gs)) + [2 * N - 1]


def _fft_const_names(N: int, fft_levels: int, inverse: bool, tag: str) -> list[list[str]]:
    out = []
    for k, (h, b1, ms) in enumerate(fft_plan(N, fft_levels, inverse)):
        out.append([f"{tag}{k}_g{m // b1}_b{m % b1}" for m in ms])
    return out


def const_levels(top: int, n: int, r: int, N: int = 0, fft_levels: int = 0, boost: tuple = (0, 0),
                 ds_sq: int = 0) -> dict:
    """Level of every plaintext constant (the same schedule as run())."""
    F = max(1, fft_levels)
    if fft_levels:
        lv = {nm: top - k for k, names in enumerate(_fft_const_names(N, fft_levels, True, "cts")) for nm in names}
    else:
        lv = {f"cts_{d}": top for d in range(n)}
    if boost[0]:
        lv["boost_cts"] = top
    l1 = top - F
    lv["mono_mi"] = l1
    m = 2 if ds_sq else 1                                   # primes per rescale while EvalMod is at ~q^2
    m_th = 2 if (boost[0] or ds_sq) else 1                  # theta's product ends in a Double Rescale
    for tag in ("re", "im"):
        lv[f"{tag}theta"] = l1
        pw = {1: l1 - m_th}                                 # y^k levels
        for a, b in ((1, 1), (2, 1), (2, 2), (4, 1), (4, 2), (4, 3)):
            pw[a + b] = min(pw[a], pw[b]) - m
        for k in range(1, D_TAYLOR + 1):
            lv[f"{tag}c{k}"] = pw[k]
        le = min(pw.values()) - m
        lv[f"{tag}c0"] = le
        for i in range(r):
            le -= _sq_primes(i, ds_sq)
        lv[f"{tag}sin"] = le
    lf = lv["resin"] - 1
    lv["mono_i"] = lf
    if boost[1]:
        lv["boost_stc"] = lf
    if fft_levels:
        for k, names in enumerate(_fft_const_names(N, fft_levels, False, "stc")):
            lv.update({nm: lf - k for nm in names})
    else:
        for d in range(n):
            lv[f"stc_{d}"] = lf
    return lv


def hoisted_rotations(N: int, n: int, fft_levels: int = 0) -> list[int]:
    """Galois elements of the hoisted rotations: the diagonal method's 5^d (d = 1 .. n-1), or the
    full-slot transforms' baby steps."""
    if fft_levels:
        return fft_rotations(N, fft_levels)[0]
    return [pow(5, d, 2 * N) for d in range(1, n)]


class Bootstrapper:
    """keys: {'relin': EvalKey, g: EvalKey for g in rotations(N, n), ('h', g): hoisted EvalKey
    (neo_evk_create_hoisted) for g in hoisted_rotations(N, n)}; consts: {name: tensor}."""

    def __init__(self, ctx: neo.Context, n: int, r: int, keys: dict, consts: dict, stream=None,
                 fft_levels: int = 0, boost: tuple = (0, 0), ds_sq: int = 0):
        self.ctx, self.n, self.r, self.keys, self.consts, self.stream = ctx, n, r, keys, consts, stream
        self.fft_levels = fft_levels
        self.boost = tuple(boost)
        self.ds_sq = ds_sq
        self.N = ctx.N
        self.top = ctx.num_q - 1
        ops = (neo.NEO_OP_HMULT, neo.NEO_OP_HROT, neo.NEO_OP_RESCALE, neo.NEO_OP_MODRAISE, neo.NEO_OP_HROT_HOISTED,
               neo.NEO_OP_HMULT_RESCALE, neo.NEO_OP_HROT_SUM, neo.NEO_OP_DOUBLE_RESCALE)
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

    def double_rescale(self, a, lv):
        out = self._ct(lv - 2, a.shape[0])
        neo.neo_double_rescale(self.ctx, a, lv, out, a.shape[0], self.ws, self.stream)
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

    def rot_hoisted(self, ct, gs, lv):
        """[sigma-rotations of ct by the Galois elements gs] sharing one ModUp."""
        out = self._ct(lv, ct.shape[0], (len(gs),))
        neo.neo_hrot_hoisted(self.ctx, [self.keys[("h", g)] for g in gs], ct, lv, out, ct.shape[0], self.ws,
                             self.stream)
        return [out[i] for i in range(len(gs))]

    def rot_sum(self, cts, gs, lv):
        """sum_k HROTATE(cts[k], gs[k]) with one ModDown (neo_hrot_sum, reading BOOT-G)."""
        out = self._ct(lv, cts[0].shape[0])
        neo.neo_hrot_sum(self.ctx, [self.keys[g] for g in gs], gs, cts, lv, out, cts[0].shape[0], self.ws,
                         self.stream)
        return out

    def pmul_sum(self, cts, names, lv):
        """sum_k PMULT(cts[k], consts[names[k]]) in one launch."""
        out = self._ct(lv, cts[0].shape[0])
        neo.neo_pmult_acc(self.ctx, cts, [self.consts[nm] for nm in names], lv, out, cts[0].shape[0],
                          pt_shared=True, stream=self.stream)
        return out

    def lintrans_fft(self, ct, lv, inverse, tag):
        """Full-slot CoeffToSlot / SlotToCoeff: fft_levels baby-step giant-step levels."""
        N, n = self.N, self.N // 2
        for k, (h, b1, ms) in enumerate(fft_plan(N, self.fft_levels, inverse)):
            babies = sorted({m % b1 for m in ms} - {0})
            rots = {0: ct}
            if babies:
                rots.update(zip(babies, self.rot_hoisted(ct, [pow(5, (b * h) % n, 2 * N) for b in babies], lv)))
            acc, rin, rg = None, [], []
            for g in sorted({m // b1 for m in ms}):
                bs = [m % b1 for m in ms if m // b1 == g]
                inner = self.pmul_sum([rots[b] for b in bs], [f"{tag}{k}_g{g}_b{b}" for b in bs], lv)
                if g:
                    rin.append(inner)
                    rg.append(pow(5, (g * b1 * h) % n, 2 * N))
                else:
                    acc = inner
            if rin:                                            # giant steps: one shared ModDown
                r = self.rot_sum(rin, rg, lv)
                acc = r if acc is None else self.add(acc, r, lv)
            ct = self.rescale(acc, lv)
            lv -= 1
        return ct, lv

    # ---- the run
    def run(self, ct0: torch.Tensor):
        """ct0 [1][2][1][N] (level 0) -> (ct, level)."""
        N, n, L = self.N, self.n, self.top
        M = N // (2 * n)
        ct = self.modraise(ct0, L)
        for j in range(int(math.log2(M))):                             # SubSum
            ct = self.add(ct, self.rot(ct, pow(5, n << j, 2 * N), L), L)
        lintrans = self.lintrans
        k1, k2 = self.boost
        if k1:                                                         # exact x 2^k1 (reading BOOT-S)
            ct = self.pmul(ct, "boost_cts", L)

        if self.fft_levels:
            ct, lv = self.lintrans_fft(ct, L, True, "cts")             # CoeffToSlot (bit-reversed)
        else:
            ct = lintrans(ct, L, "cts")                                # CoeffToSlot
            lv = L - 1
        cj = self.rot(ct, 2 * N - 1, lv)
        xs = self._ct(lv, 2)                                            # [x1, x2]: one batch of 2
        self.add(ct, cj, lv, out=xs[0:1])                               # 2 Re(w)
        self.pmul(self.sub(ct, cj, lv), "mono_mi", lv, out=xs[1:2])     # 2 Im(w)

        ds = self.ds_sq

        def rs(ct, lv, m):             # Rescale (1), Double Rescale (2), both (3) -- the oracle's rs()
            if m == 1:
                return self.rescale(ct, lv)
            ct = self.double_rescale(ct, lv)
            return self.rescale(ct, lv - 2) if m == 3 else ct

        def evalmod(x, lv, tags):
            m = 2 if ds else 1
            m_th = 2 if (k1 or ds) else 1                              # theta: Double Rescale
            y1 = rs(self.pmul(x, [f"{t}theta" for t in tags], lv), lv, m_th)
            lv -= m_th
            pw = {1: (y1, lv)}

            def mul(a, b):
                (ca, la), (cb, lb) = pw[a], pw[b]
                l0 = min(la, lb)
                if m == 1:
                    pw[a + b] = (self.hmul_rescale(self.drop(ca, la, l0), self.drop(cb, lb, l0), l0), l0 - 1)
                else:
                    pw[a + b] = (rs(self.hmul(self.drop(ca, la, l0), self.drop(cb, lb, l0), l0), l0, m), l0 - m)
            for a, b in ((1, 1), (2, 1), (2, 2), (4, 1), (4, 2), (4, 3)):
                mul(a, b)
            lt = min(l for _, l in pw.values())
            E = None
            for k in range(1, D_TAYLOR + 1):
                ck, lk = pw[k]
                term = self.drop(rs(self.pmul(ck, [f"{t}c{k}" for t in tags], lk), lk, m), lk - m, lt - m)
                E = term if E is None else self.add(E, term, lt - m)
            lv = lt - m
            E = self.padd(E, [f"{t}c0" for t in tags], lv)
            for i in range(self.r):
                mi = _sq_primes(i, ds)
                E = self.hmul_rescale(E, E, lv) if mi == 1 else rs(self.hmul(E, E, lv), lv, mi)
                lv -= mi
            cE = self.rot(E, 2 * N - 1, lv)
            f = self.rescale(self.pmul(self.sub(E, cE, lv), [f"{t}sin" for t in tags], lv), lv)
            return f, lv - 1

        # EvalMod of the real and imaginary halves as one batch of 2
        f, lv = evalmod(xs, lv, ("re", "im"))
        w = self.add(f[0:1], self.pmul(f[1:2], "mono_i", lv), lv)
        if k2:
            w = self.pmul(w, "boost_stc", lv)
        if self.fft_levels:
            return self.lintrans_fft(w, lv, False, "stc")              # SlotToCoeff
        out = lintrans(w, lv, "stc")                                   # SlotToCoeff
        return out, lv - 1
