"""CPU ORACLE of CKKS bootstrapping (PackBootstrap of L529) -- TEST
INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
``--impl reference`` legs may import this module; it shares no code with the CUDA path.

The paper names bootstrapping's three parts (CoeffToSlot, EvalMod, SlotToCoeff, L529) and the
Double Rescale it needs at 36-bit words (L138, L151) but gives no algorithm or parameters (it
cites Lattigo [34]).  Reading "BOOT" -- the textbook sparse-slot bootstrapping of
Cheon, Han, Kim, Kim, Song (EUROCRYPT'18), built only from the operations pinned elsewhere
(HROTATE, HMULT, PMULT, HADD/HSUB, Rescale) plus ModRaise:

  ModRaise  ct mod q_0 -> mod Q_L, coefficients lifted centred: m + q_0 I, I small
  SubSum    sum of the rotations by n 2^j: the trace onto the degree-2n subring (x M = N / 2n)
  CoeffToSlot  slots <- A z with A = W^-1 / M, W[k][j] = xi^(j 5^k), xi = e^(i pi / 2n): the slot
            j then holds (p_{Mj} + i p_{M(j+n)}) / q_0 (diagonal method, one PMULT level; its
            n - 1 rotations of one ciphertext are hoisted rotations: one ModUp, reading BOOT-H)
  split     Re = (w + conj w) / 2, Im = (w - conj w) / 2i   (conjugation = HROTATE, g = 2N - 1)
  EvalMod   y = theta t (theta = 2 pi / 2^r), E = sum_{k<=7} (i y)^k / k!, E <- E^2 r times
            (= exp(2 pi i t)), f = (E - conj E) (-i / 4 pi) = sin(2 pi t) / 2 pi ~ t mod 1 = m / q_0
  combine   f(Re) + i f(Im)  (i = the monomial X^(N/2): PMULT by a scale-1 plaintext, exact)
  SlotToCoeff  slots <- W v (diagonal method): the message slots, value z Delta_in / q_0

Every plaintext constant is encoded at a scale that makes the next rescale restore the
ciphertext's scale, so scales are tracked exactly; the constants are returned so the GPU run
uses the same ones (tests/test_gpu_boot.py: bit-exact).  Pinned by decoding (the output
decrypts to the input slots) and by ModRaise's exact big-integer identity."""
from __future__ import annotations

import collections
import math
from dataclasses import dataclass

import numpy as np

from . import ckks

D_TAYLOR = 7                                 # degree of the exp Taylor polynomial (powers y .. y^7)


@dataclass
class BootParams:
    prm: ckks.Params
    n: int                                   # complex slots (sparse packing), n | N/2
    r: int                                   # squarings in EvalMod
    h: int = 192                             # secret Hamming weight (bounds I)
    fft_levels: int = 0                      # 0: dense diagonal method; k: factored CtS / StC, k levels each
    boost: tuple = (0, 0)                    # (k1, k2): exact x 2^k scale boosts before CoeffToSlot / SlotToCoeff
    ds_sq: int = 0                           # EvalMod at ~q^2 (Double Rescale) up to this many squarings (< r)

    @property
    def M(self) -> int:
        return self.prm.N // (2 * self.n)

    @property
    def top(self) -> int:
        return self.prm.max_level

    def levels_used(self) -> int:            # CtS, EvalMod 1 + 3 + 1 + r + 1, StC (+ the Double Rescales)
        lt = max(1, self.fft_levels)
        extra = 1 if (self.boost[0] or self.ds_sq) else 0            # theta
        if self.ds_sq:
            extra += 3 + 1 + self.ds_sq + 2                          # powers, Taylor terms, squarings, 3-prime one
        return lt + (1 + 3 + 1 + self.r + 1) + lt + extra

    def rotations(self) -> list[int]:
        """Galois elements: SubSum (rotations by n 2^j), the linear transforms' rotations, conj."""
        N = self.prm.N
        gs = [pow(5, self.n << j, 2 * N) for j in range(int(math.log2(self.M)))]
        if self.fft_levels:
            for grp in fft_groups(N, self.fft_levels, inverse=True) + fft_groups(N, self.fft_levels, inverse=False):
                babies, giants = bsgs_amounts(grp, N)
                gs += [pow(5, d % (N // 2), 2 * N) for d in babies + giants]
        else:
            gs += [pow(5, d, 2 * N) for d in range(1, self.n)]
        return sorted(set(gs)) + [2 * N - 1]


def tiny_full(fft_levels: int = 3) -> BootParams:
    """Full-slot test set: N = 2^12 (2048 slots), r = 9, h = 32, CoeffToSlot / SlotToCoeff as
    fft_levels levels each.  3 levels: 24 Q + 2 P limbs (dnum 12: alpha = 2), output level 2;
    4 levels: 25 Q + 3 P limbs (dnum 9: alpha = 3), output level 1."""
    if fft_levels == 3:
        return BootParams(ckks.Params(12, 24, 2, 12), n=2048, r=9, h=32, fft_levels=3)
    return BootParams(ckks.Params(12, 21 + fft_levels, 3, -(-(21 + fft_levels) // 3)), n=2048, r=9, h=32,
                      fft_levels=fft_levels)


def tiny_full_boost() -> BootParams:
    """tiny_full(4) with the reading-BOOT-S scale boosts (2^12) and theta's Double Rescale:
    N = 2^12, 26 Q + 3 P limbs (dnum 9), output level 1 (its 72-bit modulus holds the
    2^12-boosted output scale; the GPU replays it bit for bit)."""
    return BootParams(ckks.Params(12, 26, 3, 9), n=2048, r=9, h=32, fft_levels=4, boost=(12, 12))


def tiny_full_ds() -> BootParams:
    """The reading-BOOT-S schedule Set-B runs with, at N = 2^12: 2^12 boosts, EvalMod at ~q^2 (Double
    Rescale) for the theta product, the Taylor powers and terms and the first 4 of r = 9 squarings;
    37 Q + 4 P limbs (dnum 10), output level 2."""
    return BootParams(ckks.Params(12, 37, 4, 10), n=2048, r=9, h=32, fft_levels=4, boost=(12, 12), ds_sq=4)


def set_b_full() -> BootParams:
    """Set-B with all N/2 = 32768 slots, CtS / StC as 4 levels of 4-4-4-3 special-FFT stages, and
    reading BOOT-S: 2^20 scale boosts before both linear transforms, EvalMod with r = 9 squarings
    whose theta product, Taylor powers and terms and first 4 squarings run at ~q^2 scale with
    Double Rescales (L138, L151: what keeps 36-bit words precise) -- levels 35 -> 1.  With
    single-prime rescales throughout (r = 12) the key-switch and rescale noise at ~2^36 scale,
    amplified 2^r by the squarings, swamps the message (decode error ~1, tools/boot_setb_diag.py)."""
    return BootParams(ckks.set_b(), n=32768, r=9, h=192, fft_levels=4, boost=(20, 20), ds_sq=4)


def tiny() -> BootParams:
    """Test set: N = 2^12, 19 Q limbs + 2 P limbs (dnum 10: alpha = 2), 8 slots, r = 9, h = 32."""
    return BootParams(ckks.Params(12, 19, 2, 10), n=8, r=9, h=32)


def set_b() -> BootParams:
    """Set-B (Table 4) with 8 sparse slots and the schedule of set_b_full (reading BOOT-S: 2^20
    boosts, EvalMod r = 9 with its first steps at ~q^2 via Double Rescale), levels 35 -> 7."""
    return BootParams(ckks.set_b(), n=8, r=9, h=192, boost=(20, 20), ds_sq=4)


# --------------------------------------------------------------------------- slot algebra

def _xi_matrix(n: int) -> np.ndarray:
    """W[k][j] = xi^(j 5^k), xi = e^(i pi / 2n): slots of a degree-2n subring polynomial."""
    e5 = [pow(5, k, 4 * n) for k in range(n)]
    return np.array([[np.exp(1j * math.pi * ((j * e) % (4 * n)) / (2 * n)) for j in range(n)] for e in e5])


def _diagonals(A: np.ndarray) -> list[np.ndarray]:
    n = A.shape[0]
    return [np.array([A[k][(k + d) % n] for k in range(n)]) for d in range(n)]


def _round_big(scale: float, x: float) -> int:
    """round(scale x), half away from zero, exactly in integers for any float scale (the product
    of two doubles is formed exactly from their integer mantissas)."""
    from fractions import Fraction
    y = Fraction(scale) * Fraction(x)
    r = abs(y).__floor__() + (1 if abs(y) - abs(y).__floor__() >= Fraction(1, 2) else 0)
    return r if y >= 0 else -r


def _pt(bp: BootParams, slots_n: np.ndarray, scale: float, level: int) -> np.ndarray:
    """Plaintext (NTT form, level) whose full-slot vector is slots_n tiled, at `scale`.  A
    constant vector c is encoded in closed form, m = round(scale Re c) + round(scale Im c) X^(N/2)
    (X^(N/2) is i in every slot; encode()'s sum is zero at every other coefficient), which is
    encode()'s result without its O(N^2) sum (pinned equal in tests/test_oracle_boot.py)."""
    prm = bp.prm
    ids = list(range(level + 1))
    v = np.asarray(slots_n, dtype=complex)
    if np.all(v == v[0]):
        m = np.zeros(prm.N, dtype=object)                                  # scales up to ~2^110: Python ints
        m[:] = 0
        m[0] = _round_big(scale, v[0].real)
        m[prm.N // 2] = _round_big(scale, v[0].imag)
    else:   # N >= 2^14: encode_fft (within 1 of encode, pinned; any valid encoding, reading BOOT-F)
        enc = ckks.encode_fft if prm.N >= 1 << 14 else ckks.encode
        m = enc(prm.N, np.tile(v, bp.M), scale)
    return ckks.ntt(prm, ckks.reduce_signed(prm, m, ids), ids)


def _const_int(prm: ckks.Params, c: int, level: int) -> np.ndarray:
    """NTT form of the constant polynomial c (an exact integer plaintext: PMULT by it multiplies
    the message by c without a Rescale)."""
    return np.stack([np.full(prm.N, c % prm.moduli[i], dtype=np.uint64) for i in range(level + 1)])


def _monomial(prm: ckks.Params, k: int, sign: int, level: int) -> np.ndarray:
    """NTT form of sign * X^k (an exact scale-1 plaintext): X^(N/2) multiplies every slot by i."""
    ids = list(range(level + 1))
    c = np.zeros(prm.N, dtype=np.int64)
    c[k] = sign
    return ckks.ntt(prm, ckks.reduce_signed(prm, c, ids), ids)


# --------------------------------------------------------------------------- special FFT (full slots)
# With n = N/2 slots the slot vector of a polynomial t (at scale 1) is z = U (t_lo + i t_hi),
# U[j][k] = zeta^(5^j k), zeta = e^(i pi / N) (zeta^(5^j N/2) = i).  U factors into log2(n)
# butterfly stages after a bit-reversal P (the "special FFT" of the CKKS encoder):
#     U = F_n ... F_4 F_2 P,   F_len: out[i+j] = u + w v, out[i+j+len/2] = u - w v,
#     u = in[i+j], v = in[i+j+len/2], w = zeta^((5^j mod 4 len) 2N / (4 len)),  j < len/2,
# so CoeffToSlot = P U^-1 = F_2^-1 ... F_n^-1 (slots end in bit-reversed order, which the
# slot-wise EvalMod does not see) and SlotToCoeff = U P^-1 = F_n ... F_2.  Every stage is three
# rotation diagonals; a level applies a group of consecutive stages merged into one matrix
# (2^(k+1) - 1 diagonals for k stages), evaluated baby-step giant-step.

def _rot(v: np.ndarray, d: int) -> np.ndarray:
    """rot_d(v)[p] = v[(p + d) mod n] (a left rotation by d, Z11)."""
    return np.roll(v, -d)


def sfft_stages(N: int, inverse: bool) -> list[dict]:
    """[F_2, F_4, ..., F_n] (inverse=False) or [F_2^-1, ..., F_n^-1], each {amount d: diagonal}
    with (F x)[p] = sum_d diag_d[p] x[p + d]."""
    n = N // 2
    e5 = np.array([pow(5, j, 2 * N) for j in range(n)], dtype=np.int64)
    p = np.arange(n)
    out = []
    ln = 2
    while ln <= n:
        lenh, lenq = ln // 2, 4 * ln
        j = p % ln
        first = j < lenh
        jj = np.where(first, j, j - lenh)
        w = np.exp(1j * np.pi * ((e5[jj] % lenq) * (2 * N // lenq)) / N)
        if not inverse:
            d0 = np.where(first, 1.0, -w)
            dp = np.where(first, w, 0.0)
            dm = np.where(first, 0.0, 1.0)
        else:                                    # [[1, w], [1, -w]]^-1 = 1/2 [[1, 1], [w^-1, -w^-1]]
            wi = np.conj(w)
            d0 = np.where(first, 0.5, -0.5 * wi)
            dp = np.where(first, 0.5, 0.0)
            dm = np.where(first, 0.0, 0.5 * wi)
        out.append({0: d0.astype(complex), lenh: dp.astype(complex), -lenh: dm.astype(complex)})
        ln *= 2
    return out


def diag_compose(B: dict, A: dict, n: int) -> dict:
    """Diagonals of B A: (B A x)[p] = sum_{d1, d2} B_d1[p] A_d2[p + d1] x[p + d1 + d2]."""
    out = {}
    for d1, b in B.items():
        for d2, a in A.items():
            d = d1 + d2
            d = (d + n // 2) % n - n // 2                     # signed representative
            out[d] = out.get(d, 0) + b * _rot(a, d1)
    return out


def fft_groups(N: int, levels: int, inverse: bool) -> list[dict]:
    """The merged matrices applied one per level.  CoeffToSlot (inverse=True) applies
    F_n^-1 first and F_2^-1 last; SlotToCoeff applies F_2 first.  The log2(n) stages split into
    `levels` consecutive groups (sizes differ by at most one, larger groups first)."""
    n = N // 2
    st = sfft_stages(N, inverse)
    order = st[::-1] if inverse else st
    L = len(order)
    sizes = [L // levels + (1 if i < L % levels else 0) for i in range(levels)]
    groups, k = [], 0
    for sz in sizes:
        M = order[k]
        for F in order[k + 1:k + sz]:
            M = diag_compose(F, M, n)
        groups.append(M)
        k += sz
    return groups


def bsgs_amounts(diags: dict, N: int) -> tuple[list[int], list[int]]:
    """Baby-step rotations (b h, b = 1 .. b1-1) and giant-step rotations (g b1 h, g != 0) of the
    baby-step giant-step evaluation of a merged group (amounts d = m h, m = g b1 + b)."""
    b1, h, ms = _bsgs_shape(diags)
    babies = sorted({m % b1 for m in ms} - {0})
    giants = sorted({m // b1 for m in ms} - {0})
    return [b * h for b in babies], [g * b1 * h for g in giants]


def _bsgs_shape(diags: dict):
    h = min(abs(d) for d in diags if d != 0)
    ms = sorted(d // h for d in diags)
    b1 = 1
    while b1 * b1 < len(ms):
        b1 *= 2
    return b1, h, ms


def _lintrans_bsgs(prm, ct, lv, diags: dict, name: str, keys: dict, const):
    """sum_d diag_d (.) rot_d(ct) = sum_g rot_{g b1 h}( sum_b rot_{-g b1 h}(diag_m) (.) rot_{b h}(ct) ),
    babies hoisted (one ModUp), one PMULT level at scale q_lv, then Rescale."""
    N, n = prm.N, prm.N // 2
    b1, h, ms = _bsgs_shape(diags)
    babies = sorted({m % b1 for m in ms} - {0})
    gs = [pow(5, (b * h) % n, 2 * N) for b in babies]
    rots = {0: ct}
    if gs:
        for b, r in zip(babies, ckks.hrot_hoisted(prm, ct, gs, lv, [keys[g] for g in gs])):
            rots[b] = r
    acc, rot_in, rot_g = None, [], []
    for g in sorted({m // b1 for m in ms}):
        inner = None
        for m in ms:
            if m // b1 != g:
                continue
            b = m % b1
            pt = const(f"{name}_g{g}_b{b}", lambda m=m, g=g: _pt_full(prm, _rot(diags[m * h], -g * b1 * h),
                                                                      float(prm.q[lv]), lv))
            t = ckks.pmult(prm, rots[b], pt, lv)
            inner = t if inner is None else ckks.hadd(prm, inner, t, lv)
        if g:
            rot_in.append(inner)
            rot_g.append(pow(5, (g * b1 * h) % n, 2 * N))
        else:
            acc = inner
    if rot_in:                                   # the giant steps' rotations share one ModDown
        r = hrot_sum(prm, rot_in, rot_g, lv, [keys[ga] for ga in rot_g])
        acc = r if acc is None else ckks.hadd(prm, acc, r, lv)
    return ckks.rescale(prm, acc, lv)


def _lintrans_plain(prm, ct, lv, diags: dict, keys: dict):
    """The textbook diagonal method (reading BOOT-P): sum_d diag_d (.) rot_d(ct) with one separate
    HROTATE per diagonal amount d and one PMULT per diagonal at scale q_lv, then Rescale -- no
    hoisting, no baby-step giant-step split, no shared ModDown.  The reference the GPU's schedule
    (hoisted baby steps, BOOT-H; giant steps summed before one ModDown, BOOT-G) is checked
    against by decryption (tests/test_oracle_boot.py, tests/test_gpu_boot.py)."""
    N, n = prm.N, prm.N // 2
    acc = None
    for d in sorted(diags):
        r = ct if d % n == 0 else ckks.hrot(prm, ct, pow(5, d % n, 2 * N), lv, keys[pow(5, d % n, 2 * N)])
        t = ckks.pmult(prm, r, _pt_full(prm, diags[d], float(prm.q[lv]), lv), lv)
        acc = t if acc is None else ckks.hadd(prm, acc, t, lv)
    return ckks.rescale(prm, acc, lv)


def plain_rotations(bp: "BootParams") -> list[int]:
    """Galois elements the plain (textbook) schedule needs beyond bp.rotations(): one per
    diagonal amount of every merged CoeffToSlot / SlotToCoeff group."""
    N = bp.prm.N
    gs = set()
    if bp.fft_levels:
        for grp in fft_groups(N, bp.fft_levels, inverse=True) + fft_groups(N, bp.fft_levels, inverse=False):
            gs |= {pow(5, d % (N // 2), 2 * N) for d in grp if d % (N // 2)}
    return sorted(gs - set(bp.rotations()))


def moddown(prm: ckks.Params, acc: np.ndarray, level: int) -> tuple:
    """Steps a7-a10 of the key-switch (Table 2, Z9) on a KeyIP output acc [2][E][N] (PQ_l,
    NTT form): (acc_c[Q] - NTT(BConv_{P->Q}(INTT(acc_c[P])))) P^-1."""
    q_ids = list(range(level + 1))
    p_ids = prm.p_ids
    pinv = [pow(prm.P % prm.moduli[i], -1, prm.moduli[i]) for i in q_ids]
    out = []
    for c in range(2):
        acc_p = ckks.intt(prm, acc[c][level + 1:], p_ids)
        conv = ckks.ntt(prm, ckks.bconv(prm, acc_p, p_ids, q_ids), q_ids)
        out.append(ckks.scalar_mul(prm, ckks.sub(prm, acc[c][: level + 1], conv, q_ids), pinv, q_ids))
    return out[0], out[1]


def hrot_sum(prm: ckks.Params, cts: list, gs: list, level: int, rotkeys: list) -> np.ndarray:
    """sum_k HROTATE(cts[k], gs[k]) with one ModDown (reading BOOT-G, the giant steps of a
    baby-step giant-step transform): the KeyIP outputs acc_k = KeyIP(ModUp(sigma_g(c1_k))) are
    summed in PQ_l and ModDown runs once:  (sum_k sigma_g(c0_k) + k0, k1), (k0, k1) =
    ModDown(sum_k acc_k).  Decrypts to the sum of the rotations (ModDown is linear up to its
    floor rounding), a different but equally valid ciphertext than summing separate HROTATEs."""
    ids = list(range(level + 1))
    E = level + 1 + prm.num_p
    ext = ids + prm.p_ids
    acc = np.zeros((2, E, prm.N), dtype=np.uint64)
    c0 = np.zeros((level + 1, prm.N), dtype=np.uint64)
    for ct, g, key in zip(cts, gs, rotkeys):
        tr = {}
        ckks.keyswitch(prm, ckks.automorphism_ntt(ct[1], g), level, key, trace=tr)
        for c in range(2):
            acc[c] = ckks.add(prm, acc[c], tr["acc"][c], ext)
        c0 = ckks.add(prm, c0, ckks.automorphism_ntt(ct[0], g), ids)
    k0, k1 = moddown(prm, acc, level)
    return np.stack([ckks.add(prm, c0, k0, ids), k1])


def fft_transform(bp: BootParams, ct: np.ndarray, lv: int, keys: dict, inverse: bool, tag: str, const=None,
                  plain: bool = False):
    """CoeffToSlot (inverse=True: slots <- P U^-1 slots) or SlotToCoeff (slots <- U P^-1 slots)
    as bp.fft_levels BSGS levels from level lv.  Returns (ct, lv - fft_levels).  `const(name,
    make)` supplies / records the plaintext diagonals (default: encode on the fly).  plain: the
    textbook diagonal method per level (_lintrans_plain)."""
    const = const or (lambda name, make: make())
    for k, grp in enumerate(fft_groups(bp.prm.N, bp.fft_levels, inverse)):
        if plain:
            ct = _lintrans_plain(bp.prm, ct, lv, grp, keys)
        else:
            ct = _lintrans_bsgs(bp.prm, ct, lv, grp, f"{tag}{k}", keys, const)
        lv -= 1
    return ct, lv


def _pt_full(prm: ckks.Params, slots: np.ndarray, scale: float, level: int) -> np.ndarray:
    ids = list(range(level + 1))
    m = ckks.encode_fft(prm.N, np.asarray(slots, dtype=complex), scale)
    return ckks.ntt(prm, ckks.reduce_signed(prm, m, ids), ids)


# --------------------------------------------------------------------------- ops

def modraise(prm: ckks.Params, ct: np.ndarray, level: int) -> np.ndarray:
    """ct [2][1][N] mod q_0 (NTT form) -> [2][level+1][N]: centred lift of each coefficient."""
    q0 = prm.q[0]
    ids = list(range(level + 1))
    out = []
    for c in range(2):
        coef = ckks.intt(prm, ct[c][0:1], [0])[0].astype(np.int64)
        signed = np.where(2 * coef > q0, coef - q0, coef)
        out.append(ckks.ntt(prm, ckks.reduce_signed(prm, signed, ids), ids))
    return np.stack(out)


def hsub(prm, a, b, level):
    ids = list(range(level + 1))
    return np.stack([ckks.sub(prm, a[0], b[0], ids), ckks.sub(prm, a[1], b[1], ids)])


def drop(ct: np.ndarray, level: int) -> np.ndarray:
    return np.ascontiguousarray(ct[:, : level + 1])


# --------------------------------------------------------------------------- keys

def boot_keys(bp: BootParams, s: np.ndarray, seed: int, plain: bool = False) -> dict:
    """Hybrid evaluation keys: 'relin' and one rotation key per Galois element of bp.rotations()
    (plain: also the textbook schedule's extra rotations, plain_rotations(bp))."""
    keys = {"relin": ckks.relin_key(bp.prm, s, seed)}
    gs = bp.rotations() + (plain_rotations(bp) if plain else [])
    for t, g in enumerate(gs):
        keys[g] = ckks.rot_key(bp.prm, s, g, seed + 1 + t)
    return keys


# --------------------------------------------------------------------------- bootstrapping

def bootstrap(bp: BootParams, ct0: np.ndarray, keys: dict, consts: dict | None = None, plain: bool = False,
              stop_after_cts: bool = False):
    """Bootstrap ct0 ([2][1][N], level 0).  Returns (ct, level, scale, consts) where the output
    decodes (at `scale` Delta_in / q_0) to the input's slots.  `consts` (plaintexts by name) are
    generated when None and returned, so another implementation can replay the same run.
    plain: the textbook schedule (separate HROTATEs, dense diagonal sums; reading BOOT-P) for
    both linear transforms -- the reference the GPU's hoisted / BOOT-G schedule is checked
    against by decryption.  stop_after_cts: return right after CoeffToSlot (ct, level, scale)."""
    prm, N, n, M = bp.prm, bp.prm.N, bp.n, bp.M
    gen = consts is None
    consts = {} if gen else consts
    q = prm.q

    def const(name, make):
        if gen:
            consts[name] = make()
        return consts[name]

    def rot(ct, g, lv):
        return ckks.hrot(prm, ct, g, lv, keys[g])

    # ModRaise: value (m + q_0 I) / q_0 at scale q_0
    L = bp.top
    ct = modraise(prm, ct0, L)
    scale = float(q[0])
    # SubSum: M x the subring projection
    for j in range(int(math.log2(M))):
        ct = ckks.hadd(prm, ct, rot(ct, pow(5, n << j, 2 * N), L), L)

    # reading BOOT-S: an exact x 2^k1 (PMULT by the integer constant, no level) raises the scale of
    # the ModRaised ciphertext before CoeffToSlot, so the key-switch noise its rotations add is
    # 2^k1 smaller relative to the message (at Set-B, full slots, it otherwise swamps it)
    k1, k2 = bp.boost
    if k1:
        ct = ckks.pmult(prm, ct, const("boost_cts", lambda: _const_int(prm, 1 << k1, L)), L)
        scale *= float(1 << k1)

    def lintrans_fft(ct, lv, inverse, tag):   # factored: fft_levels levels, BSGS per level
        return fft_transform(bp, ct, lv, keys, inverse, tag, const, plain=plain)

    def lintrans(ct, lv, A, tag):        # slots <- A slots (diagonal method), scale kept, one level
        # the n - 1 rotations of the same ciphertext are hoisted (one ModUp, reading BOOT-H);
        # plain: n - 1 separate HROTATEs
        gs = [pow(5, d, 2 * N) for d in range(1, n)]
        if plain:
            rots = [ct] + [rot(ct, g, lv) for g in gs]
        else:
            rots = [ct] + list(ckks.hrot_hoisted(prm, ct, gs, lv, [keys[g] for g in gs]))
        acc = None
        for d, dg in enumerate(_diagonals(A)):
            pt = const(f"{tag}_{d}", lambda dg=dg: _pt(bp, dg, float(q[lv]), lv))
            t = ckks.pmult(prm, rots[d], pt, lv)
            acc = t if acc is None else ckks.hadd(prm, acc, t, lv)
        return ckks.rescale(prm, acc, lv)

    if bp.fft_levels:
        W = None
        ct, lv = lintrans_fft(ct, L, True, "cts")                  # CoeffToSlot (bit-reversed slots)
    else:
        W = _xi_matrix(n)
        ct = lintrans(ct, L, np.linalg.inv(W) / M, "cts")          # CoeffToSlot
        lv = L - 1
    if stop_after_cts:
        return ct, lv, scale, consts
    cj = rot(ct, 2 * N - 1, lv)
    x1 = ckks.hadd(prm, ct, cj, lv)                                 # 2 Re(w)
    x2 = ckks.pmult(prm, hsub(prm, ct, cj, lv), const("mono_mi", lambda: _monomial(prm, N // 2, -1, lv)), lv)  # 2 Im(w)
    sx = 2.0 * scale                                                # value Re(w), Im(w) at scale 2 q_0 (x 2^k1)

    ds = bp.ds_sq                     # reading BOOT-S: EvalMod's first steps at scale ~q^2 (Double Rescale)

    def rs(ct, lv, m):                # divide by m primes: Rescale (1), Double Rescale (2, L138), both (3)
        if m == 1:
            return ckks.rescale(prm, ct, lv)
        ct = ckks.double_rescale(prm, ct, lv)
        return ckks.rescale(prm, ct, lv - 2) if m == 3 else ct

    def qq(lv, m):                    # the product of the m primes rs() divides by
        return math.prod(float(q[lv - i]) for i in range(m))

    def evalmod(x, lv, sx, tag):
        theta = 2 * math.pi / (1 << bp.r)
        m = 2 if ds else 1                                          # primes per rescale while at q^2
        S = qq(lv, m) if ds else float(q[lv])                       # y's scale after the theta product
        m_th = 2 if (k1 or ds) else 1   # a boosted input needs q_lv q_lv-1 for theta to keep ~52 bits
        y1 = rs(ckks.pmult(prm, x, const(f"{tag}theta", lambda: _pt(bp, np.full(n, theta), S * qq(lv, m_th) / sx, lv)),
                           lv), lv, m_th)
        lv -= m_th
        sc = {1: S}
        pw = {1: (y1, lv)}

        def mul(a, b):                                              # y^a y^b, levels aligned, rescaled
            (ca, la), (cb, lb) = pw[a], pw[b]
            l0 = min(la, lb)
            prod = ckks.hmult(prm, drop(ca, l0), drop(cb, l0), l0, keys["relin"])
            pw[a + b] = (rs(prod, l0, m), l0 - m)
            sc[a + b] = sc[a] * sc[b] / qq(l0, m)
        mul(1, 1)
        mul(2, 1)
        mul(2, 2)
        mul(4, 1)
        mul(4, 2)
        mul(4, 3)
        lt = min(pw[k][1] for k in pw)                              # common level of the terms
        St = qq(lt, m)                                              # their common scale
        E = None
        for k in range(1, D_TAYLOR + 1):
            ck, lk = pw[k]
            coef = (1j ** k) / math.factorial(k)
            pt = const(f"{tag}c{k}", lambda coef=coef, lk=lk, k=k: _pt(bp, np.full(n, coef), St * qq(lk, m) / sc[k], lk))
            term = drop(rs(ckks.pmult(prm, ck, pt, lk), lk, m), lt - m)
            E = term if E is None else ckks.hadd(prm, E, term, lt - m)
        lv = lt - m
        E = ckks.padd(prm, E, const(f"{tag}c0", lambda: _pt(bp, np.ones(n), St, lv)), lv)
        s_e = St
        for i in range(bp.r):                                       # E <- E^2: exp(2 pi i t)
            # ds squarings at ~q^2, then one dividing by 3 primes back to ~q, then single ones
            mi = (2 if i < ds else 3 if i == ds else 1) if ds else 1
            E = rs(ckks.hmult(prm, E, E, lv, keys["relin"]), lv, mi)
            s_e = s_e * s_e / qq(lv, mi)
            lv -= mi
        cE = rot(E, 2 * N - 1, lv)
        Dm = hsub(prm, E, cE, lv)                                   # 2 i sin(2 pi t)
        k = -1j / (4 * math.pi)
        f = ckks.rescale(prm, ckks.pmult(prm, Dm, const(f"{tag}sin", lambda: _pt(bp, np.full(n, k), float(q[lv]), lv)), lv), lv)
        return f, lv - 1, s_e

    f1, lv1, s1 = evalmod(x1, lv, sx, "re")
    f2, lv2, s2 = evalmod(x2, lv, sx, "im")
    assert (lv1, s1) == (lv2, s2)
    lv = lv1
    w = ckks.hadd(prm, f1, ckks.pmult(prm, f2, const("mono_i", lambda: _monomial(prm, N // 2, 1, lv)), lv), lv)
    if k2:                                                          # the same boost before SlotToCoeff
        w = ckks.pmult(prm, w, const("boost_stc", lambda: _const_int(prm, 1 << k2, lv)), lv)
        s1 *= float(1 << k2)
    if bp.fft_levels:
        out, lo = lintrans_fft(w, lv, False, "stc")                 # SlotToCoeff
        return out, lo, s1, consts
    out = lintrans(w, lv, W, "stc")                                 # SlotToCoeff
    return out, lv - 1, s1, consts


def encrypt_sparse(bp: BootParams, z: np.ndarray, delta: float, s: np.ndarray, seed: int) -> np.ndarray:
    """Encrypt n slots (tiled to the full N/2) at level 0, scale delta: ct [2][1][N]."""
    m = ckks.encode(bp.prm.N, np.tile(z, bp.M), delta)
    return ckks.encrypt(bp.prm, m, s, 0, seed)


def decode_sparse(bp: BootParams, ct: np.ndarray, level: int, scale: float, s: np.ndarray) -> np.ndarray:
    m = ckks.crt_centered(bp.prm, ckks.decrypt_residues(bp.prm, ct, s, level), list(range(level + 1)))
    return ckks.decode(bp.prm.N, m, scale)[: bp.n]


def make_consts(bp: BootParams) -> dict:
    """The plaintext constants bootstrap(bp, ...) generates (see dry_run)."""
    return dry_run(bp)[2]


def dry_run(bp: BootParams) -> tuple:
    """(output level, output scale, plaintext constants) of bootstrap(bp, ...), without its ciphertext arithmetic:
    the schedule's levels and scales are data-independent, so the run is replayed with every
    ciphertext operation replaced by a shape-preserving stand-in (used to give the GPU the real
    constants at Set-B, where running the oracle's bootstrap itself would take hours)."""
    N = bp.prm.N
    z = lambda L: np.zeros((2, L + 1, N), dtype=np.uint64)
    lim = lambda ct, lv: np.ascontiguousarray(ct[:, : lv + 1])
    stand_in = {
        "hrot": lambda prm, ct, g, lv, key: ct,
        "hrot_hoisted": lambda prm, ct, gs, lv, keys: [ct] * len(gs),
        "hmult": lambda prm, a, b, lv, relin, mode="fast": a,
        "pmult": lambda prm, ct, pt, lv: ct,
        "hadd": lambda prm, a, b, lv: a,
        "padd": lambda prm, ct, pt, lv: ct,
        "rescale": lambda prm, ct, lv, mode="fast": lim(ct, lv - 1),
        "double_rescale": lambda prm, ct, lv, mode="fast": lim(ct, lv - 2),
    }
    saved_ckks = {k: getattr(ckks, k) for k in stand_in}
    g = globals()
    saved_boot = {k: g[k] for k in ("modraise", "hrot_sum", "hsub")}
    try:
        for k, f in stand_in.items():
            setattr(ckks, k, f)
        g["modraise"] = lambda prm, ct, L: z(L)
        g["hrot_sum"] = lambda prm, cts, gs, lv, keys: cts[0]
        g["hsub"] = lambda prm, a, b, lv: a
        _, lv, scale, consts = bootstrap(bp, z(0), collections.defaultdict(lambda: None))
    finally:
        for k, f in saved_ckks.items():
            setattr(ckks, k, f)
        g.update(saved_boot)
    return lv, scale, consts
