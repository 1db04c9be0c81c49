"""CPU ORACLE of KLSS key-switching (Neo's default method) -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / ``--impl reference``
legs may import this module.  It shares no code with the CUDA path.

What the paper fixes (PAPER.md, "L<n>"):
* six steps ModUp, NTT, IP, INTT, Recover Limbs, ModDown (L155, Fig. 5);
* ModUp maps each of the beta digits (alpha limbs) to R_T, alpha' limbs of WordSize_T
  (Eq. 3); IP multiplies with beta~ x beta keys and turns beta groups into beta~
  groups (L175; Alg. 3 L359-382 / Alg. 4: c~_i,k += c_j,k * evk_i,j,k);
  Recover Limbs brings the limbs back to R_PQ (L175), ModDown is Hybrid's (Table 2);
* alpha' >= ceil(log(2 beta N B B~) / WordSize_T) for correctness/security (Eq. 4);
* kernel complexities (Table 2): ModUp beta alpha alpha', IP beta beta~ alpha',
  INTT 2 beta~ alpha', Recover Limbs 2 alpha' (l + alpha), ModDown 2 (l alpha + l).

Readings where the paper is silent (DESIGN.md "KLSS readings" K1-K6):
K1 the key of group i is the Hybrid key reduced modulo the group modulus:
   e_{i,j,c} = [evk_{j,c}]_{P~_i} in [0, P~_i), P~_i = product of the alpha~ limbs of group
   i of PQ_L (groups: consecutive alpha~ limbs of q_0..q_L, p_0..p_K); B~ = max P~_i.
K2 ModUp is Algorithm 1 (non-centred, Z7): the digit's integer x_j = sum y_i qhat_i lies in
   [0, alpha Q_j): B = alpha max_j Q_j.
K3 so sum_j x_j e_{i,j,c} is an integer polynomial with |coefficients| < beta N B B~; it is
   computed exactly in R_T when T > 2 beta N B B~ (Eq. 4).  One guard bit: alpha' is the
   smallest count of T primes with T > 4 beta N B B~, so the centred lift is robust.
K4 Recover Limbs = the exact centred CRT lift from T, reduced modulo each limb of group i.
   Because e = evk (mod every limb of group i) and x_j = Hybrid's ModUp integer, the
   recovered limbs equal Hybrid's KeyIP output acc exactly, so KLSS KeySwitch == Hybrid
   KeySwitch bit for bit (pinned in tests/test_oracle_klss.py).
K5 ModDown on the recovered (coefficient-form) limbs: (acc_Q - BConv_{P->Q}(acc_P)) P^-1,
   then NTT over Q_l (Z9; by linearity identical to Hybrid's NTT-domain combine).
K6 T primes: the Z4 rule at WordSize_T bits (Table 4: 48 for Set-C; Fig. 16 evaluates
   36, 48, 64).  When WordSize_T equals the Q/P word size the sequence continues after the Q
   and P primes; otherwise it starts afresh at the top of the WordSize_T range (disjoint from
   Q and P by bit length).
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field

import numpy as np

from . import _core, ckks
from ._core import ptr, u64arr


@dataclass
class KlssParams:
    """A Hybrid parameter set plus the KLSS extras (alpha~, WordSize_T, T primes, groups)."""
    base: ckks.Params
    alpha_t: int
    word_bits_t: int = 36
    t: list = field(default_factory=list)
    groups: list = field(default_factory=list)

    def __post_init__(self):
        b = self.base
        assert b.word_bits <= self.word_bits_t <= 64
        ext = list(range(b.num_q)) + b.p_ids                              # PQ_L limb ids
        self.groups = [ext[i:i + self.alpha_t] for i in range(0, len(ext), self.alpha_t)]
        self.bound = self.ip_bound()
        if self.word_bits_t == b.word_bits:                               # K6
            cand = ckks.gen_primes(b.log_n, self.word_bits_t, b.num_q + b.num_p + 64)[b.num_q + b.num_p:]
        else:
            cand = ckks.gen_primes(b.log_n, self.word_bits_t, 64)
        T, k = 1, 0
        while T <= 4 * self.bound:                                        # K3 (Eq. 4 + guard bit)
            T *= cand[k]
            k += 1
        self.t = cand[:k]
        self.T = T
        self.alpha_p = k                                                  # alpha'
        self.t_ids = list(range(b.num_q + b.num_p, b.num_q + b.num_p + k))
        self.moduli = b.moduli + self.t
        self.psi = b.psi + [ckks.min_psi(t, b.N) for t in self.t]
        self.N = b.N

    @property
    def beta_t(self) -> int:                                              # beta~
        return len(self.groups)

    def ip_bound(self) -> int:
        """beta N B B~ of Eq. 4 with B = alpha max Q_j (K2) and B~ = max P~_i (K1)."""
        b = self.base
        B = b.alpha * max(math.prod(b.moduli[i] for i in d) for d in b.digits(b.max_level))
        Bt = max(math.prod(b.moduli[i] for i in g) for g in self.groups)
        return b.dnum * b.N * B * Bt

    def groups_at(self, level: int):
        """(group index, limb ids of the group present in PQ_level) for groups with any."""
        present = set(range(level + 1)) | set(self.base.p_ids)
        out = []
        for i, g in enumerate(self.groups):
            ids = [t for t in g if t in present]
            if ids:
                out.append((i, ids))
        return out


def set_c_t36() -> KlssParams:
    """Table 4 Set-C (L504-517): N=2^16, L=35, WordSize 36, dnum=9 (P: alpha = 4 limbs, Z3),
    alpha~ = 5, with WordSize_T = 36 (K6)."""
    return KlssParams(ckks.Params(16, 36, 4, 9), alpha_t=5)


def set_c() -> KlssParams:
    """Table 4 Set-C as printed (L504-517): N=2^16, L=35, WordSize 36, WordSize_T = 48, dnum=9,
    alpha~ = 5 (P: alpha = 4 limbs, Z3)."""
    return KlssParams(ckks.Params(16, 36, 4, 9), alpha_t=5, word_bits_t=48)


def tiny48() -> KlssParams:
    """tiny() with 48-bit T primes (WordSize_T = 48, K6)."""
    return KlssParams(ckks.Params(12, 6, 2, 3), alpha_t=3, word_bits_t=48)


def tiny() -> KlssParams:
    """Small KLSS configuration for CPU pins: N=2^12, 6 Q limbs, dnum=3 (alpha=2, 2 P limbs),
    alpha~ = 3."""
    return KlssParams(ckks.Params(12, 6, 2, 3), alpha_t=3)


# --------------------------------------------------------------------------- exact CRT

def _words(x: int, W: int) -> list:
    return [(x >> (64 * w)) & ((1 << 64) - 1) for w in range(W)]


def crt_exact(moduli_in, x: np.ndarray, moduli_out, centred: bool) -> np.ndarray:
    """The CRT lift of x[n_in][N] (residues mod moduli_in) to the integer in [0, Q) (or the
    centred (-Q/2, Q/2]), reduced modulo each of moduli_out.  Exact (multi-word integers)."""
    qs = [int(q) for q in moduli_in]
    Q = math.prod(qs)
    W = (Q.bit_length() + len(qs).bit_length() + 1 + 63) // 64
    qhat = [Q // q for q in qs]
    qhat_inv = [pow(h % q, -1, q) for h, q in zip(qhat, qs)]
    flat = u64arr([w for h in qhat for w in _words(h, W)])
    x = np.ascontiguousarray(x, dtype=np.uint64)
    n = x.shape[1]
    out = np.empty((len(moduli_out), n), dtype=np.uint64)
    _core.lib().or_crt_exact(ptr(x), ptr(u64arr(qs)), ptr(u64arr(qhat_inv)), len(qs), ptr(flat),
                             ptr(u64arr(_words(Q, W))), W, ptr(u64arr(moduli_out)), len(moduli_out),
                             ptr(out), n, 1 if centred else 0)
    return out


# --------------------------------------------------------------------------- key

def klss_key(kp: KlssParams, evk: np.ndarray) -> np.ndarray:
    """K1: e[c][i][j][k] = NTT_T( [evk_{j,c}]_{P~_i} mod t_k ),  shape [2][beta~][dnum][alpha'][N].
    evk is the Hybrid key [dnum][2][num_q+num_p][N] (NTT form, Z8)."""
    b = kp.base
    out = np.empty((2, kp.beta_t, b.dnum, kp.alpha_p, b.N), dtype=np.uint64)
    for i, g in enumerate(kp.groups):
        for j in range(b.dnum):
            for c in range(2):
                coef = ckks.intt(b, evk[j, c][g], g)                       # group limbs, coeff form
                e = crt_exact([b.moduli[t] for t in g], coef, kp.t, centred=False)
                out[c, i, j] = ckks.ntt(kp, e, kp.t_ids)
    return out


# --------------------------------------------------------------------------- key-switch

def keyswitch(kp: KlssParams, d: np.ndarray, level: int, ekey: np.ndarray, trace: dict | None = None):
    """KLSS KeySwitch of d ([level+1][N], NTT form) with the key of klss_key; returns (k0, k1)
    in NTT form over Q_level.  Steps of L155 / Fig. 5 in order."""
    b = kp.base
    q_ids = list(range(level + 1))
    digits = b.digits(level)
    d_coef = ckks.intt(b, d, q_ids)                                       # INTT of d
    up = []
    for dj in digits:                                                     # Mod Up (Eq. 3, Alg. 1)
        x = ckks.bconv(kp, d_coef[dj[0]:dj[-1] + 1], dj, kp.t_ids)
        up.append(ckks.ntt(kp, x, kp.t_ids))                              # NTT over T
    groups = kp.groups_at(level)
    rec = {0: {}, 1: {}}
    for i, ids in groups:
        for c in range(2):
            acc = np.zeros((kp.alpha_p, b.N), dtype=np.uint64)            # IP (Alg. 3): c~_ik += c_jk evk_ijk
            for j in range(len(digits)):
                acc = ckks.add(kp, acc, ckks.mul(kp, up[j], ekey[c, i, j], kp.t_ids), kp.t_ids)
            acc_coef = ckks.intt(kp, acc, kp.t_ids)                       # INTT over T
            r = crt_exact(kp.t, acc_coef, [b.moduli[t] for t in ids], centred=True)   # Recover Limbs (K4)
            for k, t in enumerate(ids):
                rec[c][t] = r[k]
            if trace is not None:
                trace.setdefault("ip_coef", []).append(acc_coef)
    out = []
    p_ids = b.p_ids
    pinv = [pow(b.P % b.moduli[i], -1, b.moduli[i]) for i in q_ids]
    for c in range(2):                                                    # Mod Down (K5, Z9)
        acc_p = np.stack([rec[c][t] for t in p_ids])
        conv = ckks.bconv(b, acc_p, p_ids, q_ids)
        acc_q = np.stack([rec[c][t] for t in q_ids])
        z = ckks.scalar_mul(b, ckks.sub(b, acc_q, conv, q_ids), pinv, q_ids)
        out.append(ckks.ntt(b, z, q_ids))
        if trace is not None:
            trace.setdefault("acc_coef", []).append(np.stack([rec[c][t] for t in q_ids + p_ids]))
    return out[0], out[1]


def hmult(kp: KlssParams, ct_a, ct_b, level, ekey):
    """HMULT (L132) with KLSS relinearisation."""
    b = kp.base
    ids = list(range(level + 1))
    d0, d1, d2 = ckks.tensor(b, ct_a, ct_b, level)
    k0, k1 = keyswitch(kp, d2, level, ekey)
    return np.stack([ckks.add(b, d0, k0, ids), ckks.add(b, d1, k1, ids)])


def hrot(kp: KlssParams, ct, g, level, ekey):
    """HROTATE (L136) with a KLSS rotation key."""
    b = kp.base
    ids = list(range(level + 1))
    c0 = ckks.automorphism_ntt(ct[0], g)
    k0, k1 = keyswitch(kp, ckks.automorphism_ntt(ct[1], g), level, ekey)
    return np.stack([ckks.add(b, c0, k0, ids), k1])
