"""CPU ORACLE of Neo's Hybrid key-switching hot path -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / ``--impl reference``
legs may import this module.  It shares no code, header, table or constant generator
with the CUDA path; both sides receive their random inputs from ``synth``.

What it computes (citations are /root/reference/PAPER.md lines, "L<n>"; readings of
silent/garbled passages are SURVEY.md §8(c) Z1-Z23, listed in DESIGN.md):

* parameters    -- Table 1 (L84-105), Table 4 (L504-517); prime rule Z4, psi rule Z5,
                   alpha = ceil((L+1)/dnum) (L98), beta = ceil((l+1)/alpha) (L99)
* NTT / INTT    -- definitional a_hat[i] = a(psi^(2i+1)) (natural order, Z6); the
                   O(N log N) mode is a textbook FFT pinned against the definition
* BConv         -- Algorithm 1 (L296-319), non-centred (Z7)
* KeySwitch     -- Hybrid method, Table 2 (L140-149), Eq. 2 (L161-163), Fig. 5 (L288):
                   INTT -> ModUp BConv -> NTT -> KeyIP (Alg. 3) -> INTT ->
                   ModDown BConv -> NTT -> (acc - conv) * P^-1   (Z8, Z9)
* HMULT         -- L132: d0 = a0 b0, d1 = a0 b1 + a1 b0, d2 = a1 b1; KS(d2) added to d0, d1
* HROTATE       -- L136, L184: automorphism then KS with the rotation key (Z11)
* Rescale       -- L137: divide by the last prime, floor rounding (Z10)
* Double Rescale-- L138, L151: divide by the last two primes, floor (reading "DS")
* PMULT / HADD / PADD -- L133-135: element-wise products and sums in the NTT domain
* encode/decode, keygen, encrypt/decrypt -- L121-130 with the standard sign (Z1),
                   gadget of Z8, distributions of Z12 (host-only, never on the GPU path)

Parity pins: tests/test_oracle_*.py (closed forms, invariants, big-integer CRT,
brute force) -- see DESIGN.md "Oracle pins".  Nothing here is "parity unpinned".

Polynomials are numpy uint64 arrays [limbs][N] of canonical residues; a limb id
indexes the concatenated basis q_0..q_{num_q-1}, p_0..p_{num_p-1}.
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field

import numpy as np

import synth
from . import _core
from ._core import ptr, u64arr

# --------------------------------------------------------------------------- primes

_MR_BASES = (2, 3, 5, 7, 11, 13, 17, 19, 23, 29, 31, 37)


def is_prime(n: int) -> bool:
    """Deterministic Miller-Rabin (the 12 prime bases are exact for n < 3.3e24)."""
    if n < 2:
        return False
    for b in _MR_BASES:
        if n % b == 0:
            return n == b
    d, r = n - 1, 0
    while d % 2 == 0:
        d //= 2
        r += 1
    for b in _MR_BASES:
        x = pow(b, d, n)
        if x in (1, n - 1):
            continue
        for _ in range(r - 1):
            x = x * x % n
            if x == n - 1:
                break
        else:
            return False
    return True


def gen_primes(log_n: int, word_bits: int, count: int) -> list[int]:
    """Z4: q = k*2N + 1 for k from floor((2^W - 1)/2N) downward, bit-length W, prime."""
    two_n = 2 << log_n
    k = ((1 << word_bits) - 1) // two_n
    out = []
    while len(out) < count:
        q = k * two_n + 1
        if q.bit_length() != word_bits:
            raise ValueError("ran out of W-bit NTT primes")
        if is_prime(q):
            out.append(q)
        k -= 1
    return out


def min_psi(q: int, n: int) -> int:
    """Z5: the minimum primitive 2N-th root of unity mod q (psi^N = -1)."""
    assert (q - 1) % (2 * n) == 0
    x = 2
    while True:
        psi0 = pow(x, (q - 1) // (2 * n), q)
        if pow(psi0, n, q) == q - 1:
            break
        x += 1
    # every primitive 2N-th root is psi0^k, k odd
    best, cur, sq = psi0, psi0, psi0 * psi0 % q
    for _ in range(n - 1):
        cur = cur * sq % q
        if cur < best:
            best = cur
    return best


# --------------------------------------------------------------------------- params

@dataclass
class Params:
    """Table 1 / Table 4 parameters; moduli[id] for id in 0..num_q+num_p-1."""
    log_n: int
    num_q: int
    num_p: int
    dnum: int
    word_bits: int = 36
    q: list = field(default_factory=list)
    p: list = field(default_factory=list)

    def __post_init__(self):
        primes = gen_primes(self.log_n, self.word_bits, self.num_q + self.num_p)
        self.q = primes[: self.num_q]
        self.p = primes[self.num_q:]
        self.N = 1 << self.log_n
        self.moduli = self.q + self.p
        self.psi = [min_psi(m, self.N) for m in self.moduli]
        self.alpha = -(-self.num_q // self.dnum)                 # L98
        if -(-self.num_q // self.alpha) != self.dnum:
            raise ValueError("every digit must be non-empty: ceil(num_q/alpha) == dnum")
        self.P = math.prod(self.p)
        self.max_level = self.num_q - 1

    @property
    def p_ids(self) -> list[int]:
        return list(range(self.num_q, self.num_q + self.num_p))

    def beta(self, level: int) -> int:
        return -(-(level + 1) // self.alpha)                     # L99

    def digits(self, level: int) -> list[list[int]]:
        """Z8: digit j holds the raw limbs D_j = {j*alpha, ..., min((j+1)alpha, l+1)-1}."""
        return [list(range(j * self.alpha, min((j + 1) * self.alpha, level + 1)))
                for j in range(self.beta(level))]


def tiny() -> Params:
    """BASELINE config 1: N=2^12, 3 Q limbs + 1 P limb, dnum=1."""
    return Params(12, 3, 1, 1)


def tiny_dnum3() -> Params:
    """SURVEY Z14 precision variant: N=2^12, 3 Q + 1 P, dnum=3 (alpha=1)."""
    return Params(12, 3, 1, 3)


def set_b() -> Params:
    """Table 4 Set-B (L504-517): N=2^16, 36 Q limbs (Z2), 12 P limbs (Z3), dnum=3."""
    return Params(16, 36, 12, 3)


# --------------------------------------------------------------------------- NTT

def ntt(prm: Params, x: np.ndarray, ids, mode: str = "fast") -> np.ndarray:
    """Per-limb negacyclic NTT of x[k] mod moduli[ids[k]] (returns a new array)."""
    L = _core.lib()
    x = np.ascontiguousarray(x, dtype=np.uint64)
    ids = list(ids)
    assert x.shape == (len(ids), prm.N)
    if mode == "def":
        out = np.empty_like(x)
        for k, i in enumerate(ids):
            L.or_ntt_def(ptr(x[k]), ptr(out[k]), prm.N, prm.moduli[i], prm.psi[i])
        return out
    out = x.copy()
    L.or_ntt_fast_batch(ptr(out), len(ids), prm.N, ptr(u64arr([prm.moduli[i] for i in ids])),
                        ptr(u64arr([prm.psi[i] for i in ids])), 0)
    return out


def intt(prm: Params, x: np.ndarray, ids, mode: str = "fast") -> np.ndarray:
    L = _core.lib()
    x = np.ascontiguousarray(x, dtype=np.uint64)
    ids = list(ids)
    assert x.shape == (len(ids), prm.N)
    if mode == "def":
        out = np.empty_like(x)
        for k, i in enumerate(ids):
            L.or_intt_def(ptr(x[k]), ptr(out[k]), prm.N, prm.moduli[i], prm.psi[i])
        return out
    out = x.copy()
    L.or_ntt_fast_batch(ptr(out), len(ids), prm.N, ptr(u64arr([prm.moduli[i] for i in ids])),
                        ptr(u64arr([prm.psi[i] for i in ids])), 1)
    return out


# --------------------------------------------------------------------------- element-wise

def _vec(fn, a, b, m):
    out = np.empty_like(a)
    getattr(_core.lib(), fn)(ptr(a), ptr(b), ptr(out), a.size, m)
    return out


def mul(prm, a, b, ids):
    """ModMUL per limb (L268, L456)."""
    return np.stack([_vec("or_vec_mulmod", np.ascontiguousarray(a[k]), np.ascontiguousarray(b[k]),
                          prm.moduli[i]) for k, i in enumerate(ids)])


def add(prm, a, b, ids):
    """ModADD per limb."""
    return np.stack([_vec("or_vec_addmod", np.ascontiguousarray(a[k]), np.ascontiguousarray(b[k]),
                          prm.moduli[i]) for k, i in enumerate(ids)])


def sub(prm, a, b, ids):
    return np.stack([_vec("or_vec_submod", np.ascontiguousarray(a[k]), np.ascontiguousarray(b[k]),
                          prm.moduli[i]) for k, i in enumerate(ids)])


def scalar_mul(prm, a, scalars, ids):
    L = _core.lib()
    out = np.empty_like(a)
    for k, i in enumerate(ids):
        src = np.ascontiguousarray(a[k])
        dst = np.empty_like(src)
        L.or_vec_scalar_mulmod(ptr(src), int(scalars[k]) % prm.moduli[i], ptr(dst), src.size,
                               prm.moduli[i])
        out[k] = dst
    return out


def reduce_signed(prm, coeffs, ids) -> np.ndarray:
    """Signed integer coefficients (int64 or Python ints) -> residues per limb."""
    c = np.asarray(coeffs)
    out = np.empty((len(ids), prm.N), dtype=np.uint64)
    for k, i in enumerate(ids):
        m = prm.moduli[i]
        if c.dtype == object:
            out[k] = np.array([int(v) % m for v in c], dtype=np.uint64)
        else:
            out[k] = np.mod(c.astype(np.int64), m).astype(np.uint64)
    return out


# --------------------------------------------------------------------------- BConv

def bconv_tables(prm: Params, src_ids, dst_ids):
    """qhat_i = prod_{i' != i} q_i' ; qhat_i^-1 mod q_i ; qhat_i mod t  (Alg. 1 line 4)."""
    qs = [prm.moduli[i] for i in src_ids]
    qin = math.prod(qs)
    qhat = [qin // qi for qi in qs]
    qhat_inv = [pow(qh % qi, -1, qi) for qh, qi in zip(qhat, qs)]
    qhat_mod_t = [[qh % prm.moduli[t] for t in dst_ids] for qh in qhat]
    return qs, qhat_inv, qhat_mod_t


def bconv(prm: Params, x: np.ndarray, src_ids, dst_ids) -> np.ndarray:
    """Algorithm 1 (L296-319) on coefficient-form limbs x[len(src_ids)][N]."""
    src_ids, dst_ids = list(src_ids), list(dst_ids)
    qs, qhat_inv, qhat_mod_t = bconv_tables(prm, src_ids, dst_ids)
    x = np.ascontiguousarray(x, dtype=np.uint64)
    out = np.empty((len(dst_ids), prm.N), dtype=np.uint64)
    flat = u64arr([v for row in qhat_mod_t for v in row])
    _core.lib().or_bconv(ptr(x), len(src_ids), ptr(out), len(dst_ids), prm.N, ptr(u64arr(qs)),
                         ptr(u64arr(qhat_inv)), ptr(flat), ptr(u64arr([prm.moduli[t] for t in dst_ids])))
    return out


# --------------------------------------------------------------------------- key-switch

def keyswitch(prm: Params, d: np.ndarray, level: int, evk: np.ndarray, mode: str = "fast",
              trace: dict | None = None):
    """Hybrid KeySwitch (Table 2, Eq. 2, Fig. 5), steps a3-a10.

    d   : [level+1][N] NTT form (mod q_0..q_level)
    evk : [dnum][2][num_q+num_p][N] NTT form (key digits of Z8)
    returns (k0, k1), each [level+1][N] NTT form, with k0 + k1*s ~= d * s'.
    """
    N = prm.N
    q_ids = list(range(level + 1))
    p_ids = prm.p_ids
    ext = q_ids + p_ids                                    # basis of PQ_l
    pos = {t: k for k, t in enumerate(ext)}
    d = np.ascontiguousarray(d, dtype=np.uint64)
    d_coef = intt(prm, d, q_ids, mode)                     # a3 INTT
    acc = np.zeros((2, len(ext), N), dtype=np.uint64)
    for j, dj in enumerate(prm.digits(level)):
        targets = [t for t in ext if t not in dj]
        up = bconv(prm, d_coef[dj[0]:dj[-1] + 1], dj, targets)   # a4 ModUp BConv
        up_ntt = ntt(prm, up, targets, mode)                      # a5 NTT
        dhat = np.empty((len(ext), N), dtype=np.uint64)
        for t in dj:
            dhat[pos[t]] = d[t]                                   # digit's own limbs: d_t itself
        for k, t in enumerate(targets):
            dhat[pos[t]] = up_ntt[k]
        if trace is not None:
            trace.setdefault("modup", []).append(up)
            trace.setdefault("dhat", []).append(dhat)
        for c in range(2):                                        # a6 KeyIP (Alg. 3)
            prod_ = mul(prm, dhat, evk[j, c][ext], ext)
            acc[c] = add(prm, acc[c], prod_, ext)
    out = []
    p_pos = [pos[t] for t in p_ids]
    pinv = [pow(prm.P % prm.moduli[i], -1, prm.moduli[i]) for i in q_ids]
    for c in range(2):
        acc_p = intt(prm, acc[c][p_pos], p_ids, mode)            # a7 INTT of the P part
        conv = bconv(prm, acc_p, p_ids, q_ids)                    # a8 ModDown BConv
        conv_ntt = ntt(prm, conv, q_ids, mode)                    # a9 NTT
        diff = sub(prm, acc[c][: level + 1], conv_ntt, q_ids)     # a10 (acc - conv) * P^-1
        out.append(scalar_mul(prm, diff, pinv, q_ids))
        if trace is not None:
            trace.setdefault("acc", []).append(acc[c].copy())
            trace.setdefault("moddown", []).append(conv)
    return out[0], out[1]


def tensor(prm: Params, ct_a: np.ndarray, ct_b: np.ndarray, level: int):
    """HMULT tensor product (L132): d0 = a0 b0, d1 = a0 b1 + a1 b0, d2 = a1 b1 (NTT form)."""
    ids = list(range(level + 1))
    a0, a1, b0, b1 = ct_a[0], ct_a[1], ct_b[0], ct_b[1]
    d0 = mul(prm, a0, b0, ids)
    d1 = add(prm, mul(prm, a0, b1, ids), mul(prm, a1, b0, ids), ids)
    d2 = mul(prm, a1, b1, ids)
    return d0, d1, d2


def hmult(prm, ct_a, ct_b, level, relin, mode="fast"):
    """HMULT (L132): tensor, KeySwitch(d2), add to (d0, d1).  No rescale (Z22)."""
    ids = list(range(level + 1))
    d0, d1, d2 = tensor(prm, ct_a, ct_b, level)
    k0, k1 = keyswitch(prm, d2, level, relin, mode)
    return np.stack([add(prm, d0, k0, ids), add(prm, d1, k1, ids)])


def galois_index_map(N: int, g: int) -> np.ndarray:
    """NTT-domain form of X -> X^g: out[i] = in[(g*i + (g-1)/2) mod N] (natural order, Z6).

    a_hat[i] = a(psi^(2i+1)), so sigma_g(a)_hat[i] = a(psi^(g(2i+1))) = a_hat[i'] with
    2i'+1 = g(2i+1) mod 2N.
    """
    i = np.arange(N, dtype=np.int64)
    return (g * i + (g - 1) // 2) % N


def automorphism_ntt(x: np.ndarray, g: int) -> np.ndarray:
    """AUTO kernel (L268-270) in the NTT domain, per limb."""
    return np.ascontiguousarray(x[..., galois_index_map(x.shape[-1], g)])


def automorphism_coeff(prm: Params, x: np.ndarray, ids, g: int) -> np.ndarray:
    """Definition: sigma_g(a)(X) = a(X^g); coefficient k moves to k*g mod 2N, negated past N."""
    N = prm.N
    out = np.zeros_like(x)
    for k in range(N):
        e = (k * g) % (2 * N)
        for r, i in enumerate(ids):
            m = prm.moduli[i]
            v = int(x[r, k])
            out[r, e % N] = (m - v) % m if e >= N else v
    return out


def hrot(prm, ct, g, level, rotkey, mode="fast"):
    """HROTATE (L136): sigma_g on (c0, c1), KS(sigma_g(c1)) with KSGen(s, sigma_g(s)) (L184)."""
    ids = list(range(level + 1))
    c0 = automorphism_ntt(ct[0], g)
    c1 = automorphism_ntt(ct[1], g)
    k0, k1 = keyswitch(prm, c1, level, rotkey, mode)
    return np.stack([add(prm, c0, k0, ids), k1])


def hrot_hoisted(prm, ct, gs, level, rotkeys, mode="fast"):
    """Hoisted HROTATE: for each g, sigma_g(c0 + k0', k1') with
    (k0', k1') = KeySwitch(c1) under the key sigma_{g^-1}(rotkey_g).  The key-switch input
    c1 is the same for every g, so an implementation may run its ModUp once."""
    out = []
    ids = list(range(level + 1))
    for g, key in zip(gs, rotkeys):
        ginv = pow(g, -1, 2 * prm.N)
        kp = automorphism_ntt(key, ginv)
        k0, k1 = keyswitch(prm, ct[1], level, kp, mode)
        pre = np.stack([add(prm, ct[0], k0, ids), k1])
        out.append(automorphism_ntt(pre, g))
    return np.stack(out)


def rescale(prm, ct, level, mode="fast"):
    """Rescale (L137), floor reading Z10: c'_i = (c_i - ([c_l]_{q_l} mod q_i)) * q_l^-1 mod q_i."""
    ql = prm.moduli[level]
    ids = list(range(level))
    out = []
    for c in range(ct.shape[0]):
        last = intt(prm, ct[c][level:level + 1], [level], mode)[0]          # coeff form mod q_l
        red = np.stack([last % np.uint64(prm.moduli[i]) for i in ids])
        red_ntt = ntt(prm, red, ids, mode)
        diff = sub(prm, ct[c][:level], red_ntt, ids)
        out.append(scalar_mul(prm, diff, [pow(ql % prm.moduli[i], -1, prm.moduli[i]) for i in ids],
                              ids))
    return np.stack(out)


def double_rescale(prm, ct, level, mode="fast"):
    """Double Rescale (DS, L138, L151): divide by the last TWO primes and drop two levels.
    Reading ("DS"): floor rounding like Rescale (Z10), c' = floor(x / (q_{l-1} q_l)),
    the "noise reduction limb" being r = x mod q_{l-1} q_l recovered exactly from the last two
    limbs (Garner):  r = r_l + q_l * [(r_{l-1} - r_l) q_l^-1]_{q_{l-1}},  then
    c'_i = (c_i - [r]_{q_i}) * (q_{l-1} q_l)^-1 mod q_i  for i < l-1."""
    ql, qm = prm.moduli[level], prm.moduli[level - 1]
    ids = list(range(level - 1))
    ql_inv_m = pow(ql % qm, -1, qm)
    out = []
    for c in range(ct.shape[0]):
        r_m, r_l = intt(prm, ct[c][level - 1:level + 1], [level - 1, level], mode)   # coeff form
        g = scalar_mul(prm, sub(prm, r_m[None], (r_l % np.uint64(qm))[None], [level - 1]), [ql_inv_m],
                       [level - 1])[0]                                           # in [0, q_{l-1})
        red = np.stack([r_l % np.uint64(prm.moduli[i]) for i in ids])
        red = add(prm, red, scalar_mul(prm, np.stack([g % np.uint64(prm.moduli[i]) for i in ids]),
                                       [ql % prm.moduli[i] for i in ids], ids), ids)  # [r]_{q_i}
        red_ntt = ntt(prm, red, ids, mode)
        diff = sub(prm, ct[c][:level - 1], red_ntt, ids)
        out.append(scalar_mul(prm, diff, [pow(ql * qm % prm.moduli[i], -1, prm.moduli[i]) for i in ids], ids))
    return np.stack(out)


def pmult(prm, ct, pt, level):
    """PMULT (L133): plaintext m (NTT form, [level+1][N]) times ciphertext: (c0 m, c1 m)."""
    ids = list(range(level + 1))
    return np.stack([mul(prm, ct[0], pt, ids), mul(prm, ct[1], pt, ids)])


def hadd(prm, ct_a, ct_b, level):
    """HADD (L134): (a0 + b0, a1 + b1)."""
    ids = list(range(level + 1))
    return np.stack([add(prm, ct_a[0], ct_b[0], ids), add(prm, ct_a[1], ct_b[1], ids)])


def padd(prm, ct, pt, level):
    """PADD (L135): (c0 + m, c1) -- m joins c0, the component decryption does not multiply by
    s (Z1: decrypt = c0 + c1 s)."""
    ids = list(range(level + 1))
    return np.stack([add(prm, ct[0], pt, ids), np.array(ct[1], copy=True)])


# --------------------------------------------------------------------------- keys, enc/dec

def secret(prm: Params, seed: int, h: int = 192) -> np.ndarray:
    """Z12: ternary secret with Hamming weight h (coefficients as int64)."""
    return synth.ternary_hwt(synth.derive(seed, 0x5EC), prm.N, min(h, prm.N))


def ring_square_signed(prm: Params, s: np.ndarray) -> list:
    """s^2 in Z[X]/(X^N+1) exactly (Python ints), via its support (s is sparse ternary)."""
    N = prm.N
    out = [0] * N
    nz = [(k, int(s[k])) for k in range(N) if s[k] != 0]
    for i, si in nz:
        for j, sj in nz:
            e = i + j
            if e < N:
                out[e] += si * sj
            else:
                out[e - N] -= si * sj
    return out


def automorphism_signed(s: np.ndarray, g: int) -> np.ndarray:
    N = s.shape[0]
    out = np.zeros_like(s)
    for k in range(N):
        e = (k * g) % (2 * N)
        if e >= N:
            out[e - N] = -s[k]
        else:
            out[e] = s[k]
    return out


def ks_keygen(prm: Params, s: np.ndarray, s_prime, seed: int, mode: str = "fast") -> np.ndarray:
    """KSGen(s, s') (L184) with the Z8 gadget: for each digit j of the top level,
    b_j = -a_j s + e_j + P [i in D_j] s'  mod every limb of PQ_L;  evk[j] = (b_j, a_j).

    Returns evk[dnum][2][num_q+num_p][N] in NTT form.
    """
    ids = list(range(prm.num_q + prm.num_p))
    N = prm.N
    s_ntt = ntt(prm, reduce_signed(prm, s, ids), ids, mode)
    sp_ntt = ntt(prm, reduce_signed(prm, np.asarray(s_prime, dtype=object), ids), ids, mode)
    evk = np.empty((prm.dnum, 2, len(ids), N), dtype=np.uint64)
    for j, dj in enumerate(prm.digits(prm.max_level)):
        a = synth.uniform_residues(synth.derive(seed, 2 * j), prm.moduli, N)     # NTT form
        e = synth.rounded_gaussian(synth.derive(seed, 2 * j + 1), N)
        e_ntt = ntt(prm, reduce_signed(prm, e, ids), ids, mode)
        b = sub(prm, e_ntt, mul(prm, a, s_ntt, ids), ids)
        gad = [(prm.P % prm.moduli[i]) if i in dj else 0 for i in ids]
        b = add(prm, b, scalar_mul(prm, sp_ntt, gad, ids), ids)
        evk[j, 0] = b
        evk[j, 1] = a
    return evk


def relin_key(prm, s, seed, mode="fast"):
    return ks_keygen(prm, s, ring_square_signed(prm, s), seed, mode)


def rot_key(prm, s, g, seed, mode="fast"):
    return ks_keygen(prm, s, automorphism_signed(s, g), seed, mode)


def encrypt(prm: Params, m: np.ndarray, s: np.ndarray, level: int, seed: int, mode="fast"):
    """Z1 standard sign: ct = (-a s + m + e, a) mod Q_l, NTT form."""
    ids = list(range(level + 1))
    a = synth.uniform_residues(synth.derive(seed, 0xA), [prm.moduli[i] for i in ids], prm.N)
    e = synth.rounded_gaussian(synth.derive(seed, 0xE), prm.N)
    m = np.asarray(m)
    me = (m + e.astype(object)) if m.dtype == object else m.astype(np.int64) + e   # object: |m| >= 2^63
    me_ntt = ntt(prm, reduce_signed(prm, me, ids), ids, mode)
    s_ntt = ntt(prm, reduce_signed(prm, s, ids), ids, mode)
    c0 = sub(prm, me_ntt, mul(prm, a, s_ntt, ids), ids)
    return np.stack([c0, a])


def decrypt_residues(prm, ct, s, level, mode="fast"):
    """c0 + c1 s (Z1) in coefficient form, residues [level+1][N]."""
    ids = list(range(level + 1))
    s_ntt = ntt(prm, reduce_signed(prm, s, ids), ids, mode)
    m_ntt = add(prm, ct[0], mul(prm, ct[1], s_ntt, ids), ids)
    return intt(prm, m_ntt, ids, mode)


def crt_centered(prm: Params, res: np.ndarray, ids) -> list:
    """Big-integer CRT lift of residues to (-M/2, M/2], M = prod moduli[ids]."""
    ms = [prm.moduli[i] for i in ids]
    M = math.prod(ms)
    acc = np.zeros(res.shape[1], dtype=object)
    for k, m in enumerate(ms):
        Mk = M // m
        coef = Mk * pow(Mk % m, -1, m)
        acc = acc + res[k].astype(object) * coef
    acc = acc % M
    return [int(v) - M if v > M // 2 else int(v) for v in acc]


def crt_lift(prm: Params, res: np.ndarray, ids) -> list:
    """Big-integer CRT lift to [0, M)."""
    ms = [prm.moduli[i] for i in ids]
    M = math.prod(ms)
    acc = np.zeros(res.shape[1], dtype=object)
    for k, m in enumerate(ms):
        Mk = M // m
        acc = acc + res[k].astype(object) * (Mk * pow(Mk % m, -1, m))
    return [int(v) for v in acc % M]


def _slot_exponents(N: int) -> np.ndarray:
    """5^j mod 2N for j < N/2 (slot j sits at zeta^(5^j), zeta = e^(i pi / N); L121)."""
    e = np.empty(N // 2, dtype=np.int64)
    v = 1
    for j in range(N // 2):
        e[j] = v
        v = v * 5 % (2 * N)
    return e


_ROOTS = {}


def _roots(N: int, sign: int) -> np.ndarray:
    """exp(sign i pi e / N) for e < 2N: the same float operations as evaluating the exponential
    at the angle (e mod 2N) pi / N directly, tabulated (a lookup instead of a complex exp)."""
    key = (N, sign)
    if key not in _ROOTS:
        _ROOTS[key] = np.exp(sign * 1j * (np.arange(2 * N, dtype=np.int64).astype(np.float64) * (np.pi / N)))
    return _ROOTS[key]


def encode(N: int, z: np.ndarray, delta: float) -> np.ndarray:
    """m = round(Delta * tau^-1(z)), m_k = (2/N) Re sum_j z_j zeta_j^-k (half away from 0)."""
    ej = _slot_exponents(N)
    k = np.arange(N, dtype=np.int64)
    acc = np.zeros(N, dtype=np.float64)
    roots = _roots(N, -1)
    for lo in range(0, N // 2, 64):
        acc += np.real(z[lo:lo + 64] @ roots[np.outer(ej[lo:lo + 64], k) % (2 * N)])
    x = delta * (2.0 / N) * acc
    return (np.sign(x) * np.floor(np.abs(x) + 0.5)).astype(np.int64)


def encode_fft(N: int, z: np.ndarray, delta: float) -> np.ndarray:
    """encode() evaluated with one length-2N FFT: the slots and their conjugates placed at the
    odd exponents 5^j and 2N - 5^j give sum_e Z_e zeta^(-e k) = 2 Re sum_j z_j zeta_j^-k.  Same
    value up to floating-point rounding order (|difference| <= 1 after rounding, pinned in
    tests/test_oracle_ntt.py); used for the many plaintext diagonals of bootstrapping."""
    ej = _slot_exponents(N)
    Z = np.zeros(2 * N, dtype=np.complex128)
    Z[ej] = z
    Z[2 * N - ej] = np.conj(z)
    x = delta / N * np.real(np.fft.fft(Z)[:N])
    return (np.sign(x) * np.floor(np.abs(x) + 0.5)).astype(np.int64)


def decode(N: int, m: list, delta: float) -> np.ndarray:
    """z_j = m(zeta_j) / Delta."""
    ej = _slot_exponents(N)
    k = np.arange(N, dtype=np.int64)
    mf = np.array([float(v) for v in m], dtype=np.float64)
    z = np.empty(N // 2, dtype=np.complex128)
    roots = _roots(N, 1)
    for lo in range(0, N // 2, 64):
        z[lo:lo + 64] = roots[np.outer(ej[lo:lo + 64], k) % (2 * N)] @ mf
    return z / delta
