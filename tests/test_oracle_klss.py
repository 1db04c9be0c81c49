"""Oracle pins for KLSS key-switching (L155-180, Eq. 3-4, Table 2, Alg. 3/4; readings K1-K6
in oracle/klss.py and DESIGN.md).

Decided by things other than the KLSS oracle's own formulas: Python big-integer CRT, the
bound of Eq. 4, the (separately pinned) Hybrid key-switch it must equal bit for bit (K4),
and decryption of real ciphertexts."""
import math

import numpy as np
import pytest

import synth
from oracle import ckks, klss


def _lift(res_cols, mods, centred):
    Q = math.prod(mods)
    x = 0
    for r, m in zip(res_cols, mods):
        Mk = Q // m
        x += int(r) * Mk * pow(Mk % m, -1, m)
    x %= Q
    return x - Q if centred and 2 * x > Q else x


@pytest.mark.parametrize("centred", [False, True])
def test_crt_exact_matches_python_bigint(centred):
    mods = ckks.gen_primes(12, 36, 7)
    outs = ckks.gen_primes(12, 36, 10)[7:]
    rng = np.random.default_rng(5)
    n = 300
    x = np.stack([rng.integers(0, m, n, dtype=np.uint64) for m in mods])
    Q = math.prod(mods)
    # edge values: 0, Q-1, floor(Q/2), floor(Q/2)+1 in the first four columns
    for k, v in enumerate([0, Q - 1, Q // 2, Q // 2 + 1]):
        for r, m in enumerate(mods):
            x[r, k] = v % m
    got = klss.crt_exact(mods, x, outs, centred)
    for k in range(n):
        v = _lift(x[:, k], mods, centred)
        assert [int(g) for g in got[:, k]] == [v % t for t in outs]


def test_alpha_prime_follows_eq4_set_c():
    """Eq. 4 (L173) with K2/K3 at Set-C, WordSize_T = 36: alpha' T primes, T > 4 beta N B B~."""
    kp = klss.set_c_t36()
    b = kp.base
    assert (b.alpha, b.num_p, kp.beta_t) == (4, 4, 8)
    B = 4 * max(math.prod(b.q[4 * j:4 * j + 4]) for j in range(9))
    Bt = max(math.prod(b.moduli[i] for i in g) for g in kp.groups)
    bound = 9 * b.N * B * Bt
    assert kp.bound == bound
    T = math.prod(kp.t)
    assert T > 4 * bound and T // kp.t[-1] <= 4 * bound                  # minimal
    assert kp.alpha_p == 10 == math.ceil(math.log2(4 * bound) / 36)
    assert all(ckks.is_prime(t) and t % (2 * b.N) == 1 and t.bit_length() == 36 for t in kp.t)
    assert not set(kp.t) & set(b.moduli)


def test_alpha_prime_follows_eq4_set_c_t48():
    """Eq. 4 (L173) at Set-C as printed in Table 4 (WordSize_T = 48, L511): alpha' = 8 T primes of
    48 bits, the Z4 rule at 48 bits (K6): the largest 48-bit k 2N + 1 primes in order."""
    kp = klss.set_c()
    b = kp.base
    T = math.prod(kp.t)
    assert T > 4 * kp.bound and T // kp.t[-1] <= 4 * kp.bound
    assert kp.alpha_p == 8 == math.ceil(math.log2(4 * kp.bound) / 48)
    assert all(ckks.is_prime(t) and t % (2 * b.N) == 1 and t.bit_length() == 48 for t in kp.t)
    two_n = 2 * b.N
    ks = [(t - 1) // two_n for t in kp.t]
    assert ks == sorted(ks, reverse=True) and ks[0] <= ((1 << 48) - 1) // two_n
    for k in range(ks[-1] + 1, ((1 << 48) - 1) // two_n + 1):         # every skipped candidate composite
        if k not in ks:
            assert not ckks.is_prime(k * two_n + 1)


@pytest.mark.parametrize("mk", [klss.tiny, klss.tiny48])
def test_klss_key_is_evk_mod_group(mk):
    """K1: INTT_T of the key, lifted exactly from T, is [evk]_{P~_i} in [0, P~_i) and agrees
    with evk modulo every limb of the group."""
    kp = mk()
    b = kp.base
    evk = np.stack([np.stack([synth.uniform_residues(60 + 2 * j + c, b.moduli, b.N) for c in range(2)])
                    for j in range(b.dnum)])
    ek = klss.klss_key(kp, evk)
    for i, g in enumerate(kp.groups):
        Pt = math.prod(b.moduli[t] for t in g)
        for j in range(b.dnum):
            e_coef = ckks.intt(kp, ek[0, i, j], kp.t_ids)
            evk_coef = ckks.intt(b, evk[j, 0][g], g)
            for n in range(0, b.N, 97):
                e = _lift(e_coef[:, n], kp.t, centred=False)
                assert 0 <= e < Pt
                assert [e % b.moduli[t] for t in g] == [int(v) for v in evk_coef[:, n]]


@pytest.mark.parametrize("mk", [klss.tiny, klss.tiny48])
@pytest.mark.parametrize("level", [5, 3, 0])
def test_klss_keyswitch_equals_hybrid(level, mk):
    """K4: with the key of K1, KLSS KeySwitch returns exactly Hybrid's output (every residue);
    WordSize_T = 36 and 48 (K6)."""
    kp = mk()
    b = kp.base
    evk = np.stack([np.stack([synth.uniform_residues(80 + 2 * j + c, b.moduli, b.N) for c in range(2)])
                    for j in range(b.dnum)])
    ek = klss.klss_key(kp, evk)
    d = synth.uniform_residues(90 + level, b.q[:level + 1], b.N)
    trace = {}
    k0, k1 = klss.keyswitch(kp, d, level, ek, trace)
    h0, h1 = ckks.keyswitch(b, d, level, evk)
    assert np.array_equal(k0, h0) and np.array_equal(k1, h1)
    # Eq. 4 / K3: every IP coefficient, lifted centred from T, is inside (-T/4, T/4)
    for acc in trace["ip_coef"]:
        for n in range(0, b.N, 211):
            v = _lift(acc[:, n], kp.t, centred=True)
            assert 4 * abs(v) < kp.T


def test_klss_hmult_rescale_decrypts():
    """Real encryptions: KLSS HMULT + Rescale decodes to z_a z_b (tiny KLSS set, Delta = 2^40)."""
    kp = klss.tiny()
    b = kp.base
    delta = 2.0 ** 40
    s = ckks.secret(b, 31, 192)
    za, zb = synth.complex_slots(131, b.N // 2), synth.complex_slots(132, b.N // 2)
    lv = b.max_level
    cta = ckks.encrypt(b, ckks.encode(b.N, za, delta), s, lv, 231)
    ctb = ckks.encrypt(b, ckks.encode(b.N, zb, delta), s, lv, 232)
    ek = klss.klss_key(kp, ckks.relin_key(b, s, 331))
    ct = ckks.rescale(b, klss.hmult(kp, cta, ctb, lv, ek), lv)
    m = ckks.crt_centered(b, ckks.decrypt_residues(b, ct, s, lv - 1), list(range(lv)))
    z = ckks.decode(b.N, m, delta * delta / b.q[lv])
    assert np.max(np.abs(z - za * zb)) < 1e-6


@pytest.mark.parametrize("mk", [klss.set_c_t36, klss.set_c])
def test_klss_equals_hybrid_set_c(mk):
    """K4 at Set-C (dnum = 9, alpha~ = 5; 10 T primes of 36 bits or 8 of 48), level 35: every
    residue of every limb."""
    kp = mk()
    b = kp.base
    evk = np.stack([np.stack([synth.uniform_residues(400 + 2 * j + c, b.moduli, b.N) for c in range(2)])
                    for j in range(b.dnum)])
    ek = klss.klss_key(kp, evk)
    d = synth.uniform_residues(401, b.q, b.N)
    k0, k1 = klss.keyswitch(kp, d, 35, ek)
    h0, h1 = ckks.keyswitch(b, d, 35, evk)
    assert np.array_equal(k0, h0) and np.array_equal(k1, h1)
