"""Oracle pins for the key-switch path (Table 2, Eq. 2, Fig. 5),
HMULT (L132), HROTATE (L136, L184), Rescale (L137) and AUTO (L268-270).

Each check is decided by something other than the oracle's own formulas: big-integer
CRT, the exact ModDown rounding bound, coefficient-domain schoolbook products, the
coefficient-domain definition of X -> X^g, and the plaintext computation on slots."""
import math

import numpy as np
import pytest

import synth
from oracle import _core, ckks

H = 192


def _centered(v, M):
    v %= M
    return v - M if v > M // 2 else v


def _noise_inf(prm, ct_coef_lift, want_lift, level):
    M = math.prod(prm.q[: level + 1])
    return max(abs(_centered(a - b, M)) for a, b in zip(ct_coef_lift, want_lift))


def _ring_mul_int(a, b):
    """Exact product in Z[X]/(X^N+1) for Python-int coefficient lists (a sparse)."""
    N = len(a)
    out = [0] * N
    nz = [(i, v) for i, v in enumerate(a) if v]
    for i, ai in nz:
        for j in range(N):
            if b[j]:
                if i + j < N:
                    out[i + j] += ai * b[j]
                else:
                    out[i + j - N] -= ai * b[j]
    return out


def _zero_error_key(prm, s, s_prime):
    """KSGen with e_j = 0 (for the exact ModDown-rounding bound)."""
    ids = list(range(prm.num_q + prm.num_p))
    s_ntt = ckks.ntt(prm, ckks.reduce_signed(prm, s, ids), ids)
    sp_ntt = ckks.ntt(prm, ckks.reduce_signed(prm, np.asarray(s_prime, dtype=object), ids), ids)
    evk = np.empty((prm.dnum, 2, len(ids), prm.N), dtype=np.uint64)
    for j, dj in enumerate(prm.digits(prm.max_level)):
        a = synth.uniform_residues(synth.derive(77, j), prm.moduli, prm.N)
        gad = [(prm.P % prm.moduli[i]) if i in dj else 0 for i in ids]
        evk[j, 0] = ckks.add(prm, ckks.sub(prm, np.zeros_like(a), ckks.mul(prm, a, s_ntt, ids), ids),
                             ckks.scalar_mul(prm, sp_ntt, gad, ids), ids)
        evk[j, 1] = a
    return evk


@pytest.mark.parametrize("mk", [ckks.tiny, ckks.tiny_dnum3])
def test_keyswitch_exact_rounding_bound(mk):
    """With e_j = 0: ||dec(KS(d)) - d s'||_inf <= (K+2)(1+h)  (ModDown floor - u, Z9)."""
    prm = mk()
    level = prm.max_level
    ids = list(range(level + 1))
    s = ckks.secret(prm, 1, H)
    s2 = ckks.ring_square_signed(prm, s)
    evk = _zero_error_key(prm, s, s2)
    d = synth.uniform_residues(5, prm.q, prm.N)
    k0, k1 = ckks.keyswitch(prm, d, level, evk)
    got = ckks.crt_lift(prm, ckks.decrypt_residues(prm, np.stack([k0, k1]), s, level), ids)
    d_coef = ckks.crt_lift(prm, ckks.intt(prm, d, ids), ids)
    want = _ring_mul_int(s2, d_coef)
    bound = (prm.num_p + 1) * (1 + H)
    assert _noise_inf(prm, got, want, level) <= bound


@pytest.mark.parametrize("mk,level", [(ckks.tiny, 2), (ckks.tiny_dnum3, 2), (ckks.tiny_dnum3, 1)])
def test_keyswitch_real_key_noise_bound(mk, level):
    """Real keys: noise <= beta N (alpha+1) max Q_j 19 / P + (K+2)(1+h)  (worst case)."""
    prm = mk()
    ids = list(range(level + 1))
    s = ckks.secret(prm, 2, H)
    s2 = ckks.ring_square_signed(prm, s)
    evk = ckks.ks_keygen(prm, s, s2, 9)
    d = synth.uniform_residues(6, prm.q[: level + 1], prm.N)
    k0, k1 = ckks.keyswitch(prm, d, level, evk)
    got = ckks.crt_lift(prm, ckks.decrypt_residues(prm, np.stack([k0, k1]), s, level), ids)
    want = _ring_mul_int(s2, ckks.crt_lift(prm, ckks.intt(prm, d, ids), ids))
    qj = max(math.prod(prm.moduli[i] for i in dj) for dj in prm.digits(level))
    bound = prm.beta(level) * prm.N * (prm.alpha + 1) * qj * 19 // prm.P + (prm.num_p + 1) * (1 + H)
    assert _noise_inf(prm, got, want, level) <= bound


def test_keyip_convolution_theorem():
    """KeyIP in the NTT domain (a6) equals sum_j d_hat_j * evk_j by coefficient schoolbook."""
    prm = ckks.tiny_dnum3()
    level = 2
    s = ckks.secret(prm, 3, H)
    evk = ckks.relin_key(prm, s, 4)
    d = synth.uniform_residues(8, prm.q, prm.N)
    tr = {}
    ckks.keyswitch(prm, d, level, evk, trace=tr)
    ext = list(range(level + 1)) + prm.p_ids
    L = _core.lib()
    for c in range(2):
        for k, t in enumerate(ext):
            m = prm.moduli[t]
            acc = np.zeros(prm.N, dtype=np.uint64)
            for j in range(prm.beta(level)):
                a = ckks.intt(prm, tr["dhat"][j][k:k + 1], [t])[0]
                b = ckks.intt(prm, evk[j, c][t:t + 1], [t])[0]
                prod = np.empty_like(a)
                L.or_negacyclic_mul(_core.ptr(a), _core.ptr(b), _core.ptr(prod), prm.N, m)
                acc = ckks.add(prm, acc[None], prod[None], [t])[0]
            assert np.array_equal(ckks.intt(prm, tr["acc"][c][k:k + 1], [t])[0], acc)


def test_automorphism_ntt_index_map():
    """NTT(sigma_g(a)) (coefficient definition) == index map applied to NTT(a)."""
    prm = ckks.tiny()
    ids = [0, 3]
    a = synth.uniform_residues(21, [prm.moduli[i] for i in ids], prm.N)
    for g in (5, 25, 2 * prm.N - 1, 5 ** 7 % (2 * prm.N)):
        lhs = ckks.ntt(prm, ckks.automorphism_coeff(prm, a, ids, g), ids)
        rhs = ckks.automorphism_ntt(ckks.ntt(prm, a, ids), g)
        assert np.array_equal(lhs, rhs)


def test_rescale_is_exact_floor():
    """Z10: rescale = floor(x / q_l) on the big-integer CRT lift, for both components."""
    prm = ckks.tiny()
    level = 2
    ct = np.stack([synth.uniform_residues(30 + c, prm.q, prm.N) for c in range(2)])
    out = ckks.rescale(prm, ct, level)
    for c in range(2):
        x = ckks.crt_lift(prm, ckks.intt(prm, ct[c], [0, 1, 2]), [0, 1, 2])
        y = ckks.crt_lift(prm, ckks.intt(prm, out[c], [0, 1]), [0, 1])
        M = prm.q[0] * prm.q[1]
        assert all(yy == (xx // prm.q[2]) % M for xx, yy in zip(x, y))


def test_encode_decode_roundtrip():
    N = 1 << 10
    z = synth.complex_slots(1, N // 2)
    m = ckks.encode(N, z, 2.0 ** 40)
    assert np.max(np.abs(ckks.decode(N, list(m), 2.0 ** 40) - z)) < 1e-9


@pytest.fixture(scope="module")
def enc_setup():
    prm = ckks.tiny_dnum3()
    delta = 2.0 ** 40
    s = ckks.secret(prm, 11, H)
    za = synth.complex_slots(101, prm.N // 2)
    zb = synth.complex_slots(102, prm.N // 2)
    cta = ckks.encrypt(prm, ckks.encode(prm.N, za, delta), s, 2, 201)
    ctb = ckks.encrypt(prm, ckks.encode(prm.N, zb, delta), s, 2, 202)
    return prm, delta, s, za, zb, cta, ctb


def test_encrypt_decrypt(enc_setup):
    prm, delta, s, za, zb, cta, ctb = enc_setup
    m = ckks.crt_centered(prm, ckks.decrypt_residues(prm, cta, s, 2), [0, 1, 2])
    assert np.max(np.abs(ckks.decode(prm.N, m, delta) - za)) < 1e-9


def test_hmult_rescale_precision(enc_setup):
    """HMULT then Rescale decodes to z_a * z_b within 1e-6 at Delta = 2^40 (north_star)."""
    prm, delta, s, za, zb, cta, ctb = enc_setup
    relin = ckks.relin_key(prm, s, 301)
    ct = ckks.hmult(prm, cta, ctb, 2, relin)
    ct = ckks.rescale(prm, ct, 2)
    m = ckks.crt_centered(prm, ckks.decrypt_residues(prm, ct, s, 1), [0, 1])
    z = ckks.decode(prm.N, m, delta * delta / prm.q[2])
    assert np.max(np.abs(z - za * zb)) < 1e-6


@pytest.mark.parametrize("r", [1, 5, 0])
def test_hrot_rotates_slots(enc_setup, r):
    """HROTATE with g = 5^r mod 2N rotates slots left by r (Z11)."""
    prm, delta, s, za, zb, cta, ctb = enc_setup
    g = pow(5, r, 2 * prm.N)
    key = ckks.rot_key(prm, s, g, 400 + r)
    ct = ckks.hrot(prm, cta, g, 2, key)
    m = ckks.crt_centered(prm, ckks.decrypt_residues(prm, ct, s, 2), [0, 1, 2])
    z = ckks.decode(prm.N, m, delta)
    assert np.max(np.abs(z - np.roll(za, -r))) < 1e-6


def test_hrot_conjugation(enc_setup):
    prm, delta, s, za, zb, cta, ctb = enc_setup
    g = 2 * prm.N - 1
    ct = ckks.hrot(prm, cta, g, 2, ckks.rot_key(prm, s, g, 500))
    m = ckks.crt_centered(prm, ckks.decrypt_residues(prm, ct, s, 2), [0, 1, 2])
    assert np.max(np.abs(ckks.decode(prm.N, m, delta) - np.conj(za))) < 1e-6


@pytest.mark.slow
def test_set_b_keyswitch_exact_rounding_bound():
    """Set-B (N=2^16, 36+12 limbs, dnum=3, l=35): with e_j = 0 the key-switch output
    decrypts to d * s' up to (K+2)(1+h), on sampled coefficients (s' = sigma_5(s))."""
    prm = ckks.set_b()
    level = 35
    ids = list(range(level + 1))
    s = ckks.secret(prm, 1, H)
    sp = ckks.automorphism_signed(s, 5)
    evk = _zero_error_key(prm, s, sp)
    d = synth.uniform_residues(5, prm.q, prm.N)
    k0, k1 = ckks.keyswitch(prm, d, level, evk)
    dec = ckks.decrypt_residues(prm, np.stack([k0, k1]), s, level)
    d_coef = ckks.crt_lift(prm, ckks.intt(prm, d, ids), ids)
    M = math.prod(prm.q)
    nz = [(i, int(sp[i])) for i in range(prm.N) if sp[i]]
    bound = (prm.num_p + 1) * (1 + H)
    for k in list(range(0, prm.N, 4099)) + [prm.N - 1]:
        want = 0
        for i, v in nz:
            want += v * d_coef[k - i] if k >= i else -v * d_coef[k - i + prm.N]
        got = ckks.crt_lift(prm, dec[:, k:k + 1], ids)[0]
        assert abs(_centered(got - want, M)) <= bound


def test_hrot_hoisted_rotates_slots(enc_setup):
    """Hoisted HROTATE (one ModUp, automorphism after ModDown) decodes to the rotations."""
    prm, delta, s, za, zb, cta, ctb = enc_setup
    rs = [1, 3]
    gs = [pow(5, r, 2 * prm.N) for r in rs]
    keys = [ckks.rot_key(prm, s, g, 600 + r) for g, r in zip(gs, rs)]
    out = ckks.hrot_hoisted(prm, cta, gs, 2, keys)
    for r, ct in zip(rs, out):
        m = ckks.crt_centered(prm, ckks.decrypt_residues(prm, ct, s, 2), [0, 1, 2])
        assert np.max(np.abs(ckks.decode(prm.N, m, delta) - np.roll(za, -r))) < 1e-6


@pytest.mark.parametrize("mk,level", [(ckks.tiny, 2), (ckks.tiny_dnum3, 2), (ckks.tiny_dnum3, 0)])
def test_moddown_exact_floor_pin(mk, level):
    """Z9 pinned on its own (not through a noise bound, which a sign error in the combine
    (acc - conv) -> (acc + conv) survives: with e_j = 0 the extra 2 conv / P term decrypts to a
    small multiple of (1 + h)).  For every coefficient, with A the exact big-integer CRT lift of
    the KeyIP output acc_c over PQ_l, ModDown's output must equal floor(A / P) - u (mod Q_l) with
    the BConv overflow u in [0, K+1) (Algorithm 1 non-centred, Z7)."""
    prm = mk()
    q_ids = list(range(level + 1))
    ext = q_ids + prm.p_ids
    d = synth.uniform_residues(41, prm.q[: level + 1], prm.N)
    evk = np.stack([np.stack([synth.uniform_residues(50 + 2 * j + c, prm.moduli, prm.N) for c in range(2)])
                    for j in range(prm.dnum)])
    tr = {}
    out = ckks.keyswitch(prm, d, level, evk, trace=tr)
    Q = math.prod(prm.q[: level + 1])
    for c in range(2):
        A = ckks.crt_lift(prm, ckks.intt(prm, tr["acc"][c], ext), ext)
        got = ckks.crt_lift(prm, ckks.intt(prm, out[c], q_ids), q_ids)
        us = {((a // prm.P) - g) % Q for a, g in zip(A, got)}
        assert us <= set(range(prm.num_p)), sorted(us)[:4]
