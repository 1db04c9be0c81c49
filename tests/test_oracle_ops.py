"""Oracle pins for PMULT (L133), HADD (L134), PADD (L135) and Double Rescale (L138, L151).

Decided by something other than the oracle's formulas: the exact big-integer floor on the
CRT lift, the identity floor(floor(x/a)/b) = floor(x/(ab)) against the (separately pinned)
single Rescale, and the plaintext computation on decoded slots."""
import numpy as np
import pytest

import synth
from oracle import ckks

H = 192


@pytest.mark.parametrize("mk,level", [(ckks.tiny_dnum3, 2), (ckks.set_b, 3)])
def test_double_rescale_is_exact_floor(mk, level):
    """DS = floor(x / (q_{l-1} q_l)) on the big-integer CRT lift (reading "DS")."""
    prm = mk()
    ct = np.stack([synth.uniform_residues(40 + c, prm.q[: level + 1], prm.N) for c in range(2)])
    out = ckks.double_rescale(prm, ct, level)
    assert out.shape == (2, level - 1, prm.N)
    ids_in, ids_out = list(range(level + 1)), list(range(level - 1))
    div = prm.q[level] * prm.q[level - 1]
    M = int(np.prod([prm.q[i] for i in ids_out], dtype=object))
    for c in range(2):
        x = ckks.crt_lift(prm, ckks.intt(prm, ct[c], ids_in), ids_in)
        y = ckks.crt_lift(prm, ckks.intt(prm, out[c], ids_out), ids_out)
        assert all(yy == (xx // div) % M for xx, yy in zip(x, y))


def test_double_rescale_equals_two_rescales():
    """floor(floor(x / q_l) / q_{l-1}) = floor(x / (q_{l-1} q_l)): DS == Rescale o Rescale, bit for bit."""
    prm = ckks.set_b()
    level = 4
    ct = np.stack([synth.uniform_residues(50 + c, prm.q[: level + 1], prm.N) for c in range(2)])
    two = ckks.rescale(prm, ckks.rescale(prm, ct, level), level - 1)
    assert np.array_equal(ckks.double_rescale(prm, ct, level), two)


def test_hadd_padd_pmult_are_slotwise():
    prm = ckks.tiny_dnum3()
    delta = 2.0 ** 40
    s = ckks.secret(prm, 12, H)
    za, zb = synth.complex_slots(111, prm.N // 2), synth.complex_slots(112, prm.N // 2)
    ids = [0, 1, 2]
    cta = ckks.encrypt(prm, ckks.encode(prm.N, za, delta), s, 2, 211)
    ctb = ckks.encrypt(prm, ckks.encode(prm.N, zb, delta), s, 2, 212)
    pt = ckks.ntt(prm, ckks.reduce_signed(prm, ckks.encode(prm.N, zb, delta), ids), ids)

    def dec(ct, level, scale):
        m = ckks.crt_centered(prm, ckks.decrypt_residues(prm, ct, s, level), list(range(level + 1)))
        return ckks.decode(prm.N, m, scale)

    assert np.max(np.abs(dec(ckks.hadd(prm, cta, ctb, 2), 2, delta) - (za + zb))) < 1e-6
    assert np.max(np.abs(dec(ckks.padd(prm, cta, pt, 2), 2, delta) - (za + zb))) < 1e-6
    pm = ckks.rescale(prm, ckks.pmult(prm, cta, pt, 2), 2)
    assert np.max(np.abs(dec(pm, 1, delta * delta / prm.q[2]) - za * zb)) < 1e-6


def test_double_rescale_decodes():
    """A ciphertext at scale 2^30 q_1 q_2 decodes at scale 2^30 after DS.  Tolerance: the floor
    adds at most (1 + ||s||_1) = 1 + h per coefficient, i.e. <= N (1 + h) / 2^30 ~ 7e-4 per
    slot in the worst case; 1e-4 holds with the random signs of that error by a wide margin."""
    prm = ckks.tiny_dnum3()
    s = ckks.secret(prm, 13, H)
    z = synth.complex_slots(121, prm.N // 2)
    m = ckks.encode(prm.N, z, 2.0 ** 30).astype(object) * (prm.q[1] * prm.q[2])   # scale 2^30 q_1 q_2
    ct = ckks.encrypt(prm, m, s, 2, 221)
    out = ckks.double_rescale(prm, ct, 2)
    m = ckks.crt_centered(prm, ckks.decrypt_residues(prm, out, s, 0), [0])
    assert np.max(np.abs(ckks.decode(prm.N, m, 2.0 ** 30) - z)) < 1e-4
