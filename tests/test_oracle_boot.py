"""Oracle pins for bootstrapping (reading BOOT in DESIGN.md): ModRaise's exact
big-integer identity, the slot-algebra matrix W, and that a bootstrapped ciphertext decrypts
to the input slots at a fresh, higher level."""
import math

import numpy as np
import pytest

import synth
from oracle import boot, ckks


def test_modraise_is_centred_lift():
    """dec(ModRaise(ct)) over Z equals c0' + c1' s for the centred lifts: = dec(ct) (mod q_0),
    with the quotient I bounded by (||s||_1 + 1) / 2 + 1."""
    bp = boot.tiny()
    prm = bp.prm
    s = ckks.secret(prm, 5, bp.h)
    ct = boot.encrypt_sparse(bp, synth.complex_slots(7, bp.n), 2.0 ** 26, s, 9)
    L = bp.top
    up = boot.modraise(prm, ct, L)
    big = ckks.crt_centered(prm, ckks.decrypt_residues(prm, up, s, L), list(range(L + 1)))
    small = ckks.crt_centered(prm, ckks.decrypt_residues(prm, ct, s, 0), [0])
    q0 = prm.q[0]
    bound = (int(np.abs(s).sum()) + 1) // 2 + 1
    for a, b in zip(big, small):
        assert (a - b) % q0 == 0 and abs((a - b) // q0) <= bound


def test_xi_matrix_maps_subring_coefficients_to_slots():
    """W w gives the slots of sum_j (Re w_j) X^(Mj) + (Im w_j) X^(M(j+n)) (decode's definition)."""
    bp = boot.tiny()
    N, n, M = bp.prm.N, bp.n, bp.M
    rng = np.random.default_rng(3)
    w = rng.standard_normal(n) + 1j * rng.standard_normal(n)
    coef = np.zeros(N)
    coef[M * np.arange(n)] = w.real
    coef[M * (np.arange(n) + n)] = w.imag
    z = ckks.decode(N, [float(v) for v in coef], 1.0)[:n]
    assert np.max(np.abs(boot._xi_matrix(n) @ w - z)) < 1e-9


@pytest.fixture(scope="module")
def booted():
    bp = boot.tiny()
    s = ckks.secret(bp.prm, 21, bp.h)
    keys = boot.boot_keys(bp, s, 500)
    z = synth.complex_slots(23, bp.n)
    delta = 2.0 ** 31
    ct0 = boot.encrypt_sparse(bp, z, delta, s, 25)
    out, lv, scale, consts = boot.bootstrap(bp, ct0, keys)
    return bp, s, z, delta, out, lv, scale


def test_bootstrap_decodes_to_input(booted):
    """Tolerance (Delta_in = 2^31, q_0 ~ 2^36, scales ~2^36 inside, r = 9): the coefficient-level
    rounding noise of E_0 = exp(i theta t), ~(1 + h) sqrt(N) / 2^36 ~ 3e-8, is amplified 2^r = 512
    by the squarings: ~2.4e-6 in t = m / q_0, i.e. ~3e-4 on the slots after x q_0 / Delta_in = 32
    and the coefficient-to-slot gain sqrt(2n) = 4; the sine's own error (2 pi t)^2 / 6 at
    t <= 0.012 is ~9e-4 relative (1.3e-3 on |z| <= sqrt 2).  4e-3 absolute is 2x the sum."""
    bp, s, z, delta, out, lv, scale = booted
    assert lv == bp.top - bp.levels_used()
    got = boot.decode_sparse(bp, out, lv, scale * delta / bp.prm.q[0], s)
    assert np.max(np.abs(got - z)) < 4e-3
