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


_RUN = {}


@pytest.fixture(scope="module")
def booted():
    bp = boot.tiny()
    s = ckks.secret(bp.prm, 21, bp.h)
    keys = boot.boot_keys(bp, s, 500)
    z = synth.complex_slots(23, bp.n)
    delta = 2.0 ** 31
    ct0 = boot.encrypt_sparse(bp, z, delta, s, 25)
    out, lv, scale, consts = boot.bootstrap(bp, ct0, keys)
    _RUN["sparse"] = consts
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


# --------------------------------------------------------------------------- full-slot (special FFT)

def _u_matrix(N):
    n = N // 2
    e5 = [pow(5, j, 2 * N) for j in range(n)]
    return np.array([[np.exp(1j * math.pi * ((e5[j] * k) % (2 * N)) / N) for k in range(n)] for j in range(n)])


def _brev_perm(n):
    bits = n.bit_length() - 1
    return np.array([int(format(i, f"0{bits}b")[::-1], 2) for i in range(n)])


def _apply(diags, x):
    return sum(v * np.roll(x, -d) for d, v in diags.items())


def test_special_fft_factorises_the_slot_matrix():
    """U = F_n ... F_2 P with U[j][k] = zeta^(5^j k) (decode's definition, checked against
    ckks.decode) and P the bit reversal; the inverse stages give P U^-1."""
    N = 1 << 8
    n = N // 2
    U = _u_matrix(N)
    rng = np.random.default_rng(5)
    t = rng.standard_normal(N)
    z_dec = ckks.decode(N, [float(v) for v in t], 1.0)
    assert np.max(np.abs(U @ (t[:n] + 1j * t[n:]) - z_dec)) < 1e-9
    x = rng.standard_normal(n) + 1j * rng.standard_normal(n)
    px = np.empty(n, dtype=complex)
    px[_brev_perm(n)] = x                                   # (P x)[brev(i)] = x[i]
    y = px
    for F in boot.sfft_stages(N, inverse=False):
        y = _apply(F, y)
    assert np.max(np.abs(y - U @ x)) < 1e-9
    y = U @ x
    for F in boot.sfft_stages(N, inverse=True)[::-1]:
        y = _apply(F, y)
    assert np.max(np.abs(y - px)) < 1e-9


def test_fft_groups_equal_the_stage_products():
    N = 1 << 10
    rng = np.random.default_rng(6)
    x = rng.standard_normal(N // 2) + 1j * rng.standard_normal(N // 2)
    for inverse in (True, False):
        st = boot.sfft_stages(N, inverse)
        want = x
        for F in (st[::-1] if inverse else st):
            want = _apply(F, want)
        got = x
        for G in boot.fft_groups(N, 3, inverse):
            got = _apply(G, got)
        assert np.max(np.abs(got - want)) < 1e-9
        for G in boot.fft_groups(N, 3, inverse):          # k = 3 stages: <= 2^(k+1) - 1 diagonals
            assert len(G) <= 15                          # (fewer when amounts wrap mod n)


@pytest.fixture(scope="module")
def full_keys():
    bp = boot.tiny_full()
    s = ckks.secret(bp.prm, 51, bp.h)
    return bp, s, boot.boot_keys(bp, s, 600)


def test_homomorphic_coeff_to_slot_full(full_keys):
    """Encrypted full-slot CoeffToSlot decodes to P U^-1 z (the bit-reversed complex packing of
    the coefficients), and SlotToCoeff brings it back to z.  Tolerances: CoeffToSlot's entries
    are O(1/n), so its output carries only the key-switch noise of ~10 rotations per level at
    scale ~2^36 (~2^-26 relative each): 1e-5 absolute.  SlotToCoeff = U P^-1 has entries of
    modulus 1 summed over n = 2048 terms, so iid input noise of rms s becomes sqrt(n) s ~ 45 s
    (s ~ 2^-22 here), plus its own rotations: 2e-4 absolute on the round trip."""
    bp, s, keys = full_keys
    prm = bp.prm
    z = synth.complex_slots(43, prm.N // 2)
    delta = float(prm.q[prm.max_level])
    L = prm.max_level
    ct = ckks.encrypt(prm, ckks.encode(prm.N, z, delta), s, L, 45)
    cts, lv = boot.fft_transform(bp, ct, L, keys, True, "cts")
    assert lv == L - bp.fft_levels
    m = ckks.crt_centered(prm, ckks.decrypt_residues(prm, cts, s, lv), list(range(lv + 1)))
    w = ckks.decode(prm.N, m, delta)
    U = _u_matrix(prm.N)
    want = np.empty_like(z)
    want[_brev_perm(prm.N // 2)] = np.linalg.solve(U, z)
    assert np.max(np.abs(w - want)) < 1e-5
    back, lv2 = boot.fft_transform(bp, cts, lv, keys, False, "stc")
    m = ckks.crt_centered(prm, ckks.decrypt_residues(prm, back, s, lv2), list(range(lv2 + 1)))
    assert np.max(np.abs(ckks.decode(prm.N, m, delta) - z)) < 2e-4


@pytest.fixture(scope="module")
def booted_full(full_keys):
    bp, s, keys = full_keys
    z = synth.complex_slots(53, bp.prm.N // 2)
    delta = 2.0 ** 31
    ct0 = boot.encrypt_sparse(bp, z, delta, s, 55)
    out, lv, scale, consts = boot.bootstrap(bp, ct0, keys)
    return bp, s, z, delta, out, lv, scale


def test_full_slot_bootstrap_decodes_to_input(booted_full):
    """All N/2 slots.  The sparse test's budget (EvalMod's 2^r = 512 amplification of the
    ~2^-30 coefficient-level rounding noise: ~3e-4 on the slots after x q_0 / Delta_in = 32 and
    the gain sqrt(2n) = 4) with the full packing's gain sqrt(N) = 64 instead (16x): ~5e-3.  The
    sine's cubic error is negligible here (t = m / q_0 <= ~1e-3 for a random full-slot message).
    1e-2 absolute is 2x -- the precision loss at 36-bit scales that makes the paper use Double
    Rescale in bootstrapping (L151)."""
    bp, s, z, delta, out, lv, scale = booted_full
    assert lv == bp.top - bp.levels_used()
    got = boot.decode_sparse(bp, out, lv, scale * delta / bp.prm.q[0], s)
    assert np.max(np.abs(got - z)) < 1e-2


def test_hrot_sum_pins():
    """hrot_sum of one ciphertext is HROTATE itself (moddown = the key-switch's a7-a10), and a
    sum of several decrypts to the sum of the slot rotations (BOOT-G)."""
    prm = ckks.Params(12, 4, 2, 2)
    s = ckks.secret(prm, 61, 32)
    L = prm.max_level
    gs = [pow(5, r, 2 * prm.N) for r in (1, 3, 7)]
    keys = [ckks.rot_key(prm, s, g, 620 + i) for i, g in enumerate(gs)]
    zs = [synth.complex_slots(630 + i, prm.N // 2) for i in range(3)]
    delta = 2.0 ** 40
    cts = [ckks.encrypt(prm, ckks.encode(prm.N, z, delta), s, L, 640 + i) for i, z in enumerate(zs)]
    assert np.array_equal(boot.hrot_sum(prm, cts[:1], gs[:1], L, keys[:1]), ckks.hrot(prm, cts[0], gs[0], L, keys[0]))
    out = boot.hrot_sum(prm, cts, gs, L, keys)
    m = ckks.crt_centered(prm, ckks.decrypt_residues(prm, out, s, L), list(range(L + 1)))
    want = sum(np.roll(z, -r) for z, r in zip(zs, (1, 3, 7)))
    assert np.max(np.abs(ckks.decode(prm.N, m, delta) - want)) < 1e-6


# --------------------------------------------------------------------------- plain vs schedule
# The GPU replays oracle/boot.py's schedule bit for bit (tests/test_gpu_boot.py): hoisted baby
# rotations (BOOT-H), giant steps summed before one ModDown (BOOT-G), baby-step giant-step
# levels.  These tests pin that schedule to the textbook one (reading BOOT-P: separate HROTATEs,
# dense diagonal sums) by decryption, so a performance choice in the schedule cannot silently
# change what is computed.
#
# Derived bound at the CoeffToSlot output.  Both schedules compute the same linear map; they
# differ only in rounding: the key noise terms of a rotation are identical (sigma commutes with
# the digit decomposition), so each key-switch contributes at most its ModDown floor rounding,
# ||e||_inf <= (K+2)(1+h) (Z9, pinned in test_oracle_ks.py), and each Rescale its floor rounding
# <= 1 + h; a coefficient error e becomes a slot error <= ||e||_1 <= N ||e||_inf, multiplied by
# the largest diagonal entry it is later scaled with (D_max) and divided by the ciphertext scale
# q_0.  Summing over every key-switch and Rescale of both runs gives B_cts below.

def _cts_bound(bp, n_ks, n_rs, dmax):
    prm = bp.prm
    e_ks = (prm.num_p + 1) * (1 + bp.h)
    return prm.N * (n_ks * e_ks * dmax + n_rs * (1 + bp.h)) / prm.q[0]


def _slot_values(bp, ct, lv, s):
    """Decrypt + decode at scale q_0 (the CoeffToSlot output's value scale), all N/2 slots."""
    m = ckks.crt_centered(bp.prm, ckks.decrypt_residues(bp.prm, ct, s, lv), list(range(lv + 1)))
    return ckks.decode(bp.prm.N, m, float(bp.prm.q[0]))


def test_plain_vs_schedule_sparse(booted):
    bp, s, z, delta, out, lv, scale = booted
    keys = boot.boot_keys(bp, s, 500, plain=True)
    ct0 = boot.encrypt_sparse(bp, z, delta, s, 25)
    # CoeffToSlot stage: hoisted n - 1 rotations vs n - 1 separate HROTATEs
    a, la, _, _ = boot.bootstrap(bp, ct0, keys, stop_after_cts=True)
    b, lb, _, _ = boot.bootstrap(bp, ct0, keys, plain=True, stop_after_cts=True)
    assert la == lb
    dmax = np.max(np.abs(np.linalg.inv(boot._xi_matrix(bp.n)) / bp.M))
    B = _cts_bound(bp, 2 * (bp.n - 1), 2, dmax)
    diff = np.max(np.abs(_slot_values(bp, a, la, s) - _slot_values(bp, b, lb, s)))
    assert diff <= B, (diff, B)
    # whole bootstrap: both decode to the input (test_bootstrap_decodes_to_input's gate)
    p, lp, sp, _ = boot.bootstrap(bp, ct0, keys, plain=True)
    assert (lp, sp) == (lv, scale)
    assert np.max(np.abs(boot.decode_sparse(bp, p, lp, sp * delta / bp.prm.q[0], s) - z)) < 4e-3


@pytest.mark.slow
def test_plain_vs_schedule_full_slot():
    """Full slots, 3 factored levels per transform: BSGS + hoisting + shared giant-step ModDown
    against one HROTATE and one PMULT per diagonal."""
    bp = boot.tiny_full(3)
    prm = bp.prm
    s = ckks.secret(prm, 51, bp.h)
    keys = boot.boot_keys(bp, s, 600, plain=True)
    z = synth.complex_slots(53, prm.N // 2)
    delta = 2.0 ** 31
    ct0 = boot.encrypt_sparse(bp, z, delta, s, 55)
    a, la, _, _ = boot.bootstrap(bp, ct0, keys, stop_after_cts=True)
    b, lb, _, _ = boot.bootstrap(bp, ct0, keys, plain=True, stop_after_cts=True)
    assert la == lb
    groups = boot.fft_groups(prm.N, bp.fft_levels, inverse=True)
    n_ks = sum(len(g) for g in groups) * 2            # >= the key-switches of either schedule
    dmax = max(np.max(np.abs(v)) for g in groups for v in g.values())
    B = _cts_bound(bp, n_ks, 2 * len(groups), max(1.0, dmax))
    diff = np.max(np.abs(_slot_values(bp, a, la, s) - _slot_values(bp, b, lb, s)))
    assert diff <= B, (diff, B)
    p, lp, sp, _ = boot.bootstrap(bp, ct0, keys, plain=True)
    assert np.max(np.abs(boot.decode_sparse(bp, p, lp, sp * delta / prm.q[0], s) - z)) < 1e-2


def test_constant_plaintext_closed_form():
    """_pt's closed form for a constant slot vector c (round(D Re c) + round(D Im c) X^(N/2)) equals
    encode()'s O(N^2) definition, for the constants and scales bootstrapping uses."""
    bp = boot.tiny()
    prm = bp.prm
    rng = np.random.default_rng(9)
    for scale in (2.0 ** 20, 2.0 ** 36, float(prm.q[3]) * 3.7):
        c = complex(rng.standard_normal(), rng.standard_normal())
        lv = 4
        ids = list(range(lv + 1))
        want = ckks.ntt(prm, ckks.reduce_signed(prm, ckks.encode(prm.N, np.full(prm.N // 2, c), scale), ids), ids)
        assert np.array_equal(boot._pt(bp, np.full(bp.n, c), scale, lv), want)


def test_make_consts_matches_a_real_run(booted):
    """make_consts (the schedule replayed without arithmetic) gives the constants a real run makes."""
    bp, s, z, delta, out, lv, scale = booted
    real = _RUN.get("sparse")
    dlv, dscale, dry = boot.dry_run(bp)
    assert (dlv, dscale) == (lv, scale)
    if real is None:
        real = boot.bootstrap(bp, boot.encrypt_sparse(bp, z, delta, s, 25), boot.boot_keys(bp, s, 500))[3]
    assert set(dry) == set(real) and all(np.array_equal(dry[k], real[k]) for k in real)


def test_boosted_full_slot_bootstrap_decodes():
    """Reading BOOT-S (exact x 2^k scale boosts before both linear transforms, theta's product as a
    Double Rescale, L138): the same full-slot bootstrap decodes, at least as accurately as without
    (the boosts shrink the key-switch noise relative to the message; EvalMod's noise remains)."""
    bp = boot.tiny_full_boost()
    prm = bp.prm
    s = ckks.secret(prm, 51, bp.h)
    keys = boot.boot_keys(bp, s, 600)
    z = synth.complex_slots(53, prm.N // 2)
    delta = 2.0 ** 31
    out, lv, scale, _ = boot.bootstrap(bp, boot.encrypt_sparse(bp, z, delta, s, 55), keys)
    assert lv == bp.top - bp.levels_used() == 1
    assert np.max(np.abs(boot.decode_sparse(bp, out, lv, scale * delta / prm.q[0], s) - z)) < 1e-2


def test_ds_evalmod_bootstrap_decodes():
    """Reading BOOT-S with EvalMod's theta product, Taylor powers and terms and first 4 squarings at
    ~q^2 scale (Double Rescale, L138/L151), the schedule Set-B runs with, at N = 2^12."""
    bp = boot.tiny_full_ds()
    prm = bp.prm
    s = ckks.secret(prm, 51, bp.h)
    keys = boot.boot_keys(bp, s, 600)
    z = synth.complex_slots(53, prm.N // 2)
    delta = 2.0 ** 31
    out, lv, scale, _ = boot.bootstrap(bp, boot.encrypt_sparse(bp, z, delta, s, 55), keys)
    assert lv == bp.top - bp.levels_used() == 2
    # 1e-3 (the single-scale schedule's gate is 1e-2, measured 5.0e-3; this one measures 1.8e-4: the
    # noise EvalMod amplifies now enters at ~2^72 scale, what remains is the last 4 squarings' and
    # the sine's noise at ~2^36, amplified at most 2^4)
    assert np.max(np.abs(boot.decode_sparse(bp, out, lv, scale * delta / prm.q[0], s) - z)) < 1e-3
