"""Oracle pins for the application traces (reading APP in DESIGN.md): the
HELR iteration and the ResNet-20 convolution layer decode to the plaintext computation of the
same formulas (numpy, float64), and the op counts follow the schedule's closed form."""
import math

import numpy as np
import pytest

import synth
from oracle import apps, ckks


def app_params() -> ckks.Params:
    """N = 2^12, 10 Q limbs + 2 P limbs, dnum 5 (alpha = 2): levels for either trace."""
    return ckks.Params(12, 10, 2, 5)


DELTA = 2.0 ** 36                     # ~ q: products and rescales keep every scale near 2^36
# Tolerance (both traces): a key-switch adds sum_j dhat_j e_j / P to the coefficients; with
# alpha = 2 (Q_j ~ P ~ 2^72), beta = 5 digits, N = 4096, sigma = 3.2 its std is about
# sqrt(beta N) 0.58 sigma ~ 2^8, i.e. ~ sqrt(N) 2^8 / 2^36 = 2.4e-7 per slot after a rotation at
# scale 2^36 (the rotations that run at ~2^36 dominate; rescale rounding is ~2^-26 smaller).
# Worst slot of 2048 ~ 4 sigma ~ 1e-6, summed over up to 9 baby-step rotations weighted by
# |w| <= 1/6 (conv) or by gamma/n-scaled sums (HELR): 5e-6 bounds both with margin 2.
TOL = 5e-6


@pytest.fixture(scope="module")
def helr_run():
    prm = app_params()
    sh = apps.HelrShape(prm.N, f=16, batch=2, gamma=2.0)
    s = ckks.secret(prm, 31, 64)
    keys = apps.app_keys(prm, s, sh.rotations(), 700)
    Z = 2.0 * synth.uniform_unit(synth.derive(41, 1), sh.n * sh.f).reshape(sh.n, sh.f) - 1.0
    w = (2.0 * synth.uniform_unit(synth.derive(41, 2), sh.f) - 1.0) / math.sqrt(sh.f)
    zs, wv = apps.helr_pack(sh, Z, w)
    L = prm.max_level
    Zs = [apps.encrypt_slots(prm, zs[b], DELTA, s, L, 50 + b) for b in range(sh.batch)]
    W = apps.encrypt_slots(prm, wv, DELTA, s, L, 60)
    Wn, consts, counts = apps.helr_iteration(sh, prm, Zs, W, keys)
    return prm, sh, s, Z, w, Wn, counts, consts, Zs, W


def test_helr_iteration_decodes_to_plain_step(helr_run):
    prm, sh, s, Z, w, Wn, counts, *_ = helr_run
    got = np.real(apps.decrypt_slots(prm, Wn, s))
    want = apps.helr_plain(sh, Z, w)
    assert Wn[1] == prm.max_level - apps.HELR_LEVELS
    assert np.max(np.abs(got.reshape(sh.rows, sh.f) - want[None, :])) < TOL
    # the step moved w (the check is not vacuous)
    assert np.max(np.abs(want - w)) > 1e-2


def test_helr_op_counts(helr_run):
    prm, sh, s, Z, w, Wn, counts, *_ = helr_run
    lf, lr = int(math.log2(sh.f)), int(math.log2(sh.rows))
    B = sh.batch
    assert counts["hmult"] == 4 * B
    assert counts["hrot"] == (2 * lf + lr) * B
    assert counts["pmult"] == 3 * B + 1
    assert counts["rescale"] == 7 * B + 1


@pytest.fixture(scope="module")
def conv_run():
    prm = app_params()
    sh = apps.ConvShape(prm.N, C=4, H=8)
    s = ckks.secret(prm, 33, 64)
    baby, giant = sh.rotations()
    keys = apps.app_keys(prm, s, baby + giant, 800)
    x = 2.0 * synth.uniform_unit(synth.derive(43, 1), sh.C * sh.H * sh.H).reshape(sh.C, sh.H, sh.H) - 1.0
    w = (2.0 * synth.uniform_unit(synth.derive(43, 2), sh.C * sh.C * 9).reshape(sh.C, sh.C, 3, 3) - 1.0) / 6.0
    bias = 0.2 * (2.0 * synth.uniform_unit(synth.derive(43, 3), sh.C) - 1.0)
    L = prm.max_level
    X = apps.encrypt_slots(prm, apps.conv_pack(sh, x), DELTA, s, L, 70)
    out, consts, counts = apps.conv_layer(sh, prm, X, w, bias, keys)
    return prm, sh, s, x, w, bias, out, counts


def test_conv_layer_decodes_to_plain_layer(conv_run):
    prm, sh, s, x, w, bias, out, counts = conv_run
    z = apps.decrypt_slots(prm, out, s)
    got = apps.conv_unpack(sh, z)
    want = apps.conv_plain(sh, x, w, bias)
    assert out[1] == prm.max_level - apps.CONV_LEVELS
    assert np.max(np.abs(got - want)) < TOL
    # every tiled copy holds the same layer output
    blk = sh.C * sh.H * sh.H
    zz = np.real(z).reshape(-1, blk)
    assert np.max(np.abs(zz - zz[0])) < TOL


def test_conv_plain_matches_direct_definition():
    """conv_plain's loop nest against an independent gather formulation on one output pixel."""
    sh = apps.ConvShape(4096, C=3, H=5)
    rng = np.random.default_rng(9)
    x, w, b = rng.standard_normal((3, 5, 5)), rng.standard_normal((3, 3, 3, 3)), rng.standard_normal(3)
    got = apps.conv_plain(sh, x, w, b)
    co, y0, x0 = 2, 0, 3
    acc = b[co]
    for ci in range(3):
        for ky in range(3):
            for kx in range(3):
                yy, xx = y0 + ky - 1, x0 + kx - 1
                if 0 <= yy < 5 and 0 <= xx < 5:
                    acc += w[co, ci, ky, kx] * x[ci, yy, xx]
    a0, a1, a2, a4 = apps.RELU_A
    assert abs(got[co, y0, x0] - (a0 + a1 * acc + a2 * acc ** 2 + a4 * acc ** 4)) < 1e-12


def test_relu_polynomial_is_the_legendre_fit():
    """a(x) = (x + p(x)) / 2 with p the L2-optimal even quartic for |x| on [-1, 1]:
    the residual |x| - p(x) is orthogonal to 1, x^2 and x^4."""
    a0, a1, a2, a4 = apps.RELU_A
    assert a1 == 0.5
    xs = np.linspace(-1, 1, 200001)
    r = np.abs(xs) - 2 * (a0 + a2 * xs ** 2 + a4 * xs ** 4)
    for k in (0, 2, 4):
        assert abs(np.trapezoid(r * xs ** k, xs)) < 1e-6


def test_conv_op_counts(conv_run):
    prm, sh, s, x, w, bias, out, counts = conv_run
    assert counts["hrot"] == 8 + (sh.C - 1)
    assert counts["pmult"] == 9 * sh.C + 3
    assert counts["hmult"] == 2


def block_params() -> ckks.Params:
    """N = 2^12, 13 Q limbs + 2 P limbs, dnum 7 (alpha = 2): 12 levels for a block + the head."""
    return ckks.Params(12, 13, 2, 7)


def block_inputs(sh):
    r = lambda k, n: synth.uniform_unit(synth.derive(47, k), n)
    x = 2.0 * r(1, sh.C * sh.H * sh.H).reshape(sh.C, sh.H, sh.H) - 1.0
    w1 = (2.0 * r(2, sh.C * sh.C * 9).reshape(sh.C, sh.C, 3, 3) - 1.0) / 6.0
    w2 = (2.0 * r(3, sh.C * sh.C * 9).reshape(sh.C, sh.C, 3, 3) - 1.0) / 6.0
    b1, b2 = 0.2 * (2.0 * r(4, sh.C) - 1.0), 0.2 * (2.0 * r(5, sh.C) - 1.0)
    wfc = (2.0 * r(6, 3 * sh.C).reshape(3, sh.C) - 1.0) / 2.0
    bfc = 0.1 * (2.0 * r(7, 3) - 1.0)
    return x, w1, b1, w2, b2, wfc, bfc


def test_block_plain_is_the_residual_definition():
    """block_plain = relu(conv2(relu(conv1 x)) + x) with conv_plain's convolution (pinned above)."""
    sh = apps.ConvShape(4096, C=3, H=5)
    rng = np.random.default_rng(4)
    x, w1, w2 = rng.standard_normal((3, 5, 5)), rng.standard_normal((3, 3, 3, 3)), rng.standard_normal((3, 3, 3, 3))
    b1, b2 = rng.standard_normal(3), rng.standard_normal(3)
    assert np.allclose(apps.relu_poly(apps.conv_linear_plain(sh, x, w1, b1)), apps.conv_plain(sh, x, w1, b1))
    h = apps.conv_plain(sh, x, w1, b1)
    want = apps.relu_poly(apps.conv_linear_plain(sh, h, w2, b2) + x)
    assert np.allclose(apps.block_plain(sh, x, w1, b1, w2, b2), want)


def test_resnet_block_and_head_decode():
    """A stride-1 ResNet-20 basic block then the network head (pooling + FC) decode to the plain
    computation (tolerance as above: the block's key-switches and rescales at ~2^36 scales)."""
    prm = block_params()
    sh = apps.ConvShape(prm.N, C=4, H=8)
    s = ckks.secret(prm, 35, 64)
    baby, giant = sh.rotations()
    pool_r, fc_r = apps.head_rotations(sh)
    keys = apps.app_keys(prm, s, baby + giant + pool_r, 810)
    x, w1, b1, w2, b2, wfc, bfc = block_inputs(sh)
    L = prm.max_level
    X = apps.encrypt_slots(prm, apps.conv_pack(sh, x), DELTA, s, L, 71)
    out, _, counts = apps.basic_block(sh, prm, X, w1, b1, w2, b2, keys)
    assert out[1] == L - apps.BLOCK_LEVELS
    want_b = apps.block_plain(sh, x, w1, b1, w2, b2)
    got_b = apps.conv_unpack(sh, apps.decrypt_slots(prm, out, s))
    assert np.max(np.abs(got_b - want_b)) < TOL
    assert counts["hrot"] == 2 * (8 + sh.C - 1) and counts["hmult"] == 4
    hd, _, hc = apps.head(sh, prm, out, wfc, bfc, keys)
    z = np.real(apps.decrypt_slots(prm, hd, s))
    got_h = z[: 3 * sh.H * sh.H: sh.H * sh.H]
    assert np.max(np.abs(got_h - apps.head_plain(want_b, wfc, bfc))) < TOL
    assert hc["hrot"] == len(pool_r) + sh.C - 1


def test_dry_run_gives_the_same_constants(helr_run):
    """apps.DryEv (no ciphertext arithmetic, used for the Set-B GPU decode tests) makes exactly the
    constants, levels and scales the full evaluation makes: HELR and the convolution layer."""
    prm, sh, s, Z, w, Wn, counts, consts, Zs, W = helr_run
    dry_in = [(None, z[1], z[2]) for z in Zs]
    Wd, cd, nd = apps.helr_iteration(sh, prm, dry_in, (None, W[1], W[2]), {}, dry=True)
    assert (Wd[1], Wd[2]) == (Wn[1], Wn[2]) and nd == counts
    assert sorted(cd) == sorted(consts) and all(np.array_equal(cd[k], consts[k]) for k in consts)
    sh2 = apps.ConvShape(prm.N, C=4, H=8)
    baby, giant = sh2.rotations()
    keys = apps.app_keys(prm, s, baby + giant, 800)
    x = 2.0 * synth.uniform_unit(synth.derive(43, 1), sh2.C * sh2.H * sh2.H).reshape(sh2.C, sh2.H, sh2.H) - 1.0
    wc = (2.0 * synth.uniform_unit(synth.derive(43, 2), sh2.C * sh2.C * 9).reshape(sh2.C, sh2.C, 3, 3) - 1.0) / 6.0
    bias = 0.2 * (2.0 * synth.uniform_unit(synth.derive(43, 3), sh2.C) - 1.0)
    X = apps.encrypt_slots(prm, apps.conv_pack(sh2, x), DELTA, s, prm.max_level, 70)
    out, cc, nc = apps.conv_layer(sh2, prm, X, wc, bias, keys)
    outd, ccd, ncd = apps.conv_layer(sh2, prm, (None, X[1], X[2]), wc, bias, {}, dry=True)
    assert (outd[1], outd[2]) == (out[1], out[2]) and ncd == nc
    assert sorted(ccd) == sorted(cc) and all(np.array_equal(ccd[k], cc[k]) for k in cc)
