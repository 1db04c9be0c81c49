"""GPU parity of the application traces (reading APP): the HELR iteration and
the ResNet-20 convolution layer run through the C-ABI (paper_conf_isca_jiaodwfcm0z25_b200.apps)
with the oracle's keys and plaintext constants are bit-exact against oracle/apps.py and decode
to the plaintext computation; neo_pmult_acc equals PMULT + HADD residue for residue."""
import math

import numpy as np
import pytest
import torch

import synth
from oracle import apps, ckks
from test_oracle_apps import DELTA, TOL, app_params

pytestmark = pytest.mark.gpu

neo = pytest.importorskip("paper_conf_isca_jiaodwfcm0z25_b200.neo")
gapps = pytest.importorskip("paper_conf_isca_jiaodwfcm0z25_b200.apps")


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.uint64)).cuda()


def gpu_keys(ctx, keys_np, hoisted=()):
    keys = {k: neo.EvalKey(ctx, dev(v)) for k, v in keys_np.items()}
    for g in hoisted:
        keys[("h", g)] = neo.EvalKey(ctx, dev(keys_np[g]), hoisted_galois=g)
    return keys


def test_helr_iteration_bit_exact_and_decodes():
    prm = app_params()
    sh = apps.HelrShape(prm.N, f=16, batch=3, gamma=2.0)
    assert gapps.helr_rotations(prm.N, sh.f) == sh.rotations()
    s = ckks.secret(prm, 31, 64)
    keys_np = apps.app_keys(prm, s, sh.rotations(), 700)
    Z = 2.0 * synth.uniform_unit(synth.derive(41, 1), sh.n * sh.f).reshape(sh.n, sh.f) - 1.0
    w = (2.0 * synth.uniform_unit(synth.derive(41, 2), sh.f) - 1.0) / math.sqrt(sh.f)
    zs, wv = apps.helr_pack(sh, Z, w)
    L = prm.max_level
    Zs = [apps.encrypt_slots(prm, zs[b], DELTA, s, L, 50 + b) for b in range(sh.batch)]
    W = apps.encrypt_slots(prm, wv, DELTA, s, L, 60)
    want, consts, _ = apps.helr_iteration(sh, prm, Zs, W, keys_np)
    assert sorted(consts) == sorted(gapps.helr_const_names())

    ctx = neo.Context(prm.log_n, prm.num_q, prm.num_p, prm.dnum)
    ev = gapps.Evaluator(ctx, gpu_keys(ctx, keys_np), {k: dev(v) for k, v in consts.items()}, max_batch=sh.batch)
    Zd = dev(np.stack([z[0] for z in Zs]))
    got, lv = gapps.helr_iteration(ev, sh.f, Zd, dev(W[0][None]), L)
    torch.cuda.synchronize()
    assert lv == want[1]
    got = got.cpu().numpy()[0]
    assert np.array_equal(got, want[0])
    dec = np.real(apps.decrypt_slots(prm, (got, lv, want[2]), s))
    assert np.max(np.abs(dec.reshape(sh.rows, sh.f) - apps.helr_plain(sh, Z, w)[None, :])) < TOL


def test_conv_layer_bit_exact_and_decodes():
    prm = app_params()
    sh = apps.ConvShape(prm.N, C=4, H=8)
    baby, giant = sh.rotations()
    assert gapps.conv_rotations(sh.C, sh.H) == (baby, giant)
    s = ckks.secret(prm, 33, 64)
    keys_np = apps.app_keys(prm, s, baby + giant, 800)
    x = 2.0 * synth.uniform_unit(synth.derive(43, 1), sh.C * sh.H * sh.H).reshape(sh.C, sh.H, sh.H) - 1.0
    w = (2.0 * synth.uniform_unit(synth.derive(43, 2), sh.C * sh.C * 9).reshape(sh.C, sh.C, 3, 3) - 1.0) / 6.0
    bias = 0.2 * (2.0 * synth.uniform_unit(synth.derive(43, 3), sh.C) - 1.0)
    L = prm.max_level
    X = apps.encrypt_slots(prm, apps.conv_pack(sh, x), DELTA, s, L, 70)
    want, consts, _ = apps.conv_layer(sh, prm, X, w, bias, keys_np)
    assert sorted(consts) == sorted(gapps.conv_const_names(sh.C))

    ctx = neo.Context(prm.log_n, prm.num_q, prm.num_p, prm.dnum)
    hoisted = [gapps.galois(prm.N, r) for r in baby]
    ev = gapps.Evaluator(ctx, gpu_keys(ctx, keys_np, hoisted), {k: dev(v) for k, v in consts.items()})
    got, lv = gapps.conv_layer(ev, sh.C, sh.H, dev(X[0][None]), L)
    torch.cuda.synchronize()
    assert lv == want[1]
    got = got.cpu().numpy()[0]
    assert np.array_equal(got, want[0])
    dec = apps.conv_unpack(sh, apps.decrypt_slots(prm, (got, lv, want[2]), s))
    assert np.max(np.abs(dec - apps.conv_plain(sh, x, w, bias))) < TOL


@pytest.mark.parametrize("n_terms,batch,shared", [(1, 1, True), (9, 2, False), (32, 3, True)])
def test_pmult_acc_matches_pmult_hadd(n_terms, batch, shared):
    prm = app_params()
    lv = 6
    ids = list(range(lv + 1))
    mods = [prm.moduli[i] for i in ids]
    cts = [np.stack([np.stack([synth.uniform_residues(1000 + 7 * k + 3 * b + c, mods, prm.N) for c in range(2)])
                     for b in range(batch)]) for k in range(n_terms)]
    pts = [synth.uniform_residues(2000 + k, mods, prm.N) if shared else
           np.stack([synth.uniform_residues(3000 + 5 * k + b, mods, prm.N) for b in range(batch)])
           for k in range(n_terms)]
    want = np.empty_like(cts[0])
    for b in range(batch):
        acc = None
        for k in range(n_terms):
            t = ckks.pmult(prm, cts[k][b], pts[k] if shared else pts[k][b], lv)
            acc = t if acc is None else ckks.hadd(prm, acc, t, lv)
        want[b] = acc
    ctx = neo.Context(prm.log_n, prm.num_q, prm.num_p, prm.dnum)
    out = torch.empty(want.shape, dtype=torch.uint64, device="cuda")
    neo.neo_pmult_acc(ctx, [dev(c) for c in cts], [dev(p) for p in pts], lv, out, batch, pt_shared=shared)
    torch.cuda.synchronize()
    assert np.array_equal(out.cpu().numpy(), want)


def test_pmult_acc_rejects_bad_arguments():
    prm = app_params()
    ctx = neo.Context(prm.log_n, prm.num_q, prm.num_p, prm.dnum)
    ct = torch.zeros((1, 2, 3, prm.N), dtype=torch.uint64, device="cuda")
    pt = torch.zeros((3, prm.N), dtype=torch.uint64, device="cuda")
    with pytest.raises(neo.NeoError):
        neo.neo_pmult_acc(ctx, [ct] * 33, [pt] * 33, 2, torch.empty_like(ct), 1, pt_shared=True)
    with pytest.raises(neo.NeoError):
        neo.neo_pmult_acc(ctx, [ct], [pt], 2, ct, 1, pt_shared=True)          # aliasing
    with pytest.raises(neo.NeoError):
        neo.neo_pmult_acc(ctx, [ct], [pt], prm.max_level + 1, torch.empty_like(ct), 1, pt_shared=True)


def test_resnet_block_and_head_bit_exact():
    """The ResNet-20 layer mix (reading R4): a stride-1 basic block then the head, GPU vs oracle bit
    for bit, decoding to the plain computation."""
    from test_oracle_apps import block_inputs, block_params
    prm = block_params()
    sh = apps.ConvShape(prm.N, C=4, H=8)
    s = ckks.secret(prm, 35, 64)
    baby, giant = sh.rotations()
    pool_r, fc_r = apps.head_rotations(sh)
    assert gapps.head_rotations(sh.C, sh.H) == (pool_r, fc_r)
    keys_np = apps.app_keys(prm, s, baby + giant + pool_r, 810)
    x, w1, b1, w2, b2, wfc, bfc = block_inputs(sh)
    L = prm.max_level
    X = apps.encrypt_slots(prm, apps.conv_pack(sh, x), DELTA, s, L, 71)
    want_b, cb, _ = apps.basic_block(sh, prm, X, w1, b1, w2, b2, keys_np)
    want_h, ch, _ = apps.head(sh, prm, want_b, wfc, bfc, keys_np)
    assert sorted(cb) == sorted(gapps.block_const_names(sh.C)) and sorted(ch) == sorted(gapps.head_const_names(sh.C))
    ctx = neo.Context(prm.log_n, prm.num_q, prm.num_p, prm.dnum)
    hoisted = [gapps.galois(prm.N, r) for r in baby + fc_r]
    consts = {k: dev(v) for k, v in {**cb, **ch}.items()}
    ev = gapps.Evaluator(ctx, gpu_keys(ctx, keys_np, hoisted), consts)
    gb, lb = gapps.basic_block(ev, sh.C, sh.H, dev(X[0][None]), L)
    gh, lh = gapps.head(ev, sh.C, sh.H, gb, lb)
    torch.cuda.synchronize()
    assert (lb, lh) == (want_b[1], want_h[1])
    assert np.array_equal(gb.cpu().numpy()[0], want_b[0])
    assert np.array_equal(gh.cpu().numpy()[0], want_h[0])
    z = np.real(apps.decrypt_slots(prm, (gh.cpu().numpy()[0], lh, want_h[2]), s))
    got = z[: 3 * sh.H * sh.H: sh.H * sh.H]
    assert np.max(np.abs(got - apps.head_plain(apps.block_plain(sh, x, w1, b1, w2, b2), wfc, bfc))) < TOL
