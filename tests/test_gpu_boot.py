"""GPU parity of bootstrapping (reading BOOT): the GPU run of
paper_conf_isca_jiaodwfcm0z25_b200.boot with the oracle's keys and plaintext constants is
bit-exact against oracle/boot.py, and decodes to the input slots."""
import numpy as np
import pytest
import torch

import synth
from oracle import boot, ckks

pytestmark = pytest.mark.gpu

neo = pytest.importorskip("paper_conf_isca_jiaodwfcm0z25_b200.neo")
gboot = pytest.importorskip("paper_conf_isca_jiaodwfcm0z25_b200.boot")


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.uint64)).cuda()


def test_bootstrap_bit_exact_and_decodes():
    bp = boot.tiny()
    prm = bp.prm
    s = ckks.secret(prm, 21, bp.h)
    keys_np = boot.boot_keys(bp, s, 500)
    z = synth.complex_slots(23, bp.n)
    delta = 2.0 ** 31
    ct0 = boot.encrypt_sparse(bp, z, delta, s, 25)
    want, lv, scale, consts = boot.bootstrap(bp, ct0, keys_np)

    ctx = neo.Context(prm.log_n, prm.num_q, prm.num_p, prm.dnum)
    assert gboot.rotations(prm.N, bp.n) == bp.rotations()
    keys = {k: neo.EvalKey(ctx, dev(v)) for k, v in keys_np.items()}
    for g in gboot.hoisted_rotations(prm.N, bp.n):
        keys[("h", g)] = neo.EvalKey(ctx, dev(keys_np[g]), hoisted_galois=g)
    cl = gboot.const_levels(bp.top, bp.n, bp.r)
    assert set(cl) == set(consts) and all(consts[k].shape[0] == cl[k] + 1 for k in cl)
    b = gboot.Bootstrapper(ctx, bp.n, bp.r, keys, {k: dev(v) for k, v in consts.items()})
    got, glv = b.run(dev(ct0[None]))
    torch.cuda.synchronize()
    assert glv == lv
    got = got.cpu().numpy()[0]
    assert np.array_equal(got, want)
    zz = boot.decode_sparse(bp, got, lv, scale * delta / prm.q[0], s)
    assert np.max(np.abs(zz - z)) < 4e-3


def test_bootstrap_graph_replay_bit_exact():
    """The bootstrap captured as one CUDA graph (how bench.py times it) replays to the oracle's
    result."""
    bp = boot.tiny()
    prm = bp.prm
    s = ckks.secret(prm, 21, bp.h)
    keys_np = boot.boot_keys(bp, s, 500)
    ct0 = boot.encrypt_sparse(bp, synth.complex_slots(23, bp.n), 2.0 ** 31, s, 25)
    want, lv, scale, consts = boot.bootstrap(bp, ct0, keys_np)
    ctx = neo.Context(prm.log_n, prm.num_q, prm.num_p, prm.dnum)
    keys = {k: neo.EvalKey(ctx, dev(v)) for k, v in keys_np.items()}
    for g in gboot.hoisted_rotations(prm.N, bp.n):
        keys[("h", g)] = neo.EvalKey(ctx, dev(keys_np[g]), hoisted_galois=g)
    b = gboot.Bootstrapper(ctx, bp.n, bp.r, keys, {k: dev(v) for k, v in consts.items()})
    x = dev(ct0[None])
    side = torch.cuda.Stream()
    side.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(side):
        b.run(x)
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=side):
            out, glv = b.run(x)
    torch.cuda.current_stream().wait_stream(side)
    out.zero_()
    g.replay()
    torch.cuda.synchronize()
    assert glv == lv and np.array_equal(out.cpu().numpy()[0], want)


@pytest.mark.parametrize("fft_levels", [3, 4])
def test_full_slot_bootstrap_bit_exact_and_decodes(fft_levels):
    """All N/2 slots: factored CoeffToSlot / SlotToCoeff (3 BSGS levels each, hoisted baby steps,
    fused PMULT sums) + EvalMod, bit-exact vs oracle/boot.py and decoding to the input."""
    bp = boot.tiny_full(fft_levels)
    prm = bp.prm
    s = ckks.secret(prm, 51, bp.h)
    keys_np = boot.boot_keys(bp, s, 600)
    z = synth.complex_slots(53, prm.N // 2)
    delta = 2.0 ** 31
    ct0 = boot.encrypt_sparse(bp, z, delta, s, 55)
    want, lv, scale, consts = boot.bootstrap(bp, ct0, keys_np)
    ctx = neo.Context(prm.log_n, prm.num_q, prm.num_p, prm.dnum)
    assert gboot.rotations(prm.N, bp.n, bp.fft_levels) == bp.rotations()
    cl = gboot.const_levels(bp.top, bp.n, bp.r, prm.N, bp.fft_levels)
    assert set(cl) == set(consts) and all(consts[k].shape[0] == cl[k] + 1 for k in cl)
    keys = {k: neo.EvalKey(ctx, dev(v)) for k, v in keys_np.items()}
    for g in gboot.hoisted_rotations(prm.N, bp.n, bp.fft_levels):
        keys[("h", g)] = neo.EvalKey(ctx, dev(keys_np[g]), hoisted_galois=g)
    b = gboot.Bootstrapper(ctx, bp.n, bp.r, keys, {k: dev(v) for k, v in consts.items()}, fft_levels=bp.fft_levels)
    got, glv = b.run(dev(ct0[None]))
    torch.cuda.synchronize()
    assert glv == lv
    got = got.cpu().numpy()[0]
    assert np.array_equal(got, want)
    zz = boot.decode_sparse(bp, got, lv, scale * delta / prm.q[0], s)
    assert np.max(np.abs(zz - z)) < 1e-2          # test_oracle_boot.py: sqrt(N) slot gain
