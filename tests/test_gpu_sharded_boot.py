"""GPU: limb-sharded evaluation and bootstrapping (paper_conf_isca_jiaodwfcm0z25_b200.sharded_boot;
SURVEY §8(f) row 2 / config 4) with 1 rank and with 2 ranks sharing cuda:0 over gloo (on an
8-GPU box the same code exchanges over NCCL).  Every rank's rows of HMULT+Rescale, HROTATE,
ModRaise and of the whole bootstrap are compared with the oracle bit for bit."""
import os
import socket
import sys
import tempfile

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(rank, world, port, path, q, full=False):
    try:
        q.put((rank, _run_full(rank, world, port) if full else _run_inner(rank, world, port, path)))
    except Exception as e:                       # report instead of hanging the parent
        import traceback
        q.put((rank, "".join(traceback.format_exception(e))))


def _run_inner(rank, world, port, path):
    sys.path.insert(0, ROOT)
    from oracle import boot
    from paper_conf_isca_jiaodwfcm0z25_b200 import boot as gboot
    from paper_conf_isca_jiaodwfcm0z25_b200 import neo
    from paper_conf_isca_jiaodwfcm0z25_b200.sharded_boot import ShardedBootstrapper
    if world > 1:
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)
        z = np.load(path, allow_pickle=True)
        bp = boot.tiny()
        prm = bp.prm
        ctx = neo.Context(prm.log_n, prm.num_q, prm.num_p, prm.dnum)
        dev = lambda a: torch.from_numpy(np.ascontiguousarray(a, dtype=np.uint64)).cuda()
        keys_np = z["keys"].item()
        keys = {k: neo.EvalKey(ctx, dev(v)) for k, v in keys_np.items()}
        for g in gboot.hoisted_rotations(prm.N, bp.n):
            keys[("h", g)] = neo.EvalKey(ctx, dev(keys_np[g]), hoisted_galois=g)
        consts = {k: dev(v) for k, v in z["consts"].item().items()}
        sb = ShardedBootstrapper(ctx, bp.n, bp.r, keys, consts, world, rank)
        fails = []
        # single ops at level L: HMULT + Rescale, HROTATE, ModRaise
        L = prm.max_level
        a, b = dev(z["a"]), dev(z["b"])
        own = sb.own(L - 1)
        got = sb.hmul_rescale(sb.shard(a, L), sb.shard(b, L), L)
        if not np.array_equal(got.cpu().numpy(), z["hmr"][:, :, own]):
            fails.append("hmult_rescale")
        g5 = pow(5, 1, 2 * prm.N)
        got = sb.rot(sb.shard(a, L), g5, L)
        if not np.array_equal(got.cpu().numpy(), z["hrot"][:, :, sb.own(L)]):
            fails.append("hrot")
        ct0 = dev(z["ct0"][None])
        got = sb.modraise(sb.shard(ct0, 0), L)
        if not np.array_equal(got.cpu().numpy(), z["mr"][None][:, :, sb.own(L)]):
            fails.append("modraise")
        out, lv = sb.run(sb.shard(ct0, 0))
        torch.cuda.synchronize()
        if lv != int(z["lv"]) or not np.array_equal(out.cpu().numpy(), z["boot"][None][:, :, sb.own(lv)]):
            fails.append("bootstrap")
        return True if not fails else fails
    finally:
        if world > 1:
            dist.destroy_process_group()


def _run_full(rank, world, port):
    """Full-slot bootstrap (special-FFT CoeffToSlot / SlotToCoeff) on shards against the
    single-GPU Bootstrapper on the same inputs (bit-exact; the single-GPU full-slot run is
    itself checked against oracle/boot.py in test_gpu_boot.py).  Keys, constants and the input
    are seeded uniform residues: the comparison is exact modular arithmetic, so no oracle run
    (and no multi-GB key file) is needed here."""
    sys.path.insert(0, ROOT)
    import synth
    from oracle import boot
    from paper_conf_isca_jiaodwfcm0z25_b200 import boot as gboot
    from paper_conf_isca_jiaodwfcm0z25_b200 import neo
    from paper_conf_isca_jiaodwfcm0z25_b200.sharded_boot import ShardedBootstrapper
    if world > 1:
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)
        bp = boot.tiny_full()
        prm = bp.prm
        ctx = neo.Context(prm.log_n, prm.num_q, prm.num_p, prm.dnum)
        dev = lambda a: torch.from_numpy(np.ascontiguousarray(a, dtype=np.uint64)).cuda()
        evk = np.stack([np.stack([synth.uniform_residues(800 + 2 * j + c, prm.moduli, prm.N) for c in range(2)])
                        for j in range(prm.dnum)])
        keys = {"relin": neo.EvalKey(ctx, dev(evk))}
        for g in gboot.rotations(prm.N, bp.n, bp.fft_levels):
            keys[g] = neo.EvalKey(ctx, dev(evk))
        for g in gboot.hoisted_rotations(prm.N, bp.n, bp.fft_levels):
            keys[("h", g)] = neo.EvalKey(ctx, dev(evk), hoisted_galois=g)
        cl = gboot.const_levels(bp.top, bp.n, bp.r, prm.N, bp.fft_levels)
        consts = {k: dev(synth.uniform_residues(900 + i, prm.q[: l + 1], prm.N)) for i, (k, l) in
                  enumerate(sorted(cl.items()))}
        ct0 = dev(np.stack([synth.uniform_residues(990 + c, prm.q[:1], prm.N) for c in range(2)])[None])
        ref, lv = gboot.Bootstrapper(ctx, bp.n, bp.r, keys, consts, fft_levels=bp.fft_levels).run(ct0)
        sb = ShardedBootstrapper(ctx, bp.n, bp.r, keys, consts, world, rank, fft_levels=bp.fft_levels)
        out, glv = sb.run(sb.shard(ct0, 0))
        torch.cuda.synchronize()
        ok = glv == lv and np.array_equal(out.cpu().numpy(), ref.cpu().numpy()[:, :, sb.own(lv)])
        return True if ok else ["full-slot bootstrap"]
    finally:
        if world > 1:
            dist.destroy_process_group()


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.fixture(scope="module")
def oracle_file():
    import synth
    from oracle import boot, ckks
    bp = boot.tiny()
    prm = bp.prm
    s = ckks.secret(prm, 21, bp.h)
    keys = boot.boot_keys(bp, s, 500)
    ct0 = boot.encrypt_sparse(bp, synth.complex_slots(23, bp.n), 2.0 ** 31, s, 25)
    want, lv, _, consts = boot.bootstrap(bp, ct0, keys)
    L = prm.max_level
    ids = list(range(L + 1))
    a = np.stack([synth.uniform_residues(700 + c, [prm.moduli[i] for i in ids], prm.N) for c in range(2)])[None]
    b = np.stack([synth.uniform_residues(710 + c, [prm.moduli[i] for i in ids], prm.N) for c in range(2)])[None]
    hmr = ckks.rescale(prm, ckks.hmult(prm, a[0], b[0], L, keys["relin"]), L)[None]
    g5 = pow(5, 1, 2 * prm.N)
    hrot = ckks.hrot(prm, a[0], g5, L, keys[g5])[None]
    mr = boot.modraise(prm, ct0, L)
    d = tempfile.mkdtemp()
    path = os.path.join(d, "sharded_boot.npz")
    np.savez(path, keys=np.array(keys, dtype=object), consts=np.array(consts, dtype=object), ct0=ct0, a=a, b=b,
             hmr=hmr, hrot=hrot, mr=mr, boot=want, lv=lv)
    return path


@pytest.mark.parametrize("world", [1, 2])
def test_sharded_bootstrap_bit_exact(world, oracle_file):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=_run, args=(r, world, port, oracle_file, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=600) for _ in procs)
    for p in procs:
        p.join(timeout=60)
    assert all(res[r] is True for r in range(world)), res


def test_sharded_full_slot_bootstrap_bit_exact():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=_run, args=(r, world, port, None, q, True)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=900) for _ in procs)
    for p in procs:
        p.join(timeout=60)
    assert all(res[r] is True for r in range(world)), res
