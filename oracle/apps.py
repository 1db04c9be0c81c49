"""CPU ORACLE of the CKKS application traces (BASELINE configs[4]) -- TEST
INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
``--impl reference`` legs may import this module; it shares no code with the CUDA path.

The paper evaluates two applications besides bootstrapping (§5; Table 5):
HELR [17, 18] (logistic-regression training, 196 features of 14x14 MNIST images, batches of
1,024 images, one iteration timed) and ResNet-20 inference [32] on a 32x32x3 CIFAR-10 image.
It prints only their total times and no operation counts, so the traces are readings
("APP" in DESIGN.md), built only from the pinned operations (HMULT, HROTATE, hoisted HROTATE,
PMULT, HADD, PADD, Rescale):

HELR iteration (reading H1-H4).  n = rows x B samples, f features (196 -> f = 256 at Set-B);
ciphertext b packs rows x f values z_{i,j} = y_i x_{i,j} row-major (slot i f + j); W packs
the weight w_j replicated over the rows.  One gradient-ascent step on the log-likelihood,
    w <- w + (gamma / n) sum_i sigma3(-z_i . w) z_i,   sigma3(x) = 0.5 + 0.15012 x - 0.001593 x^3
(HELR's degree-3 least-squares sigmoid on [-8, 8]), evaluated as
    1  T = Rescale(HMULT(Z_b, W))                     z_{i,j} w_j
    2  T += HROT(T, 2^k), k < log f                    slot i f: z_i . w
    3  T = Rescale(PMULT(T, mask))                     keep slot i f
    4  T += HROT(T, -2^k), k < log f                   replicate over the row
    5  S = 0.5 - 0.15012 T + 0.001593 T^3              (T^2, 0.001593 T, their product)
    6  G = Rescale(HMULT(S, Z_b))
    7  G += HROT(G, f 2^k), k < log rows               sum over the rows of a ciphertext
    8  G = sum_b G_b                                   sum over the batch
    9  W' = W + Rescale(PMULT(G, gamma / n))           six levels in all

ResNet-20 layer (reading R1-R3): one convolution block of the first stage of [32]'s network,
C channels of H x H (16 x 32 x 32 at Set-B), channel c at slots [c H^2, (c+1) H^2), tiled to
fill N/2 slots:
    1  R_o = HROT(X, o) for the 8 offsets o = dy H + dx (hoisted: one ModUp)
    2  Y = sum_d HROT( sum_o PMULT(R_o, V_{d,o}), d H^2 )  then Rescale   (baby-step giant-step
       diagonal method: V_{d,o} = rot_{-d H^2}(w[c][c + d][dy][dx] masked at the image border))
    3  Y = PADD(Y, bias)
    4  out = a0 + a1 Y + a2 Y^2 + a4 Y^4     (ReLU(x) = (x + |x|)/2 with the Legendre
       least-squares |x| ~ 15/128 + 105/64 x^2 - 105/128 x^4 on [-1, 1]); four levels in all
The convolution is 3 x 3, stride 1, zero padding, C -> C channels.

Every plaintext constant is encoded at a scale chosen so that the following Rescale lands
exactly on the tracked target scale (the same discipline as oracle/boot.py), and returned, so
the GPU run (paper_conf_isca_jiaodwfcm0z25_b200/apps.py) replays the same operands.  Pinned by
decoding against the plaintext computation (tests/test_oracle_apps.py)."""
from __future__ import annotations

import math
from dataclasses import dataclass

import numpy as np

from . import ckks

SIG_C1, SIG_C3 = 0.15012, -0.001593            # sigma3(x) = 0.5 + C1 x + C3 x^3 (HELR [17])
RELU_A = (15 / 256, 0.5, 105 / 128, -105 / 256)  # a0, a1, a2, a4 (ReLU from the |x| fit)


def _g(N: int, r: int) -> int:
    """Galois element of a left rotation by r slots (Z11), r taken mod N/2."""
    return pow(5, r % (N // 2), 2 * N)


def _encode(N: int, z, scale: float) -> np.ndarray:
    """ckks.encode below N = 2^14; its one-FFT evaluation encode_fft above (within 1 of encode,
    pinned in tests/test_oracle_ntt.py; any valid encoding -- as for bootstrapping, reading BOOT-F)."""
    z = np.asarray(z, dtype=complex)
    return ckks.encode(N, z, scale) if N < (1 << 14) else ckks.encode_fft(N, z, scale)


def _enc(prm: ckks.Params, slots, scale: float, level: int) -> np.ndarray:
    """Plaintext (NTT form, [level+1][N]) of the slot vector `slots` (length N/2) at `scale`."""
    ids = list(range(level + 1))
    m = _encode(prm.N, slots, scale)
    return ckks.ntt(prm, ckks.reduce_signed(prm, m, ids), ids)


def _drop(ct: np.ndarray, level: int) -> np.ndarray:
    return np.ascontiguousarray(ct[:, : level + 1])


class Ev:
    """Scale-tracking evaluator over the oracle's pinned operations.  A value is
    (ct [2][l+1][N], level, scale).  `consts` (name -> plaintext) are made on first use when
    generating, else read (replay)."""

    def __init__(self, prm: ckks.Params, keys: dict, consts: dict | None = None):
        self.prm, self.keys = prm, keys
        self.gen = consts is None
        self.consts = {} if consts is None else consts
        self.counts = {"hmult": 0, "hrot": 0, "pmult": 0, "hadd": 0, "padd": 0, "rescale": 0}

    def const(self, name, slots, scale, level):
        # precision guard: the encoded constant must carry >= 24 bits (rounding <= 2^-25 relative)
        assert scale * np.max(np.abs(slots)) >= 2.0 ** 24, (name, scale)
        if self.gen:
            self.consts[name] = _enc(self.prm, slots, scale, level)
        return self.consts[name]

    def rescale(self, v):
        ct, l, s = v
        self.counts["rescale"] += 1
        return ckks.rescale(self.prm, ct, l), l - 1, s / self.prm.q[l]

    def drop(self, v, level):
        ct, l, s = v
        return _drop(ct, level), level, s

    def add(self, a, b):
        (ca, la, sa), (cb, lb, sb) = a, b
        assert la == lb and abs(sa - sb) <= 1e-9 * sa, (la, lb, sa, sb)
        self.counts["hadd"] += 1
        return ckks.hadd(self.prm, ca, cb, la), la, sa

    def mul(self, a, b):
        (ca, la, sa), (cb, lb, sb) = a, b
        assert la == lb
        self.counts["hmult"] += 1
        return ckks.hmult(self.prm, ca, cb, la, self.keys["relin"]), la, sa * sb

    def rot(self, v, r):
        ct, l, s = v
        g = _g(self.prm.N, r)
        self.counts["hrot"] += 1
        return ckks.hrot(self.prm, ct, g, l, self.keys[g]), l, s

    def rot_hoisted(self, v, rs):
        ct, l, s = v
        gs = [_g(self.prm.N, r) for r in rs]
        self.counts["hrot"] += len(rs)
        outs = ckks.hrot_hoisted(self.prm, ct, gs, l, [self.keys[g] for g in gs])
        return [(o, l, s) for o in outs]

    def pmul(self, v, name, slots, scale):
        ct, l, s = v
        self.counts["pmult"] += 1
        return ckks.pmult(self.prm, ct, self.const(name, slots, scale, l), l), l, s * scale

    def padd(self, v, name, slots):
        ct, l, s = v
        self.counts["padd"] += 1
        return ckks.padd(self.prm, ct, self.const(name, slots, s, l), l), l, s

    def pmul_to(self, v, name, slots, target):
        """Rescale(PMULT(v, slots)) with the constant's scale chosen so the result has `target`."""
        ct, l, s = v
        return self.rescale(self.pmul(v, name, slots, target * self.prm.q[l] / s))


class DryEv(Ev):
    """Ev without the ciphertext arithmetic: levels and scales tracked exactly as Ev tracks them,
    plaintext constants made as Ev makes them.  A value is (None, level, scale).  Gives the
    constants of a trace at sizes where running the oracle's ciphertext arithmetic is too slow
    (Set-B); the GPU run with those constants is then checked by decryption."""

    def __init__(self, prm: ckks.Params):
        super().__init__(prm, {}, None)

    def rescale(self, v):
        _, l, s = v
        self.counts["rescale"] += 1
        return None, l - 1, s / self.prm.q[l]

    def drop(self, v, level):
        return None, level, v[2]

    def add(self, a, b):
        (_, la, sa), (_, lb, sb) = a, b
        assert la == lb and abs(sa - sb) <= 1e-9 * sa, (la, lb, sa, sb)
        self.counts["hadd"] += 1
        return None, la, sa

    def mul(self, a, b):
        (_, la, sa), (_, lb, sb) = a, b
        assert la == lb
        self.counts["hmult"] += 1
        return None, la, sa * sb

    def rot(self, v, r):
        self.counts["hrot"] += 1
        return None, v[1], v[2]

    def rot_hoisted(self, v, rs):
        self.counts["hrot"] += len(rs)
        return [(None, v[1], v[2]) for _ in rs]

    def pmul(self, v, name, slots, scale):
        _, l, s = v
        self.counts["pmult"] += 1
        self.const(name, slots, scale, l)
        return None, l, s * scale

    def padd(self, v, name, slots):
        _, l, s = v
        self.counts["padd"] += 1
        self.const(name, slots, s, l)
        return None, l, s


def _ev(prm, keys, consts, dry):
    return DryEv(prm) if dry else Ev(prm, keys, consts)


# --------------------------------------------------------------------------- HELR

@dataclass
class HelrShape:
    N: int
    f: int                   # features per sample (power of two)
    batch: int               # ciphertexts per iteration
    gamma: float = 1.0       # learning rate

    @property
    def rows(self) -> int:
        return self.N // 2 // self.f

    @property
    def n(self) -> int:
        return self.rows * self.batch

    def rotations(self) -> list[int]:
        """Left-rotation amounts of steps 2, 4 and 7."""
        lf, lr = int(math.log2(self.f)), int(math.log2(self.rows))
        return [1 << k for k in range(lf)] + [-(1 << k) for k in range(lf)] + [self.f << k for k in range(lr)]


HELR_LEVELS = 6


def helr_pack(sh: HelrShape, Z: np.ndarray, w: np.ndarray):
    """Z [n][f] (z_i = y_i x_i), w [f] -> slot vectors: Z_b [batch][N/2], W [N/2]."""
    zs = Z.reshape(sh.batch, sh.rows * sh.f)
    return zs, np.tile(w, sh.rows)


def helr_plain(sh: HelrShape, Z: np.ndarray, w: np.ndarray) -> np.ndarray:
    """The plaintext iteration (the same sigma3): w + gamma/n sum_i sigma3(-z_i . w) z_i."""
    ip = Z @ w
    s = 0.5 - SIG_C1 * ip - SIG_C3 * ip ** 3
    return w + sh.gamma / sh.n * (s @ Z)


def helr_iteration(sh: HelrShape, prm: ckks.Params, Zs: list, W, keys: dict, consts: dict | None = None,
                   dry: bool = False):
    """Zs: list of `batch` values (ct, level, scale); W likewise (same level and scale).
    Returns (W', consts, counts); W' = (ct, level - 6, W's scale).  dry: constants only (DryEv)."""
    ev = _ev(prm, keys, consts, dry)
    N, f, rows = sh.N, sh.f, sh.rows
    lf, lr = int(math.log2(f)), int(math.log2(rows))
    half = N // 2
    mask = np.zeros(half)
    mask[::f] = 1.0
    Gs = []
    for b, Z in enumerate(Zs):
        T = ev.rescale(ev.mul(Z, W))                              # 1
        for k in range(lf):                                       # 2
            T = ev.add(T, ev.rot(T, 1 << k))
        T = ev.rescale(ev.pmul(T, "mask", mask, float(prm.q[T[1]])))   # 3
        for k in range(lf):                                       # 4
            T = ev.add(T, ev.rot(T, -(1 << k)))
        lT, sT = T[1], T[2]                                       # 5: sigma3(-T)
        S_f = sT                                                  # target scale of sigma3's terms
        T2 = ev.rescale(ev.mul(T, T))                             # level lT-1
        sU = S_f * prm.q[lT - 1] / T2[2]                          # U * T2 / q_{lT-1} = S_f
        U = ev.pmul_to(T, "sig_c3", np.full(half, -SIG_C3), sU)   # level lT-1: +0.001593 T
        T3 = ev.rescale(ev.mul(T2, U))                            # level lT-2, scale S_f
        T1 = ev.drop(ev.pmul_to(T, "sig_c1", np.full(half, -SIG_C1), S_f), lT - 2)
        S = ev.padd(ev.add(T3, T1), "sig_c0", np.full(half, 0.5))
        Zd = ev.drop(Z, S[1])
        G = ev.rescale(ev.mul(S, Zd))                             # 6
        for k in range(lr):                                       # 7
            G = ev.add(G, ev.rot(G, f << k))
        Gs.append(G)
    G = Gs[0]
    for Gb in Gs[1:]:                                             # 8
        G = ev.add(G, Gb)
    upd = ev.pmul_to(G, "gamma", np.full(half, sh.gamma / sh.n), W[2])   # 9
    Wn = ev.add(ev.drop(W, upd[1]), upd)
    assert Wn[1] == W[1] - HELR_LEVELS
    return Wn, ev.consts, ev.counts


# --------------------------------------------------------------------------- ResNet-20 layer

@dataclass
class ConvShape:
    N: int
    C: int                   # channels in and out
    H: int                   # image side

    @property
    def offsets(self) -> list[int]:
        return [dy * self.H + dx for dy in (-1, 0, 1) for dx in (-1, 0, 1) if (dy, dx) != (0, 0)]

    def rotations(self) -> tuple[list[int], list[int]]:
        """(hoisted baby steps, giant steps) as left-rotation amounts."""
        return self.offsets, [d * self.H * self.H for d in range(1, self.C)]


CONV_LEVELS = 4


def conv_pack(sh: ConvShape, x: np.ndarray) -> np.ndarray:
    """x [C][H][H] -> slot vector (channel-major, tiled to N/2)."""
    flat = x.reshape(-1)
    return np.tile(flat, sh.N // 2 // flat.size)


def conv_unpack(sh: ConvShape, z: np.ndarray) -> np.ndarray:
    return np.real(z[: sh.C * sh.H * sh.H]).reshape(sh.C, sh.H, sh.H)


def conv_plain(sh: ConvShape, x, w, bias) -> np.ndarray:
    """3x3 conv (stride 1, zero padding) + bias + the degree-4 ReLU polynomial."""
    C, H = sh.C, sh.H
    xp = np.zeros((C, H + 2, H + 2))
    xp[:, 1:-1, 1:-1] = x
    y = np.zeros((C, H, H))
    for co in range(C):
        for ci in range(C):
            for dy in (-1, 0, 1):
                for dx in (-1, 0, 1):
                    y[co] += w[co, ci, dy + 1, dx + 1] * xp[ci, 1 + dy:1 + dy + H, 1 + dx:1 + dx + H]
    y += bias[:, None, None]
    a0, a1, a2, a4 = RELU_A
    return a0 + a1 * y + a2 * y ** 2 + a4 * y ** 4


def conv_diag(sh: ConvShape, w: np.ndarray, d: int, dy: int, dx: int) -> np.ndarray:
    """V_{d,o}: slot (c H^2 + y H + x) of the unrotated diagonal holds w[c][(c+d) % C][dy][dx]
    where (y+dy, x+dx) is inside the image; the vector is then rotated right by d H^2 (so the
    giant-step rotation by d H^2 lines it up) and tiled to N/2."""
    C, H = sh.C, sh.H
    yy, xx = np.meshgrid(np.arange(H), np.arange(H), indexing="ij")
    valid = ((yy + dy >= 0) & (yy + dy < H) & (xx + dx >= 0) & (xx + dx < H)).astype(float)
    v = np.concatenate([w[c, (c + d) % C, dy + 1, dx + 1] * valid.reshape(-1) for c in range(C)])
    v = np.roll(v, d * H * H)                                     # rot_{-d H^2}
    return np.tile(v, sh.N // 2 // v.size)


def _conv(sh: ConvShape, ev: Ev, X, w: np.ndarray, bias: np.ndarray, pre: str = ""):
    """Steps 1-3: 3x3 convolution (hoisted baby steps, baby-step giant-step diagonal method),
    Rescale, bias.  One level; the output keeps X's scale."""
    prm = ev.prm
    C, H, half = sh.C, sh.H, sh.N // 2
    lx = X[1]
    offs = [(dy, dx) for dy in (-1, 0, 1) for dx in (-1, 0, 1)]
    rots = dict(zip([o for o in offs if o != (0, 0)], ev.rot_hoisted(X, sh.offsets)))   # 1
    rots[(0, 0)] = X
    S_w = float(prm.q[lx])                                        # weights' scale: Rescale restores sx
    Y = None
    for d in range(C):                                            # 2
        acc = None
        for dy, dx in offs:
            t = ev.pmul(rots[(dy, dx)], f"{pre}w_{d}_{dy}_{dx}", conv_diag(sh, w, d, dy, dx), S_w)
            acc = t if acc is None else ev.add(acc, t)
        if d:
            acc = ev.rot(acc, d * H * H)
        Y = acc if Y is None else ev.add(Y, acc)
    Y = ev.rescale(Y)
    bias_slots = np.tile(np.repeat(bias, H * H), half // (C * H * H))
    return ev.padd(Y, f"{pre}bias", bias_slots)                   # 3


def _relu(sh: ConvShape, ev: Ev, Y, pre: str = ""):
    """Step 4: the degree-4 ReLU polynomial; three levels, the output keeps Y's scale."""
    prm, half = ev.prm, sh.N // 2
    a0, a1, a2, a4 = RELU_A
    lY, S_a = Y[1], Y[2]
    Y2 = ev.rescale(ev.mul(Y, Y))                                 # level lY-1
    sU = S_a * prm.q[lY - 2] / Y2[2]                              # Y2 * U / q_{lY-2} = S_a
    U = ev.pmul_to(Y2, f"{pre}relu_a4", np.full(half, a4), sU)    # level lY-2
    Y4 = ev.rescale(ev.mul(ev.drop(Y2, lY - 2), U))               # level lY-3
    Y2c = ev.drop(ev.pmul_to(Y2, f"{pre}relu_a2", np.full(half, a2), S_a), lY - 3)
    Y1c = ev.drop(ev.pmul_to(Y, f"{pre}relu_a1", np.full(half, a1), S_a), lY - 3)
    return ev.padd(ev.add(ev.add(Y4, Y2c), Y1c), f"{pre}relu_a0", np.full(half, a0))


def conv_layer(sh: ConvShape, prm: ckks.Params, X, w: np.ndarray, bias: np.ndarray, keys: dict,
               consts: dict | None = None, dry: bool = False):
    """X = (ct, level, scale).  Returns (out, consts, counts); out at level - 4, X's scale.
    dry: constants only (DryEv)."""
    ev = _ev(prm, keys, consts, dry)
    out = _relu(sh, ev, _conv(sh, ev, X, w, bias))
    assert out[1] == X[1] - CONV_LEVELS
    return out, ev.consts, ev.counts


# --------------------------------------------------------------------------- ResNet-20 mix
# Reading R4 (APP): the layer types of [32]'s ResNet-20 beyond one convolution -- a stride-1
# basic block (conv, ReLU, conv, + shortcut, ReLU: the block of all three stages, here at the
# first stage's shape) and the network head (global average pooling, 64 -> 10 fully connected
# layer, here C -> K with K <= C).  The stride-2 blocks that change the packing between stages
# are not built.

BLOCK_LEVELS = 2 * CONV_LEVELS
HEAD_LEVELS = 2


def basic_block(sh: ConvShape, prm: ckks.Params, X, w1, b1, w2, b2, keys: dict, consts: dict | None = None):
    """out = ReLU(conv2(ReLU(conv1(X))) + X): 8 levels, X's scale.  Returns (out, consts, counts)."""
    ev = Ev(prm, keys, consts)
    h = _relu(sh, ev, _conv(sh, ev, X, w1, b1, "c1_"), "r1_")
    y = _conv(sh, ev, h, w2, b2, "c2_")
    out = _relu(sh, ev, ev.add(y, ev.drop(X, y[1])), "r2_")
    assert out[1] == X[1] - BLOCK_LEVELS
    return out, ev.consts, ev.counts


def head_rotations(sh: ConvShape) -> tuple[list[int], list[int]]:
    """(pooling's rotate-and-sum amounts 2^k < H^2, the FC layer's hoisted amounts d H^2)."""
    return [1 << k for k in range(int(math.log2(sh.H * sh.H)))], [d * sh.H * sh.H for d in range(1, sh.C)]


def head(sh: ConvShape, prm: ckks.Params, X, wfc: np.ndarray, bfc: np.ndarray, keys: dict,
         consts: dict | None = None):
    """Global average pooling per channel then a K x C fully connected layer (K = len(bfc) <= C):
    class k at slot k H^2.  2 levels, X's scale.  Returns (out, consts, counts)."""
    ev = Ev(prm, keys, consts)
    C, H, half = sh.C, sh.H, sh.N // 2
    K = len(bfc)
    pool_r, fc_r = head_rotations(sh)
    P = X
    for r in pool_r:                                              # slot c H^2: sum over channel c
        P = ev.add(P, ev.rot(P, r))
    m = np.zeros(C * H * H)
    m[:: H * H] = 1.0 / (H * H)
    P = ev.pmul_to(P, "pool_mask", np.tile(m, half // m.size), X[2])   # pooled[c] at slot c H^2
    rots = [P] + ev.rot_hoisted(P, fc_r)
    S_w = float(prm.q[P[1]])
    acc = None
    for d in range(C):                                            # diagonal method on the H^2 grid
        diag = np.zeros(C * H * H)
        for k in range(K):
            diag[k * H * H] = wfc[k, (k + d) % C]
        t = ev.pmul(rots[d], f"fc_{d}", np.tile(diag, half // diag.size), S_w)
        acc = t if acc is None else ev.add(acc, t)
    out = ev.rescale(acc)
    bb = np.zeros(C * H * H)
    bb[: K * H * H: H * H] = bfc
    out = ev.padd(out, "fc_bias", np.tile(bb, half // bb.size))
    assert out[1] == X[1] - HEAD_LEVELS
    return out, ev.consts, ev.counts


def relu_poly(y):
    a0, a1, a2, a4 = RELU_A
    return a0 + a1 * y + a2 * y ** 2 + a4 * y ** 4


def conv_linear_plain(sh: ConvShape, x, w, bias) -> np.ndarray:
    """3x3 conv (stride 1, zero padding) + bias, no activation."""
    C, H = sh.C, sh.H
    xp = np.zeros((C, H + 2, H + 2))
    xp[:, 1:-1, 1:-1] = x
    y = np.zeros((C, H, H))
    for co in range(C):
        for ci in range(C):
            for dy in (-1, 0, 1):
                for dx in (-1, 0, 1):
                    y[co] += w[co, ci, dy + 1, dx + 1] * xp[ci, 1 + dy:1 + dy + H, 1 + dx:1 + dx + H]
    return y + bias[:, None, None]


def block_plain(sh: ConvShape, x, w1, b1, w2, b2) -> np.ndarray:
    return relu_poly(conv_linear_plain(sh, relu_poly(conv_linear_plain(sh, x, w1, b1)), w2, b2) + x)


def head_plain(x, wfc, bfc) -> np.ndarray:
    return wfc @ x.mean(axis=(1, 2)) + bfc


# --------------------------------------------------------------------------- keys, encryption

def app_keys(prm: ckks.Params, s: np.ndarray, rotations: list[int], seed: int) -> dict:
    """'relin' and one rotation key per Galois element of the left-rotation amounts."""
    keys = {"relin": ckks.relin_key(prm, s, seed)}
    for t, g in enumerate(sorted({_g(prm.N, r) for r in rotations})):
        keys[g] = ckks.rot_key(prm, s, g, seed + 1 + t)
    return keys


def encrypt_slots(prm: ckks.Params, z, delta: float, s: np.ndarray, level: int, seed: int):
    m = _encode(prm.N, z, delta)
    return ckks.encrypt(prm, m, s, level, seed), level, delta


def decrypt_slots(prm: ckks.Params, v, s: np.ndarray) -> np.ndarray:
    ct, l, sc = v
    m = ckks.crt_centered(prm, ckks.decrypt_residues(prm, ct, s, l), list(range(l + 1)))
    return ckks.decode(prm.N, m, sc)
