"""CKKS application traces on the GPU (BASELINE configs[4]; reading APP in
DESIGN.md): one HELR training iteration [17, 18] and one ResNet-20 convolution layer [32],
issued through the C-ABI in the order the oracle (oracle/apps.py) defines -- the same
operations on the same operands, so the results are bit-exact.

HELR iteration (L530, "batch sizes of 1,024 images", 196 features -> f = 256):
  T = Rescale(HMULT(Z, W)); T += HROT(T, 2^k) (k < log f); T = Rescale(PMULT(T, mask));
  T += HROT(T, -2^k); S = sigma3(-T) (two HMULTs, two PMULTs); G = Rescale(HMULT(S, Z));
  G += HROT(G, f 2^k) (k < log rows); G = sum over the batch; W' = W + Rescale(PMULT(G, gamma/n)).
  The batch of ciphertexts is one batched call per step (the library's batch dimension).
ResNet-20 layer (L572, [32]'s 16-channel 32 x 32 stage): 8 hoisted baby-step rotations of the
  input (one ModUp), per channel diagonal d one fused plaintext inner product over the 9 kernel
  offsets (neo_pmult_acc) and one giant-step HROT by d H^2, Rescale, bias PADD, and the degree-4
  ReLU polynomial (two HMULTs, three PMULTs).  The layer mix (reading R4): a stride-1 basic
  block (conv, ReLU, conv, + shortcut, ReLU) and the head (average pooling by rotate-and-sum,
  a fully connected layer by the diagonal method on the H^2-strided grid).

Plaintext constants are inputs (name -> device tensor [l+1][N], NTT form), like evaluation
keys: tests produce them with the oracle's encoder, bench.py with random residues (the cost is
data-independent).  Keys: {'relin': EvalKey, g: EvalKey} plus, for the conv layer's baby steps,
hoisted keys {('h', g): EvalKey(hoisted_galois=g)}."""
from __future__ import annotations

import math

import torch

from . import neo


def galois(N: int, r: int) -> int:
    """Galois element of a left rotation by r slots (Z11), r taken mod N/2."""
    return pow(5, r % (N // 2), 2 * N)


def helr_rotations(N: int, f: int) -> list[int]:
    rows = N // 2 // f
    lf, lr = int(math.log2(f)), int(math.log2(rows))
    return [1 << k for k in range(lf)] + [-(1 << k) for k in range(lf)] + [f << k for k in range(lr)]


def conv_rotations(C: int, H: int) -> tuple[list[int], list[int]]:
    """(hoisted baby steps dy H + dx, giant steps d H^2)."""
    baby = [dy * H + dx for dy in (-1, 0, 1) for dx in (-1, 0, 1) if (dy, dx) != (0, 0)]
    return baby, [d * H * H for d in range(1, C)]


def helr_const_names() -> list[str]:
    return ["mask", "sig_c3", "sig_c1", "sig_c0", "gamma"]


def conv_const_names(C: int) -> list[str]:
    ws = [f"w_{d}_{dy}_{dx}" for d in range(C) for dy in (-1, 0, 1) for dx in (-1, 0, 1)]
    return ws + ["bias", "relu_a4", "relu_a2", "relu_a1", "relu_a0"]


class Evaluator:
    """Thin sequencing of C-ABI calls on one stream; every op allocates its output."""

    def __init__(self, ctx: neo.Context, keys: dict, consts: dict, max_batch: int = 1, stream=None):
        self.ctx, self.keys, self.consts, self.stream = ctx, keys, consts, stream
        self.N = ctx.N
        top = ctx.num_q - 1
        ops = (neo.NEO_OP_HMULT, neo.NEO_OP_HROT, neo.NEO_OP_RESCALE, neo.NEO_OP_HROT_HOISTED,
               neo.NEO_OP_HMULT_RESCALE)
        wsn = max(ctx.workspace_size(op, top, max_batch) for op in ops)
        self.ws = torch.empty(wsn // 8, dtype=torch.uint64, device="cuda")
        self._bc = {}

    def _ct(self, level, B=1, lead=()):
        return torch.empty((*lead, B, 2, level + 1, self.N), dtype=torch.uint64, device="cuda")

    def _pt_batched(self, name, B):
        """A shared plaintext repeated for B ciphertexts (neo_padd takes one per ciphertext)."""
        if (name, B) not in self._bc:
            self._bc[(name, B)] = self.consts[name].unsqueeze(0).expand(B, -1, -1).contiguous()
        return self._bc[(name, B)]

    def rot(self, ct, r, lv):
        g = galois(self.N, r)
        out = self._ct(lv, ct.shape[0])
        neo.neo_hrot(self.ctx, self.keys[g], g, ct, lv, out, ct.shape[0], self.ws, self.stream)
        return out

    def rot_hoisted(self, ct, rs, lv):
        keys = [self.keys[("h", galois(self.N, r))] for r in rs]
        out = self._ct(lv, ct.shape[0], (len(rs),))
        neo.neo_hrot_hoisted(self.ctx, keys, ct, lv, out, ct.shape[0], self.ws, self.stream)
        return out

    def add(self, a, b, lv):
        out = self._ct(lv, a.shape[0])
        neo.neo_hadd(self.ctx, a, b, lv, out, a.shape[0], self.stream)
        return out

    def hmul(self, a, b, lv):
        out = self._ct(lv, a.shape[0])
        neo.neo_hmult(self.ctx, self.keys["relin"], a, b, lv, out, a.shape[0], self.ws, self.stream)
        return out

    def hmul_rescale(self, a, b, lv):
        """Rescale(HMULT(a, b)) as one fused call (bit-identical)."""
        out = self._ct(lv - 1, a.shape[0])
        neo.neo_hmult_rescale(self.ctx, self.keys["relin"], a, b, lv, out, a.shape[0], self.ws, self.stream)
        return out

    def rescale(self, a, lv):
        out = self._ct(lv - 1, a.shape[0])
        neo.neo_rescale(self.ctx, a, lv, out, a.shape[0], self.ws, self.stream)
        return out

    def drop(self, a, li, lo):
        if li == lo:
            return a
        out = self._ct(lo, a.shape[0])
        neo.neo_drop_levels(self.ctx, a, li, out, lo, a.shape[0], self.stream)
        return out

    def pmul(self, a, name, lv):
        """PMULT by one shared plaintext (neo_pmult_acc with one term)."""
        return self.pmul_acc([a], [name], lv)

    def pmul_acc(self, cts, names, lv):
        out = self._ct(lv, cts[0].shape[0])
        neo.neo_pmult_acc(self.ctx, cts, [self.consts[n] for n in names], lv, out, cts[0].shape[0],
                          pt_shared=True, stream=self.stream)
        return out

    def padd(self, a, name, lv):
        out = self._ct(lv, a.shape[0])
        neo.neo_padd(self.ctx, a, self._pt_batched(name, a.shape[0]), lv, out, a.shape[0], self.stream)
        return out


def helr_iteration(ev: Evaluator, f: int, Z: torch.Tensor, W: torch.Tensor, level: int):
    """Z [B][2][level+1][N] (B ciphertexts of rows x f samples), W [1][2][level+1][N] ->
    (W' [1][2][level-5][N], level - 6)."""
    N, B = ev.N, Z.shape[0]
    rows = N // 2 // f
    lf, lr = int(math.log2(f)), int(math.log2(rows))
    L = level
    Wb = W.expand(B, -1, -1, -1).contiguous() if B > 1 else W
    T = ev.hmul_rescale(Z, Wb, L)                          # 1
    lv = L - 1
    for k in range(lf):                                           # 2
        T = ev.add(T, ev.rot(T, 1 << k, lv), lv)
    T = ev.rescale(ev.pmul(T, "mask", lv), lv)                    # 3
    lv -= 1
    for k in range(lf):                                           # 4
        T = ev.add(T, ev.rot(T, -(1 << k), lv), lv)
    lT = lv                                                       # 5
    T2 = ev.hmul_rescale(T, T, lT)
    U = ev.rescale(ev.pmul(T, "sig_c3", lT), lT)
    T3 = ev.hmul_rescale(T2, U, lT - 1)
    T1 = ev.drop(ev.rescale(ev.pmul(T, "sig_c1", lT), lT), lT - 1, lT - 2)
    S = ev.padd(ev.add(T3, T1, lT - 2), "sig_c0", lT - 2)
    G = ev.hmul_rescale(S, ev.drop(Z, L, lT - 2), lT - 2)   # 6
    lg = lT - 3
    for k in range(lr):                                           # 7
        G = ev.add(G, ev.rot(G, f << k, lg), lg)
    while G.shape[0] > 1:                                         # 8 (a tree: modular sums are exact)
        h = G.shape[0] // 2
        S2 = ev.add(G[:h], G[h:2 * h], lg)
        G = S2 if G.shape[0] == 2 * h else torch.cat([S2, G[2 * h:]])
    upd = ev.rescale(ev.pmul(G, "gamma", lg), lg)                 # 9
    Wn = ev.add(ev.drop(W, L, lg - 1), upd, lg - 1)
    return Wn, lg - 1


def conv(ev: Evaluator, C: int, H: int, X: torch.Tensor, level: int, pre: str = ""):
    """Convolution + Rescale + bias (the oracle's _conv): X at `level` -> level - 1."""
    baby, _ = conv_rotations(C, H)
    lv = level
    R = ev.rot_hoisted(X, baby, lv)                               # 1: [8][1][2][l+1][N]
    offs = [(dy, dx) for dy in (-1, 0, 1) for dx in (-1, 0, 1)]
    src, k = [], 0
    for o in offs:
        if o == (0, 0):
            src.append(X)
        else:
            src.append(R[k])
            k += 1
    Y = None
    for d in range(C):                                            # 2
        acc = ev.pmul_acc(src, [f"{pre}w_{d}_{dy}_{dx}" for dy, dx in offs], lv)
        if d:
            acc = ev.rot(acc, d * H * H, lv)
        Y = acc if Y is None else ev.add(Y, acc, lv)
    Y = ev.rescale(Y, lv)
    return ev.padd(Y, f"{pre}bias", lv - 1)                       # 3


def relu(ev: Evaluator, Y: torch.Tensor, lY: int, pre: str = ""):
    """The degree-4 ReLU polynomial (the oracle's _relu): lY -> lY - 3."""
    Y2 = ev.hmul_rescale(Y, Y, lY)                                # 4
    U = ev.rescale(ev.pmul(Y2, f"{pre}relu_a4", lY - 1), lY - 1)
    Y4 = ev.hmul_rescale(ev.drop(Y2, lY - 1, lY - 2), U, lY - 2)
    Y2c = ev.drop(ev.rescale(ev.pmul(Y2, f"{pre}relu_a2", lY - 1), lY - 1), lY - 2, lY - 3)
    Y1c = ev.drop(ev.rescale(ev.pmul(Y, f"{pre}relu_a1", lY), lY), lY - 1, lY - 3)
    return ev.padd(ev.add(ev.add(Y4, Y2c, lY - 3), Y1c, lY - 3), f"{pre}relu_a0", lY - 3)


def conv_layer(ev: Evaluator, C: int, H: int, X: torch.Tensor, level: int):
    """X [1][2][level+1][N] -> (out [1][2][level-3][N], level - 4)."""
    return relu(ev, conv(ev, C, H, X, level), level - 1), level - 4


# ---- ResNet-20 layer mix (reading R4): a stride-1 basic block and the network head

def block_const_names(C: int) -> list[str]:
    names = []
    for pre in ("c1_", "c2_"):
        names += [f"{pre}w_{d}_{dy}_{dx}" for d in range(C) for dy in (-1, 0, 1) for dx in (-1, 0, 1)]
        names.append(f"{pre}bias")
    for pre in ("r1_", "r2_"):
        names += [f"{pre}relu_a{k}" for k in (4, 2, 1, 0)]
    return names


def head_rotations(C: int, H: int) -> tuple[list[int], list[int]]:
    """(pooling's rotate-and-sum amounts 2^k < H^2, the FC layer's hoisted amounts d H^2)."""
    return [1 << k for k in range(int(math.log2(H * H)))], [d * H * H for d in range(1, C)]


def head_const_names(C: int) -> list[str]:
    return ["pool_mask"] + [f"fc_{d}" for d in range(C)] + ["fc_bias"]


def basic_block(ev: Evaluator, C: int, H: int, X: torch.Tensor, level: int):
    """ReLU(conv2(ReLU(conv1(X))) + X): level -> level - 8."""
    h = relu(ev, conv(ev, C, H, X, level, "c1_"), level - 1, "r1_")
    y = conv(ev, C, H, h, level - 4, "c2_")
    z = ev.add(y, ev.drop(X, level, level - 5), level - 5)
    return relu(ev, z, level - 5, "r2_"), level - 8


def head(ev: Evaluator, C: int, H: int, X: torch.Tensor, level: int):
    """Global average pooling + fully connected layer (class k at slot k H^2): level -> level - 2."""
    pool_r, fc_r = head_rotations(C, H)
    P = X
    for r in pool_r:
        P = ev.add(P, ev.rot(P, r, level), level)
    P = ev.rescale(ev.pmul(P, "pool_mask", level), level)
    lv = level - 1
    R = ev.rot_hoisted(P, fc_r, lv)
    acc = ev.pmul_acc([P] + [R[k] for k in range(C - 1)], [f"fc_{d}" for d in range(C)], lv)
    out = ev.rescale(acc, lv)
    return ev.padd(out, "fc_bias", lv - 1), lv - 1
