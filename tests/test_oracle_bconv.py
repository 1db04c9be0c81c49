"""Oracle pins: BConv (Algorithm 1; non-centred reading Z7), checked against
exact big-integer CRT and a pure-Python transcription."""
import math

import numpy as np
import pytest

import synth
from oracle import ckks


def _alg1_python(prm, x, src, dst):
    qs = [prm.moduli[i] for i in src]
    Q = math.prod(qs)
    out = [[0] * prm.N for _ in dst]
    for a, i in enumerate(src):
        qh = Q // qs[a]
        qinv = pow(qh % qs[a], -1, qs[a])
        for b, t in enumerate(dst):
            m = prm.moduli[t]
            for l in range(prm.N):
                out[b][l] = (out[b][l] + (int(x[a, l]) * qinv % qs[a]) * qh) % m
    return out


@pytest.mark.parametrize("src,dst", [([0, 1, 2], [3, 4]), ([3, 4], [0, 1, 2]), ([1], [0, 4])])
def test_bconv_bruteforce_small(src, dst):
    prm = ckks.Params(4, 3, 2, 1)          # N = 16, 5 moduli
    x = synth.uniform_residues(3, [prm.moduli[i] for i in src], prm.N)
    got = ckks.bconv(prm, x, src, dst)
    assert [[int(v) for v in row] for row in got] == _alg1_python(prm, x, src, dst)


@pytest.mark.parametrize("src,dst", [([0, 1, 2], [3]), ([3], [0, 1, 2]), ([0, 2], [1, 3])])
def test_bconv_exact_crt_overflow(src, dst):
    """out[t] = (x + u*Q_in) mod t with x = CRT(c) in [0,Q_in), u = floor(sum_i y_i/q_i) in
    [0, alpha) (SURVEY §8(c) pin); alpha = 1 reduces to plain reduction (u = 0)."""
    prm = ckks.tiny()
    qs = [prm.moduli[i] for i in src]
    Q = math.prod(qs)
    x = synth.uniform_residues(17, qs, prm.N)
    got = ckks.bconv(prm, x, src, dst)
    X = ckks.crt_lift(prm, x, src)
    for l in range(0, prm.N, 7):
        y = [(int(x[a, l]) * pow((Q // qs[a]) % qs[a], -1, qs[a])) % qs[a] for a in range(len(src))]
        num = sum(yi * (Q // qi) for yi, qi in zip(y, qs))        # = X + u Q exactly
        u, rem = divmod(num, Q)
        assert rem == X[l] and 0 <= u < len(src)
        if len(src) == 1:
            assert u == 0
        for b, t in enumerate(dst):
            assert int(got[b, l]) == (X[l] + u * Q) % prm.moduli[t]
