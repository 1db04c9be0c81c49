"""Oracle pins: NTT / INTT (radix-16 NTT of L438-450 computes a(psi^(2i+1)), Z6) and the
negacyclic ring product of R_q (Table 1)."""
import numpy as np
import pytest

import synth
from oracle import _core, ckks


def _brute_negacyclic(a, b, q):
    """Pure-Python schoolbook product in Z_q[X]/(X^N+1)."""
    n = len(a)
    out = [0] * n
    for i in range(n):
        for j in range(n):
            if i + j < n:
                out[i + j] += int(a[i]) * int(b[j])
            else:
                out[i + j - n] -= int(a[i]) * int(b[j])
    return [v % q for v in out]


@pytest.fixture(scope="module")
def small():
    return ckks.Params(4, 2, 1, 1)            # N = 16


@pytest.fixture(scope="module")
def tiny():
    return ckks.tiny()


def test_ntt_closed_form_monomials(small):
    """NTT(X^k)[i] = psi^((2i+1)k); NTT(1) = all ones."""
    N = small.N
    for lid in range(len(small.moduli)):
        q, psi = small.moduli[lid], small.psi[lid]
        for k in range(N):
            x = np.zeros((1, N), dtype=np.uint64)
            x[0, k] = 1
            for mode in ("def", "fast"):
                got = ckks.ntt(small, x, [lid], mode)[0]
                want = [pow(psi, (2 * i + 1) * k, q) for i in range(N)]
                assert [int(v) for v in got] == want


@pytest.mark.parametrize("log_n", [4, 6, 10, 12])
def test_fast_equals_definition_and_inverse(log_n):
    prm = ckks.Params(log_n, 2, 1, 1)
    ids = [0, 1, 2]
    x = synth.uniform_residues(7 + log_n, prm.moduli, prm.N)
    d = ckks.ntt(prm, x, ids, "def")
    f = ckks.ntt(prm, x, ids, "fast")
    assert np.array_equal(d, f)
    assert np.array_equal(ckks.intt(prm, d, ids, "def"), x)
    assert np.array_equal(ckks.intt(prm, f, ids, "fast"), x)


def test_schoolbook_matches_bruteforce(small):
    q = small.moduli[0]
    a = synth.uniform_residues(1, [q], small.N)[0]
    b = synth.uniform_residues(2, [q], small.N)[0]
    out = np.empty_like(a)
    _core.lib().or_negacyclic_mul(_core.ptr(a), _core.ptr(b), _core.ptr(out), small.N, q)
    assert [int(v) for v in out] == _brute_negacyclic(a, b, q)


def test_convolution_theorem(tiny):
    """INTT(NTT(a) . NTT(b)) equals the schoolbook negacyclic product (N = 4096)."""
    ids = [0, 3]
    a = synth.uniform_residues(11, [tiny.moduli[i] for i in ids], tiny.N)
    b = synth.uniform_residues(12, [tiny.moduli[i] for i in ids], tiny.N)
    prod = ckks.intt(tiny, ckks.mul(tiny, ckks.ntt(tiny, a, ids), ckks.ntt(tiny, b, ids), ids), ids)
    for k, i in enumerate(ids):
        ref = np.empty(tiny.N, dtype=np.uint64)
        _core.lib().or_negacyclic_mul(_core.ptr(a[k]), _core.ptr(b[k]), _core.ptr(ref), tiny.N,
                                      tiny.moduli[i])
        assert np.array_equal(prod[k], ref)


@pytest.mark.slow
def test_set_b_fast_ntt_sampled_against_definition():
    """At N = 2^16 the fast transform agrees with the definition at sampled outputs."""
    prm = ckks.set_b()
    ids = [0, 35, 47]
    x = synth.uniform_residues(99, [prm.moduli[i] for i in ids], prm.N)
    f = ckks.ntt(prm, x, ids, "fast")
    L = _core.lib()
    rng = np.random.default_rng(5)
    for k, i in enumerate(ids):
        row = np.ascontiguousarray(x[k])
        for idx in list(rng.integers(0, prm.N, 6)) + [0, prm.N - 1]:
            assert int(f[k, idx]) == L.or_ntt_point(_core.ptr(row), prm.N, prm.moduli[i],
                                                    prm.psi[i], int(idx))
    assert np.array_equal(ckks.intt(prm, f, ids), x)


def test_encode_fft_matches_the_definition():
    """encode_fft (one FFT) and encode (the definition, direct sums) agree to within one after
    rounding (floating-point order only; almost all coefficients equal), and decode back."""
    import synth
    for N, delta in ((1 << 8, 2.0 ** 30), (1 << 12, 2.0 ** 36)):
        z = synth.complex_slots(17, N // 2)
        a, b = ckks.encode(N, z, delta), ckks.encode_fft(N, z, delta)
        assert np.max(np.abs(a - b)) <= 1
        assert np.mean(a != b) < 0.01
        assert np.max(np.abs(ckks.decode(N, [float(v) for v in b], delta) - z)) < 1e-6
