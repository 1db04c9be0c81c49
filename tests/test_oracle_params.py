"""Oracle pins: RNS parameters (Table 1, Table 4; readings Z2-Z5)."""
import pytest
import sympy
from sympy.ntheory import primitive_root

from oracle import ckks


@pytest.mark.parametrize("log_n,num_q,num_p", [(12, 3, 1), (16, 36, 12)])
def test_prime_rule_exhaustive(log_n, num_q, num_p):
    """Z4: the chosen primes are exactly the first num_q+num_p primes k*2N+1 going down
    from 2^36 -- every skipped candidate is composite (checked with sympy, not ckks.is_prime)."""
    two_n = 2 << log_n
    primes = ckks.gen_primes(log_n, 36, num_q + num_p)
    k = ((1 << 36) - 1) // two_n
    found = []
    while len(found) < len(primes):
        c = k * two_n + 1
        if sympy.isprime(c):
            found.append(c)
        k -= 1
    assert found == primes
    for q in primes:
        assert q % two_n == 1 and q.bit_length() == 36


def test_prime_test_vectors():
    """Z4 test vectors."""
    t = ckks.tiny()
    assert t.q == [68719403009, 68719230977, 68719206401] and t.p == [68719190017]
    b = ckks.set_b()
    assert b.q[0] == 68718428161 and b.q[1] == 68712923137
    assert b.p[0] == 68662460417 and b.moduli[47] == 68644896769
    assert b.alpha == 12 and b.beta(35) == 3 and len(b.moduli) == 48


def test_psi_minimal_primitive():
    """Z5: psi is a primitive 2N-th root (psi^N = -1) and the smallest one; recomputed from
    sympy's primitive root g as min over odd k of g^((q-1)/2N * k)."""
    for prm in (ckks.tiny(), ckks.Params(4, 2, 1, 1)):
        N = prm.N
        for q, psi in zip(prm.moduli, prm.psi):
            assert pow(psi, N, q) == q - 1
            g = primitive_root(q)
            w = pow(g, (q - 1) // (2 * N), q)
            assert psi == min(pow(w, k, q) for k in range(1, 2 * N, 2))
    t = ckks.tiny()
    assert t.psi[0] == 24250113
    b = ckks.set_b()
    assert b.psi[0] == 1987404 and b.psi[36] == 2913696


def test_digits():
    """L98-99, Z8: alpha = ceil((L+1)/dnum), beta = ceil((l+1)/alpha); digits are raw limbs."""
    b = ckks.set_b()
    assert b.digits(35) == [list(range(0, 12)), list(range(12, 24)), list(range(24, 36))]
    assert b.digits(13) == [list(range(0, 12)), [12, 13]]
    assert b.digits(0) == [[0]]
    t = ckks.tiny()
    assert t.alpha == 3 and t.digits(2) == [[0, 1, 2]]
    assert ckks.tiny_dnum3().digits(2) == [[0], [1], [2]]
