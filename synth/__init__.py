"""Seeded synthetic input generators shared by the oracle tests, the GPU tests and bench.py.

This module holds NO arithmetic of the method (no modular products, no NTT, no
basis conversion).  It only turns a seed into deterministic random numbers:

* ``splitmix64(seed, count)``     -- the raw 64-bit stream (SplitMix64, Steele et al.)
* ``uniform_residues(seed, moduli, n)`` -- one uniform row per modulus (values x mod m)
* ``ternary_hwt(seed, n, h)``     -- ternary secret with Hamming weight h
* ``rounded_gaussian(seed, n, sigma, bound)`` -- rounded Gaussian error
* ``complex_slots(seed, n_slots)`` -- slot values with Re, Im uniform in [-1, 1)

Random numbers the method draws (the key/encryption randomness ``a``, ``s``, ``e``)
are produced here and passed to the oracle as inputs, so that any other
implementation fed the same arrays computes the same residues.

Seed recipe: base seed 0x4E454F ("NEO"); ciphertext b of a
batch uses base + b; sub-streams are derived with ``derive(seed, tag)``.
"""
from __future__ import annotations

import numpy as np

BASE_SEED = 0x4E454F
_GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)


def splitmix64(seed: int, count: int) -> np.ndarray:
    """Return ``count`` outputs of SplitMix64 started at state ``seed`` (uint64 array).

    z_k = mix(seed + (k+1) * 0x9E3779B97F4A7C15), mix = the SplitMix64 finaliser.
    """
    with np.errstate(over="ignore"):
        k = np.arange(1, count + 1, dtype=np.uint64)
        z = np.uint64(seed & 0xFFFFFFFFFFFFFFFF) + k * _GOLDEN
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
        z = z ^ (z >> np.uint64(31))
    return z


def derive(seed: int, tag: int) -> int:
    """Derive an independent sub-stream seed from (seed, tag)."""
    return int(splitmix64((seed * 0x100000001B3 + tag) & 0xFFFFFFFFFFFFFFFF, 1)[0])


def uniform_residues(seed: int, moduli, n: int) -> np.ndarray:
    """[len(moduli)][n] uint64 array, row r uniform in [0, moduli[r]) (x mod m; bias < 2^-27)."""
    moduli = [int(m) for m in moduli]
    out = np.empty((len(moduli), n), dtype=np.uint64)
    for r, m in enumerate(moduli):
        out[r] = splitmix64(derive(seed, r), n) % np.uint64(m)
    return out


def uniform_unit(seed: int, count: int) -> np.ndarray:
    """``count`` doubles uniform in [0, 1) from the top 53 bits of the stream."""
    return (splitmix64(seed, count) >> np.uint64(11)).astype(np.float64) * (2.0 ** -53)


def ternary_hwt(seed: int, n: int, h: int) -> np.ndarray:
    """int64 array of length n with exactly h entries in {-1, +1} and the rest 0.

    Positions come from a partial Fisher-Yates shuffle driven by the stream, signs from
    one further bit of the stream.
    """
    stream = splitmix64(seed, 2 * h)
    perm = np.arange(n, dtype=np.int64)
    for k in range(h):
        j = k + int(stream[k] % np.uint64(n - k))
        perm[k], perm[j] = perm[j], perm[k]
    s = np.zeros(n, dtype=np.int64)
    signs = np.where((stream[h:2 * h] & np.uint64(1)) == 1, 1, -1)
    s[perm[:h]] = signs
    return s


def rounded_gaussian(seed: int, n: int, sigma: float = 3.2, bound: int = 19) -> np.ndarray:
    """int64 array: round(sigma * N(0,1)) via Box-Muller, clipped to [-bound, bound]."""
    u = uniform_unit(seed, 2 * n)
    u1 = np.maximum(u[:n], 2.0 ** -53)
    u2 = u[n:]
    g = np.sqrt(-2.0 * np.log(u1)) * np.cos(2.0 * np.pi * u2)
    e = np.rint(sigma * g).astype(np.int64)
    return np.clip(e, -bound, bound)


def complex_slots(seed: int, n_slots: int) -> np.ndarray:
    """complex128 array, real and imaginary parts uniform in [-1, 1)."""
    u = uniform_unit(seed, 2 * n_slots)
    return (2.0 * u[:n_slots] - 1.0) + 1j * (2.0 * u[n_slots:] - 1.0)
