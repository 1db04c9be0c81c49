"""ctypes loader for oracle_core.c -- CPU ORACLE, TEST INFRASTRUCTURE ONLY.

Built by ``build()`` (gcc -O2 -fopenmp).  Only tests/, __graft_entry__.smoke() and
bench.py's cpu_baseline / --impl reference legs may use it.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle_core.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None

_U64P = ctypes.POINTER(ctypes.c_uint64)


def build(force: bool = False) -> str:
    """Compile oracle_core.c into liboracle.so (if missing or stale)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-shared", "-fPIC", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        u64, i32, i64 = ctypes.c_uint64, ctypes.c_int, ctypes.c_long
        L.or_ntt_point.restype = u64
        L.or_ntt_point.argtypes = [_U64P, i32, u64, u64, i32]
        L.or_ntt_def.argtypes = [_U64P, _U64P, i32, u64, u64]
        L.or_intt_def.argtypes = [_U64P, _U64P, i32, u64, u64]
        L.or_ntt_fast.argtypes = [_U64P, i32, u64, u64]
        L.or_intt_fast.argtypes = [_U64P, i32, u64, u64]
        L.or_ntt_fast_batch.argtypes = [_U64P, i32, i32, _U64P, _U64P, i32]
        L.or_negacyclic_mul.argtypes = [_U64P, _U64P, _U64P, i32, u64]
        L.or_bconv.argtypes = [_U64P, i32, _U64P, i32, i32, _U64P, _U64P, _U64P, _U64P]
        for name in ("or_vec_mulmod", "or_vec_addmod", "or_vec_submod"):
            getattr(L, name).argtypes = [_U64P, _U64P, _U64P, i64, u64]
        L.or_vec_scalar_mulmod.argtypes = [_U64P, u64, _U64P, i64, u64]
        L.or_vec_mod.argtypes = [_U64P, _U64P, i64, u64]
        L.or_crt_exact.argtypes = [_U64P, _U64P, _U64P, i32, _U64P, _U64P, i32, _U64P, i32, _U64P, i32, i32]
        L.or_num_threads.restype = i32
        _lib = L
    return _lib


def ptr(a: np.ndarray):
    assert a.dtype == np.uint64 and a.flags["C_CONTIGUOUS"]
    return a.ctypes.data_as(_U64P)


def u64arr(values) -> np.ndarray:
    return np.ascontiguousarray(np.array([int(v) for v in values], dtype=np.uint64))
