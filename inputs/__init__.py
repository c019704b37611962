"""Seeded synthetic inputs shared by the oracle side and the product side.

The only module both sides import (task framing ③): it fills host arrays from a
counter-based splitmix64 generator (SURVEY.md §8(d) "Generator") and holds none of the
method's arithmetic.  Arrays are numpy, column-major (Fortran order), float64.
"""
import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None

SEED_A, SEED_B, SEED_C, SEED_L, SEED_D, SEED_C2 = 1, 2, 3, 4, 5, 6
ALPHA, BETA = 1.5, -0.75  # reading Q10: exact in binary


def _lib():
    global _LIB
    if _LIB is None:
        path = os.path.join(_HERE, "libxkgen.so")
        if not os.path.exists(path):
            from tools.build_native import build_inputs
            build_inputs()
        lib = ctypes.CDLL(path)
        i64, u64, dp = ctypes.c_int64, ctypes.c_uint64, ctypes.c_void_p
        lib.xkgen_mix.restype = u64
        lib.xkgen_mix.argtypes = [u64]
        lib.xkgen_uniform.argtypes = [u64, i64, i64, dp, i64]
        lib.xkgen_int.argtypes = [u64, i64, i64, dp, i64, ctypes.c_int, ctypes.c_int]
        lib.xkgen_tri_dd.argtypes = [u64, i64, dp, i64, ctypes.c_int, ctypes.c_double]
        lib.xkgen_set_threads.argtypes = [ctypes.c_int]
        _LIB = lib
    return _LIB


def _alloc(m, n, ld, out):
    ld = max(1, m) if ld is None else ld
    if out is None:
        buf = np.zeros((ld, max(n, 0)), dtype=np.float64, order="F")
    else:
        buf = out
        assert buf.dtype == np.float64 and buf.flags.f_contiguous and buf.shape[0] == ld
    return buf, ld


def uniform(seed, m, n, ld=None, out=None):
    """a_ij = 2u-1 in [-1,1); returns the (ld x n) Fortran array (view [:m] is the matrix)."""
    buf, ld = _alloc(m, n, ld, out)
    if m > 0 and n > 0:
        _lib().xkgen_uniform(seed, m, n, buf.ctypes.data, ld)
    return buf


def integers(seed, m, n, ld=None, out=None, lo=-8, span=17):
    """a_ij = floor(span*u) + lo (default [-8,8]): exact-integer inputs."""
    buf, ld = _alloc(m, n, ld, out)
    if m > 0 and n > 0:
        _lib().xkgen_int(seed, m, n, buf.ctypes.data, ld, lo, span)
    return buf


def tri_dd(seed, n, lower=True, ld=None, fill=0.0, out=None):
    """Q9 well-conditioned triangular factor; the opposite triangle gets `fill`."""
    buf, ld = _alloc(n, n, ld, out)
    if n > 0:
        _lib().xkgen_tri_dd(seed, n, buf.ctypes.data, ld, 1 if lower else 0, fill)
    return buf


def mix(z):
    return int(_lib().xkgen_mix(z))


def set_threads(n):
    """Threads of the (counter-based, thread-count independent) fills."""
    _lib().xkgen_set_threads(int(n))
