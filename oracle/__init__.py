"""CPU oracle for the xk hot path -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py (cpu_baseline leg and --impl reference)
may import this package.  The product package (paper_conf_sc_gautierl21_b200/) never
imports it; the two share no code (task framing ③).

Thin ctypes marshalling over oracle/liboracle.so (oracle/oracle.c, plain C99 BLAS-3
definitions, PAPER.md P:376-377 / P:1187-1188).  All matrices are numpy
float64 arrays in Fortran (column-major) order; a matrix with leading dimension ld is an
(ld x ncols) array whose first rows are the matrix.  Functions return the BLAS info code
(0 or -i) and update the output array in place.

Parity status: every routine is pinned (tests/test_oracle_*.py); see DESIGN.md §Oracle.
"""
import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None


def _lib():
    global _LIB
    if _LIB is None:
        path = os.path.join(_HERE, "liboracle.so")
        src = os.path.join(_HERE, "oracle.c")
        if not os.path.exists(path) or os.path.getmtime(src) > os.path.getmtime(path):
            from tools.build_native import build_oracle
            build_oracle()
        lib = ctypes.CDLL(path)
        c, i64, d, p = ctypes.c_char, ctypes.c_int64, ctypes.c_double, ctypes.c_void_p
        lib.oracle_dgemm.argtypes = [c, c, i64, i64, i64, d, p, i64, p, i64, d, p, i64]
        lib.oracle_dsyrk.argtypes = [c, c, i64, i64, d, p, i64, d, p, i64]
        lib.oracle_dsyr2k.argtypes = [c, c, i64, i64, d, p, i64, p, i64, d, p, i64]
        lib.oracle_dsymm.argtypes = [c, c, i64, i64, d, p, i64, p, i64, d, p, i64]
        lib.oracle_dtrmm.argtypes = [c, c, c, c, i64, i64, d, p, i64, p, i64]
        lib.oracle_dtrsm.argtypes = [c, c, c, c, i64, i64, d, p, i64, p, i64]
        lib.oracle_dgemm_sampled.argtypes = [c, c, i64, d, p, i64, p, i64, d, p, p, p, i64, p]
        for f in ("oracle_dgemm", "oracle_dsyrk", "oracle_dsyr2k", "oracle_dsymm",
                  "oracle_dtrmm", "oracle_dtrsm", "oracle_dgemm_sampled", "oracle_num_threads"):
            getattr(lib, f).restype = ctypes.c_int
        _LIB = lib
    return _LIB


def _ch(x):
    return ctypes.c_char(x.encode() if isinstance(x, str) else x)


def _ptr(a):
    if a is None:
        return None
    assert a.dtype == np.float64 and (a.flags.f_contiguous or a.ndim == 1), "need float64 Fortran arrays"
    return a.ctypes.data


def _ld(a, ld):
    if ld is not None:
        return ld
    return max(1, a.shape[0]) if a is not None and a.ndim == 2 else 1


def dgemm(transA, transB, m, n, k, alpha, A, B, beta, C, lda=None, ldb=None, ldc=None):
    return _lib().oracle_dgemm(_ch(transA), _ch(transB), m, n, k, alpha, _ptr(A), _ld(A, lda),
                               _ptr(B), _ld(B, ldb), beta, _ptr(C), _ld(C, ldc))


def dsyrk(uplo, trans, n, k, alpha, A, beta, C, lda=None, ldc=None):
    return _lib().oracle_dsyrk(_ch(uplo), _ch(trans), n, k, alpha, _ptr(A), _ld(A, lda),
                               beta, _ptr(C), _ld(C, ldc))


def dsyr2k(uplo, trans, n, k, alpha, A, B, beta, C, lda=None, ldb=None, ldc=None):
    return _lib().oracle_dsyr2k(_ch(uplo), _ch(trans), n, k, alpha, _ptr(A), _ld(A, lda),
                                _ptr(B), _ld(B, ldb), beta, _ptr(C), _ld(C, ldc))


def dsymm(side, uplo, m, n, alpha, A, B, beta, C, lda=None, ldb=None, ldc=None):
    return _lib().oracle_dsymm(_ch(side), _ch(uplo), m, n, alpha, _ptr(A), _ld(A, lda),
                               _ptr(B), _ld(B, ldb), beta, _ptr(C), _ld(C, ldc))


def dtrmm(side, uplo, transA, diag, m, n, alpha, A, B, lda=None, ldb=None):
    return _lib().oracle_dtrmm(_ch(side), _ch(uplo), _ch(transA), _ch(diag), m, n, alpha,
                               _ptr(A), _ld(A, lda), _ptr(B), _ld(B, ldb))


def dtrsm(side, uplo, transA, diag, m, n, alpha, A, B, lda=None, ldb=None):
    return _lib().oracle_dtrsm(_ch(side), _ch(uplo), _ch(transA), _ch(diag), m, n, alpha,
                               _ptr(A), _ld(A, lda), _ptr(B), _ld(B, ldb))


def dgemm_sampled(transA, transB, k, alpha, A, B, beta, c0, ii, jj, lda=None, ldb=None):
    """Oracle C entries at sampled coordinates (ii[q], jj[q]); c0[q] = original C there."""
    ii = np.ascontiguousarray(ii, dtype=np.int64)
    jj = np.ascontiguousarray(jj, dtype=np.int64)
    c0 = np.ascontiguousarray(c0, dtype=np.float64)
    out = np.empty(len(ii), dtype=np.float64)
    _lib().oracle_dgemm_sampled(_ch(transA), _ch(transB), k, alpha, _ptr(A), _ld(A, lda),
                                _ptr(B), _ld(B, ldb), beta, c0.ctypes.data, ii.ctypes.data,
                                jj.ctypes.data, len(ii), out.ctypes.data)
    return out


def num_threads():
    return _lib().oracle_num_threads()


def gemm_bound(transA, transB, m, n, k, alpha, A, B, beta, C0):
    """north_star elementwise bound 4*k*2^-53*(|alpha||op(A)||op(B)| + |beta||C0|)."""
    opA = A[:k, :m].T if transA.upper() != "N" else A[:m, :k]
    opB = B[:n, :k].T if transB.upper() != "N" else B[:k, :n]
    mag = abs(alpha) * (np.abs(opA) @ np.abs(opB))
    if beta != 0:
        mag = mag + abs(beta) * np.abs(C0[:m, :n])
    return 4.0 * max(k, 1) * 2.0 ** -53 * mag
