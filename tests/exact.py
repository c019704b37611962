"""Exact rational reference arithmetic for tiny brute-force pins (Python fractions).

Matrix-level formulation (op(X) by transposition, products by np.dot over Fraction
object arrays) -- deliberately not the oracle's index loops.  On integer inputs with
dyadic alpha/beta every FP64 partial sum is exact, so any correct summation order must
reproduce these values bit for bit (SURVEY.md §8(c) "What pins each part").
"""
from fractions import Fraction

import numpy as np


def F(a):
    a = np.asarray(a)
    out = np.empty(a.shape, dtype=object)
    for idx in np.ndindex(a.shape):
        out[idx] = Fraction(float(a[idx]))
    return out


def to_float(a):
    out = np.empty(a.shape, dtype=np.float64)
    for idx in np.ndindex(a.shape):
        out[idx] = float(a[idx])
    return out


def op(X, t):
    return X.T if t.upper() in "TC" else X


def gemm(ta, tb, alpha, A, B, beta, C):
    P = np.dot(op(F(A), ta), op(F(B), tb))
    R = Fraction(alpha) * P
    if beta != 0:
        R = R + Fraction(beta) * F(C)
    return R


def tri(A, lower, unit):
    """Triangular matrix from the uplo part of A (implicit unit diagonal if unit)."""
    n = A.shape[0]
    T = np.empty((n, n), dtype=object)
    for i in range(n):
        for j in range(n):
            if i == j:
                T[i, j] = Fraction(1) if unit else Fraction(float(A[i, j]))
            elif (i > j) == lower:
                T[i, j] = Fraction(float(A[i, j]))
            else:
                T[i, j] = Fraction(0)
    return T


def sym(A, lower):
    n = A.shape[0]
    S = np.empty((n, n), dtype=object)
    for i in range(n):
        for j in range(n):
            src = (i, j) if ((i >= j) == lower or i == j) else (j, i)
            S[i, j] = Fraction(float(A[src]))
    return S


def solve_exact(Tm, Bm):
    """Solve Tm X = Bm exactly by Gauss-Jordan on Fractions (Tm any invertible)."""
    n = Tm.shape[0]
    M = np.concatenate([Tm.copy(), Bm.copy()], axis=1)
    for c in range(n):
        p = next(r for r in range(c, n) if M[r, c] != 0)
        if p != c:
            M[[c, p]] = M[[p, c]]
        piv = M[c, c]
        M[c] = M[c] / piv
        for r in range(n):
            if r != c and M[r, c] != 0:
                M[r] = M[r] - M[r, c] * M[c]
    return M[:, n:]
