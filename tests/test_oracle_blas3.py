"""Pins for oracle SYRK/SYR2K/SYMM/TRMM/TRSM (oracle/oracle.c) -- SURVEY.md §8(c).

Exact rational brute force on tiny integer inputs for every flag combination, closed
forms (rank-1 SYRK, L = I, bidiagonal L = D(I-S) with known inverse, TRSM->TRMM round
trip), OpenBLAS (scipy) cross-checks within the north_star bound, and the BLAS
"not referenced" rules (opposite triangle / unit diagonal poisoned with NaN; untouched
triangle of C bitwise unchanged).
"""
import itertools

import numpy as np
import pytest
import scipy.linalg.blas as sblas

import inputs
import oracle
from tests import exact

EPS = 2.0 ** -53


def fmat(a):
    return np.asfortranarray(a, dtype=np.float64)


def tri_mask(n, lower):
    return np.tril(np.ones((n, n), bool)) if lower else np.triu(np.ones((n, n), bool))


# ----------------------------------------------------------------------------- SYRK
@pytest.mark.parametrize("uplo,trans", list(itertools.product("LU", "NT")))
def test_syrk_exact_bruteforce(uplo, trans):
    lower = uplo == "L"
    for (n, k) in [(4, 4), (1, 3), (3, 1), (4, 2)]:
        A = fmat(inputs.integers(20 + n + k, *((n, k) if trans == "N" else (k, n))))
        C0 = fmat(inputs.integers(30 + n, n, n))
        for alpha, beta in itertools.product([1.0, -2.0, 0.5], [0.0, 1.0, -1.0]):
            C = C0.copy(order="F")
            assert oracle.dsyrk(uplo, trans, n, k, alpha, A, beta, C) == 0
            ref = exact.to_float(exact.gemm(trans, "T" if trans == "N" else "N", alpha, A, A, beta, C0))
            msk = tri_mask(n, lower)
            assert np.array_equal(C[msk], ref[msk])
            assert np.array_equal(C[~msk], C0[~msk])  # other triangle untouched


def test_syrk_rank1_outer_product():
    n = 50
    x = inputs.integers(5, n, 1)
    C = fmat(np.zeros((n, n)))
    oracle.dsyrk("L", "N", n, 1, 1.0, x, 0.0, C)
    outer = np.outer(x[:, 0], x[:, 0])
    msk = tri_mask(n, True)
    assert np.array_equal(C[msk], outer[msk])


@pytest.mark.parametrize("uplo,trans", list(itertools.product("LU", "NT")))
def test_syrk_syr2k_vs_openblas(uplo, trans):
    n, k = 131, 77
    shp = (n, k) if trans == "N" else (k, n)
    A = fmat(inputs.uniform(1, *shp)); B = fmat(inputs.uniform(2, *shp)); C0 = fmat(inputs.uniform(3, n, n))
    lower = int(uplo == "L"); tr = int(trans == "T")
    msk = tri_mask(n, bool(lower))
    C = C0.copy(order="F")
    oracle.dsyrk(uplo, trans, n, k, 1.5, A, -0.75, C)
    ref = sblas.dsyrk(1.5, A, beta=-0.75, c=C0.copy(order="F"), trans=tr, lower=lower)
    opA = A if trans == "N" else A.T
    bound = 4 * k * EPS * (1.5 * np.abs(opA) @ np.abs(opA).T + 0.75 * np.abs(C0))
    assert np.all(np.abs(C - ref)[msk] <= bound[msk])
    assert np.array_equal(C[~msk], C0[~msk])
    C = C0.copy(order="F")
    oracle.dsyr2k(uplo, trans, n, k, 1.5, A, B, -0.75, C)
    ref = sblas.dsyr2k(1.5, A, B, beta=-0.75, c=C0.copy(order="F"), trans=tr, lower=lower)
    opB = B if trans == "N" else B.T
    bound = 4 * 2 * k * EPS * (1.5 * (np.abs(opA) @ np.abs(opB).T + np.abs(opB) @ np.abs(opA).T) + 0.75 * np.abs(C0))
    assert np.all(np.abs(C - ref)[msk] <= bound[msk])
    assert np.array_equal(C[~msk], C0[~msk])


@pytest.mark.parametrize("uplo,trans", list(itertools.product("LU", "NT")))
def test_syr2k_exact_bruteforce(uplo, trans):
    lower = uplo == "L"
    for (n, k) in [(4, 4), (3, 2), (1, 1)]:
        shp = (n, k) if trans == "N" else (k, n)
        A = fmat(inputs.integers(40 + n, *shp)); B = fmat(inputs.integers(50 + k, *shp))
        C0 = fmat(inputs.integers(60, n, n))
        for alpha, beta in [(1.0, 0.0), (-2.0, 1.0), (0.5, -1.0)]:
            C = C0.copy(order="F")
            assert oracle.dsyr2k(uplo, trans, n, k, alpha, A, B, beta, C) == 0
            t2 = "T" if trans == "N" else "N"
            P = exact.gemm(trans, t2, 1.0, A, B, 0.0, C0) + exact.gemm(trans, t2, 1.0, B, A, 0.0, C0)
            ref = exact.to_float(exact.F(np.zeros((n, n))) + P * exact.Fraction(alpha) + exact.F(C0) * exact.Fraction(beta))
            msk = tri_mask(n, lower)
            assert np.array_equal(C[msk], ref[msk])
            assert np.array_equal(C[~msk], C0[~msk])


# ----------------------------------------------------------------------------- SYMM
@pytest.mark.parametrize("side,uplo", list(itertools.product("LR", "LU")))
def test_symm_exact_and_not_referenced(side, uplo):
    lower = uplo == "L"
    for (m, n) in [(4, 4), (3, 2), (1, 4)]:
        ka = m if side == "L" else n
        A = fmat(inputs.integers(70 + m, ka, ka))
        Ap = A.copy(order="F")
        Ap[~tri_mask(ka, lower)] = np.nan  # other triangle must not be read
        B = fmat(inputs.integers(80 + n, m, n)); C0 = fmat(inputs.integers(90, m, n))
        C = C0.copy(order="F")
        assert oracle.dsymm(side, uplo, m, n, -1.5 if False else 2.0, Ap, B, -1.0, C) == 0
        S = exact.sym(A, lower)
        P = np.dot(S, exact.F(B)) if side == "L" else np.dot(exact.F(B), S)
        ref = exact.to_float(P * exact.Fraction(2) - exact.F(C0))
        assert np.array_equal(C, ref)


@pytest.mark.parametrize("side,uplo", list(itertools.product("LR", "LU")))
def test_symm_vs_openblas(side, uplo):
    m, n = 97, 61
    ka = m if side == "L" else n
    A = fmat(inputs.uniform(1, ka, ka)); B = fmat(inputs.uniform(2, m, n)); C0 = fmat(inputs.uniform(3, m, n))
    C = C0.copy(order="F")
    oracle.dsymm(side, uplo, m, n, 1.5, A, B, -0.75, C)
    ref = sblas.dsymm(1.5, A, B, beta=-0.75, c=C0.copy(order="F"), side=int(side == "R"), lower=int(uplo == "L"))
    S = np.where(tri_mask(ka, uplo == "L"), A, A.T)
    mag = (np.abs(S) @ np.abs(B)) if side == "L" else (np.abs(B) @ np.abs(S))
    assert np.all(np.abs(C - ref) <= 4 * ka * EPS * (1.5 * mag + 0.75 * np.abs(C0)))


# ----------------------------------------------------------------------- TRMM / TRSM
FLAGS = list(itertools.product("LR", "LU", "NT", "NU"))


def int_tri(seed, n, lower, unit):
    """Integer triangular factor with diagonal in {1,-1,2,-2} (exact inverse arithmetic)."""
    A = fmat(inputs.integers(seed, n, n, lo=-3, span=7))
    d = np.array([1.0, -2.0, 2.0, -1.0] * n)[:n]
    A[np.diag_indices(n)] = d
    P = A.copy(order="F")
    P[~tri_mask(n, lower)] = np.nan  # opposite triangle never read
    if unit:
        P[np.diag_indices(n)] = np.nan  # diag='U': diagonal never read
    return A, P


@pytest.mark.parametrize("side,uplo,ta,diag", FLAGS)
def test_trmm_exact_bruteforce(side, uplo, ta, diag):
    lower, unit = uplo == "L", diag == "U"
    for (m, n) in [(4, 4), (3, 2), (1, 3)]:
        ka = m if side == "L" else n
        A, P = int_tri(100 + m + n, ka, lower, unit)
        B0 = fmat(inputs.integers(110 + m, m, n))
        for alpha in (1.0, -0.5, 2.0):
            B = B0.copy(order="F")
            assert oracle.dtrmm(side, uplo, ta, diag, m, n, alpha, P, B) == 0
            T = exact.op(exact.tri(A, lower, unit), ta)
            prod = np.dot(T, exact.F(B0)) if side == "L" else np.dot(exact.F(B0), T)
            assert np.array_equal(B, exact.to_float(prod * exact.Fraction(alpha)))


@pytest.mark.parametrize("side,uplo,ta,diag", FLAGS)
def test_trsm_exact_bruteforce(side, uplo, ta, diag):
    lower, unit = uplo == "L", diag == "U"
    for (m, n) in [(4, 4), (3, 2), (1, 3)]:
        ka = m if side == "L" else n
        A, P = int_tri(200 + m + n, ka, lower, unit)
        B0 = fmat(inputs.integers(210 + n, m, n))
        for alpha in (1.0, -2.0):
            B = B0.copy(order="F")
            assert oracle.dtrsm(side, uplo, ta, diag, m, n, alpha, P, B) == 0
            T = exact.op(exact.tri(A, lower, unit), ta)
            rhs = exact.F(B0) * exact.Fraction(alpha)
            if side == "L":
                X = exact.solve_exact(T, rhs)
            else:  # X T = rhs  <=>  T^T X^T = rhs^T
                X = exact.solve_exact(T.T.copy(), rhs.T.copy()).T
            assert np.array_equal(B, exact.to_float(X)), (m, n, alpha)


def test_trsm_bidiagonal_closed_form():
    """L = D(I - S), S = ones on the first sub-diagonal, D = diag(2^p):
    L^-1_ij = 2^-p_j for i >= j, so X = alpha * (column prefix sums of D^-1 B)."""
    m, n = 40, 9
    p = (np.arange(m) % 5) - 2
    D = np.diag(2.0 ** p)
    S = np.diag(np.ones(m - 1), -1)
    L = fmat(D @ (np.eye(m) - S))
    B0 = fmat(inputs.integers(7, m, n))
    B = B0.copy(order="F")
    oracle.dtrsm("L", "L", "N", "N", m, n, 2.0, L, B)
    expect = 2.0 * np.cumsum((2.0 ** -p)[:, None] * B0, axis=0)
    assert np.array_equal(B, expect)
    # L = I -> X = alpha B
    B = B0.copy(order="F")
    oracle.dtrsm("L", "L", "N", "N", m, n, -1.5, fmat(np.eye(m)), B)
    assert np.array_equal(B, -1.5 * B0)


@pytest.mark.parametrize("side,uplo,ta,diag", FLAGS)
def test_trsm_trmm_round_trip_and_openblas(side, uplo, ta, diag):
    m, n = 120, 70
    ka = m if side == "L" else n
    L = inputs.tri_dd(4, ka, lower=(uplo == "L"), fill=np.nan)  # Q9 factor, opposite triangle NaN
    B0 = fmat(inputs.uniform(2, m, n))
    alpha = 1.5
    X = B0.copy(order="F")
    assert oracle.dtrsm(side, uplo, ta, diag, m, n, alpha, L, X) == 0
    Lc = np.nan_to_num(L, nan=0.0)
    ref = sblas.dtrsm(alpha, fmat(Lc), B0.copy(order="F"), side=int(side == "R"), lower=int(uplo == "L"),
                      trans_a=int(ta == "T"), diag=int(diag == "U"))
    assert np.linalg.norm(X - ref) <= 1e-13 * np.linalg.norm(ref)
    # residual bound Q13: |op(L) X - alpha B| <= 4*ka*eps*(|op(L)||X| + |alpha||B|)
    T = np.where(tri_mask(ka, uplo == "L"), Lc, 0.0)
    if diag == "U":
        T[np.diag_indices(ka)] = 1.0
    T = T.T if ta == "T" else T
    R = (T @ X - alpha * B0) if side == "L" else (X @ T - alpha * B0)
    mag = (np.abs(T) @ np.abs(X)) if side == "L" else (np.abs(X) @ np.abs(T))
    assert np.all(np.abs(R) <= 4 * ka * EPS * (mag + alpha * np.abs(B0)) * 1.0000001)
    # round trip: TRMM(X) with alpha=1/alpha returns B0 within the bound
    Y = X.copy(order="F")
    assert oracle.dtrmm(side, uplo, ta, diag, m, n, 1.0 / alpha, L, Y) == 0
    assert np.linalg.norm(Y - B0) <= 1e-13 * np.linalg.norm(B0)
    # trmm vs openblas
    Y2 = B0.copy(order="F")
    oracle.dtrmm(side, uplo, ta, diag, m, n, alpha, L, Y2)
    ref2 = sblas.dtrmm(alpha, fmat(Lc), B0.copy(order="F"), side=int(side == "R"), lower=int(uplo == "L"),
                       trans_a=int(ta == "T"), diag=int(diag == "U"))
    mag2 = (np.abs(T) @ np.abs(B0)) if side == "L" else (np.abs(B0) @ np.abs(T))
    assert np.all(np.abs(Y2 - ref2) <= 4 * ka * EPS * alpha * mag2)


def test_blas3_argument_errors_and_quick_returns():
    A = fmat(np.zeros((4, 4)))
    assert oracle.dsyrk("X", "N", 2, 2, 1.0, A, 0.0, A) == -1
    assert oracle.dsyrk("L", "X", 2, 2, 1.0, A, 0.0, A) == -2
    assert oracle.dsyrk("L", "N", -1, 2, 1.0, A, 0.0, A) == -3
    assert oracle.dsyrk("L", "N", 2, -1, 1.0, A, 0.0, A) == -4
    assert oracle.dsyrk("L", "N", 5, 2, 1.0, A, 0.0, A, lda=4, ldc=5) == -7
    assert oracle.dsyrk("L", "N", 4, 2, 1.0, A, 0.0, A, lda=4, ldc=3) == -10
    assert oracle.dsyr2k("L", "N", 5, 2, 1.0, A, A, 0.0, A, lda=5, ldb=4, ldc=5) == -9
    assert oracle.dsyr2k("L", "N", 4, 2, 1.0, A, A, 0.0, A, lda=4, ldb=4, ldc=3) == -12
    assert oracle.dsymm("X", "L", 2, 2, 1.0, A, A, 0.0, A) == -1
    assert oracle.dsymm("L", "X", 2, 2, 1.0, A, A, 0.0, A) == -2
    assert oracle.dsymm("L", "L", 5, 2, 1.0, A, A, 0.0, A, lda=4, ldb=5, ldc=5) == -7
    assert oracle.dsymm("L", "L", 4, 2, 1.0, A, A, 0.0, A, lda=4, ldb=3, ldc=4) == -9
    assert oracle.dsymm("L", "L", 4, 2, 1.0, A, A, 0.0, A, lda=4, ldb=4, ldc=3) == -12
    for f in (oracle.dtrmm, oracle.dtrsm):
        assert f("X", "L", "N", "N", 2, 2, 1.0, A, A) == -1
        assert f("L", "X", "N", "N", 2, 2, 1.0, A, A) == -2
        assert f("L", "L", "X", "N", 2, 2, 1.0, A, A) == -3
        assert f("L", "L", "N", "X", 2, 2, 1.0, A, A) == -4
        assert f("L", "L", "N", "N", -1, 2, 1.0, A, A) == -5
        assert f("L", "L", "N", "N", 2, -1, 1.0, A, A) == -6
        assert f("L", "L", "N", "N", 5, 2, 1.0, A, A, lda=4, ldb=5) == -9
        assert f("R", "L", "N", "N", 4, 5, 1.0, A, A, lda=4, ldb=4) == -9
        assert f("L", "L", "N", "N", 4, 2, 1.0, A, A, lda=4, ldb=3) == -11
        # alpha == 0: B <- 0 without reading A
        Bz = fmat(np.ones((3, 3)))
        assert f("L", "L", "N", "N", 3, 3, 0.0, fmat(np.full((3, 3), np.nan)), Bz) == 0
        assert np.all(Bz == 0)
