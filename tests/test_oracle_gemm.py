"""Pins for oracle DGEMM (oracle/oracle.c) -- SURVEY.md §8(c) "What pins each part".

Each pin is something other than the oracle itself: exact rational arithmetic on
integer inputs (any correct order must match bitwise), closed forms (identity, 2^p
diagonal scaling), a hand-worked golden fixture, the OpenBLAS DGEMM behind scipy within
the north_star bound, and the BLAS "not referenced" rules (NaN poisoning).
"""
import itertools
import os
import subprocess
import sys

import numpy as np
import pytest
import scipy.linalg.blas as sblas

import inputs
import oracle
from tests import exact

TRANS = ["N", "T"]
HERE = os.path.dirname(os.path.abspath(__file__))


def fmat(a):
    return np.asfortranarray(a, dtype=np.float64)


def shape_of(t, rows, cols):
    return (cols, rows) if t == "T" else (rows, cols)


@pytest.mark.parametrize("ta,tb", list(itertools.product(TRANS, TRANS)))
def test_exact_rational_bruteforce(ta, tb):
    """4x4 and ragged tiny shapes, k in {1,2,3,4}, every alpha/beta in a dyadic set."""
    rng_seed = 10
    for (m, n, k) in [(4, 4, 4), (1, 1, 1), (3, 2, 1), (2, 3, 2), (4, 1, 3), (1, 4, 4)]:
        A = fmat(inputs.integers(rng_seed, *shape_of(ta, m, k)))
        B = fmat(inputs.integers(rng_seed + 1, *shape_of(tb, k, n)))
        C0 = fmat(inputs.integers(rng_seed + 2, m, n))
        rng_seed += 3
        for alpha, beta in itertools.product([1.0, -1.0, 2.0, 0.5], [0.0, 1.0, -2.0, 0.5]):
            C = C0.copy(order="F")
            assert oracle.dgemm(ta, tb, m, n, k, alpha, A, B, beta, C) == 0
            ref = exact.to_float(exact.gemm(ta, tb, alpha, A, B, beta, C0))
            assert np.array_equal(C, ref), (m, n, k, alpha, beta)


def test_golden_hand_worked():
    """tests/golden/dgemm_2x2.txt: hand-worked C = alpha*A*B + beta*C (BLAS definition [1])."""
    vals = {}
    with open(os.path.join(HERE, "golden", "dgemm_2x2.txt")) as f:
        for line in f:
            line = line.split("#")[0].strip()
            if line:
                key, rest = line.split("=")
                vals[key.strip()] = [float(x) for x in rest.split()]
    A = fmat(np.array(vals["A"]).reshape(2, 2))
    B = fmat(np.array(vals["B"]).reshape(2, 2))
    C = fmat(np.array(vals["C"]).reshape(2, 2))
    exp = np.array(vals["RESULT"]).reshape(2, 2)
    assert oracle.dgemm("N", "N", 2, 2, 2, vals["alpha"][0], A, B, vals["beta"][0], C) == 0
    assert np.array_equal(C, exp)
    # transposed operands given as the stored transposes must give the same answer
    C2 = fmat(np.array(vals["C"]).reshape(2, 2))
    At, Bt = fmat(A.T), fmat(B.T)
    assert oracle.dgemm("T", "T", 2, 2, 2, vals["alpha"][0], At, Bt, vals["beta"][0], C2) == 0
    assert np.array_equal(C2, exp)


def test_identity_and_diagonal_scaling():
    n = 37
    B = fmat(inputs.uniform(2, n, n))
    C0 = fmat(inputs.uniform(3, n, n))
    I = fmat(np.eye(n))
    C = C0.copy(order="F")
    oracle.dgemm("N", "N", n, n, n, 1.5, I, B, -0.75, C)
    assert np.array_equal(C, 1.5 * B + (-0.75) * C0)
    # A = diag(2^p): (A B)_ij = 2^p_i B_ij exactly
    p = np.arange(n) % 7 - 3
    D = fmat(np.diag(2.0 ** p))
    C = fmat(np.zeros((n, n)))
    oracle.dgemm("N", "N", n, n, n, 1.0, D, B, 0.0, C)
    assert np.array_equal(C, (2.0 ** p)[:, None] * B)
    # B = diag(2^p) on the right scales columns
    C = fmat(np.zeros((n, n)))
    oracle.dgemm("N", "T", n, n, n, 1.0, B, D, 0.0, C)
    assert np.array_equal(C, B * (2.0 ** p)[None, :])


@pytest.mark.parametrize("ta,tb", list(itertools.product(TRANS, TRANS)))
def test_vs_openblas_within_north_star_bound(ta, tb):
    for (m, n, k) in [(256, 256, 256), (67, 45, 129), (1, 300, 5), (130, 1, 77)]:
        A = fmat(inputs.uniform(1, *shape_of(ta, m, k)))
        B = fmat(inputs.uniform(2, *shape_of(tb, k, n)))
        C0 = fmat(inputs.uniform(3, m, n))
        alpha, beta = 1.5, -0.75
        C = C0.copy(order="F")
        assert oracle.dgemm(ta, tb, m, n, k, alpha, A, B, beta, C) == 0
        ref = sblas.dgemm(alpha, A, B, beta=beta, c=C0.copy(order="F"),
                          trans_a=int(ta == "T"), trans_b=int(tb == "T"))
        bound = oracle.gemm_bound(ta, tb, m, n, k, alpha, A, B, beta, C0)
        assert np.all(np.abs(C - ref) <= bound)
        assert np.linalg.norm(C - ref) <= 1e-13 * np.linalg.norm(ref)


def test_not_referenced_rules():
    m, n, k = 9, 7, 5
    A = fmat(inputs.uniform(1, m, k)); B = fmat(inputs.uniform(2, k, n))
    # beta == 0: C is not read (NaN must not propagate)
    C = fmat(np.full((m, n), np.nan))
    oracle.dgemm("N", "N", m, n, k, 2.0, A, B, 0.0, C)
    assert np.all(np.isfinite(C))
    Cr = fmat(np.zeros((m, n)))
    oracle.dgemm("N", "N", m, n, k, 2.0, A, B, 0.0, Cr)
    assert np.array_equal(C, Cr)
    # alpha == 0: A and B are not read
    An = fmat(np.full((m, k), np.nan)); Bn = fmat(np.full((k, n), np.nan))
    C0 = fmat(inputs.uniform(3, m, n)); C = C0.copy(order="F")
    oracle.dgemm("N", "N", m, n, k, 0.0, An, Bn, -0.5, C)
    assert np.array_equal(C, -0.5 * C0)
    C = C0.copy(order="F")
    oracle.dgemm("N", "N", m, n, k, 0.0, An, Bn, 0.0, C)
    assert np.all(C == 0)
    # quick return alpha==0, beta==1 and k==0, beta==1: C untouched (even NaN A/B)
    C = C0.copy(order="F")
    oracle.dgemm("N", "N", m, n, k, 0.0, An, Bn, 1.0, C)
    assert np.array_equal(C, C0)
    # padding rows (lda/ldc > m) are never written
    ldc = m + 3
    Cp = fmat(np.full((ldc, n), 7.25)); Cp[:m] = C0
    oracle.dgemm("N", "N", m, n, k, 1.0, A, B, 1.0, Cp, ldc=ldc)
    assert np.all(Cp[m:] == 7.25)


def test_argument_errors():
    A = fmat(np.zeros((4, 4)))
    assert oracle.dgemm("X", "N", 2, 2, 2, 1.0, A, A, 0.0, A) == -1
    assert oracle.dgemm("N", "Q", 2, 2, 2, 1.0, A, A, 0.0, A) == -2
    assert oracle.dgemm("N", "N", -1, 2, 2, 1.0, A, A, 0.0, A) == -3
    assert oracle.dgemm("N", "N", 2, -1, 2, 1.0, A, A, 0.0, A) == -4
    assert oracle.dgemm("N", "N", 2, 2, -1, 1.0, A, A, 0.0, A) == -5
    assert oracle.dgemm("N", "N", 5, 2, 2, 1.0, A, A, 0.0, A, lda=4, ldc=5) == -8
    assert oracle.dgemm("T", "N", 2, 2, 5, 1.0, A, A, 0.0, A, lda=4, ldb=5) == -8
    assert oracle.dgemm("N", "N", 2, 2, 5, 1.0, A, A, 0.0, A, lda=4, ldb=4) == -10
    assert oracle.dgemm("N", "N", 5, 2, 2, 1.0, A, A, 0.0, A, lda=5, ldb=4, ldc=4) == -13
    assert oracle.dgemm("n", "t", 2, 2, 2, 1.0, A, A, 0.0, A) == 0  # case-insensitive


def test_deterministic_across_thread_counts():
    code = ("import sys; sys.path.insert(0, %r); import numpy as np, inputs, oracle;"
            "n=96; A=inputs.uniform(1,n,n); B=inputs.uniform(2,n,n); C=inputs.uniform(3,n,n);"
            "oracle.dgemm('N','T',n,n,n,1.5,A,B,-0.75,C); import hashlib; print(hashlib.sha256(C.tobytes()).hexdigest())"
            % os.path.dirname(HERE))
    outs = []
    for t in ("1", "3", "8"):
        env = dict(os.environ, OMP_NUM_THREADS=t)
        outs.append(subprocess.run([sys.executable, "-c", code], env=env, capture_output=True,
                                   text=True, check=True).stdout)
    assert outs[0] == outs[1] == outs[2]


def test_sampled_matches_full():
    m, n, k = 50, 40, 33
    A = fmat(inputs.uniform(1, k, m)); B = fmat(inputs.uniform(2, k, n)); C0 = fmat(inputs.uniform(3, m, n))
    C = C0.copy(order="F")
    oracle.dgemm("T", "N", m, n, k, 1.5, A, B, -0.75, C)
    ii = np.array([0, 49, 17, 3]); jj = np.array([0, 39, 5, 22])
    s = oracle.dgemm_sampled("T", "N", k, 1.5, A, B, -0.75, C0[ii, jj], ii, jj)
    assert np.array_equal(s, C[ii, jj])
