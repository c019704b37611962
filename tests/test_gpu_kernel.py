"""GPU parity of the sm_100a FP64 tile kernel (xk_dgemm_tile_device) vs the CPU oracle.

Tolerance (north_star): |C - C_ref|_ij <= 4*k*2^-53*(|alpha||A||B| + |beta||C|)_ij and
relative Frobenius <= 1e-13; exact-integer inputs must match bit for bit (every partial
sum is an exact integer < 2^53, so any summation order gives the same result).
"""
import itertools

import numpy as np
import pytest

import inputs
import oracle
import paper_conf_sc_gautierl21_b200 as xk
from tests.gpu_util import from_dev, stream_ptr, to_dev

pytestmark = pytest.mark.gpu

SHAPES = [(256, 256, 256), (300, 257, 129), (1, 1, 1), (129, 1, 17), (7, 300, 33), (513, 385, 1000)]


def shp(t, r, c):
    return (c, r) if t == "T" else (r, c)


def run_tile(ta, tb, m, n, k, alpha, A, B, beta, C0, lda=None, ldb=None, ldc=None):
    import torch
    lda = lda or A.shape[0]; ldb = ldb or B.shape[0]; ldc = ldc or C0.shape[0]
    dA, dB, dC = to_dev(A), to_dev(B), to_dev(C0)
    rc = xk.dgemm_tile_device(ta, tb, m, n, k, alpha, dA, lda, dB, ldb, beta, dC, ldc, stream_ptr())
    assert rc == 0
    torch.cuda.synchronize()
    return from_dev(dC, ldc, C0.shape[1])


@pytest.mark.parametrize("ta,tb", list(itertools.product("NT", "NT")))
def test_tile_random_within_bound(ta, tb):
    for (m, n, k) in SHAPES:
        A = inputs.uniform(1, *shp(ta, m, k)); B = inputs.uniform(2, *shp(tb, k, n))
        C0 = inputs.uniform(3, m, n)
        for alpha, beta in [(1.5, -0.75), (1.5, 0.0), (-2.0, 1.0)]:
            Cin = C0.copy(order="F")
            if beta == 0.0:
                Cin[:] = np.nan  # beta == 0: C must not be read
            got = run_tile(ta, tb, m, n, k, alpha, A, B, beta, Cin)
            ref = C0.copy(order="F")
            oracle.dgemm(ta, tb, m, n, k, alpha, A, B, beta, ref)
            bound = oracle.gemm_bound(ta, tb, m, n, k, alpha, A, B, beta, C0)
            assert np.all(np.abs(got - ref) <= bound), (ta, tb, m, n, k, alpha, beta)
            assert np.linalg.norm(got - ref) <= 1e-13 * max(np.linalg.norm(ref), 1e-300)


@pytest.mark.parametrize("ta,tb", list(itertools.product("NT", "NT")))
def test_tile_exact_integers_bitwise(ta, tb):
    m, n, k = 300, 257, 531
    A = inputs.integers(11, *shp(ta, m, k)); B = inputs.integers(12, *shp(tb, k, n))
    C0 = inputs.integers(13, m, n)
    for alpha, beta in [(1.0, 1.0), (-2.0, 0.5), (0.5, 0.0)]:
        got = run_tile(ta, tb, m, n, k, alpha, A, B, beta, C0.copy(order="F"))
        ref = C0.copy(order="F")
        oracle.dgemm(ta, tb, m, n, k, alpha, A, B, beta, ref)
        assert np.array_equal(got, ref)


def test_tile_padded_and_odd_leading_dimensions():
    # odd ld -> 8-byte cp.async path; padding rows of C must stay untouched
    m, n, k = 131, 67, 45
    for lda, ldb, ldc in [(m + 1, k + 3, m + 5), (m + 8, k + 8, m + 8)]:
        A = inputs.uniform(1, m, k, ld=lda); B = inputs.uniform(2, k, n, ld=ldb)
        C0 = inputs.uniform(3, m, n, ld=ldc); C0[m:] = 42.0
        got = run_tile("N", "N", m, n, k, 1.5, A, B, -0.75, C0.copy(order="F"), lda, ldb, ldc)
        ref = C0.copy(order="F")
        oracle.dgemm("N", "N", m, n, k, 1.5, A, B, -0.75, ref, lda=lda, ldb=ldb, ldc=ldc)
        bound = oracle.gemm_bound("N", "N", m, n, k, 1.5, A[:m], B[:k], -0.75, C0[:m])
        assert np.all(np.abs(got[:m] - ref[:m]) <= bound)
        assert np.all(got[m:] == 42.0)


def test_tile_alpha_zero_and_k_zero():
    m, n = 70, 50
    C0 = inputs.uniform(3, m, n)
    An = np.full((m, 5), np.nan, order="F"); Bn = np.full((5, n), np.nan, order="F")
    got = run_tile("N", "N", m, n, 5, 0.0, An, Bn, -0.5, C0.copy(order="F"))
    assert np.array_equal(got, -0.5 * C0)
    got = run_tile("N", "N", m, n, 5, 0.0, An, Bn, 0.0, C0.copy(order="F"))
    assert np.all(got == 0)


def test_tile_full_size_2048_sampled():
    """The bench's tile size (T=2048, NN): sampled entries vs the oracle's dot loop."""
    import torch
    T = 2048
    A = inputs.uniform(1, T, T); B = inputs.uniform(2, T, T); C0 = inputs.uniform(3, T, T)
    got = run_tile("N", "N", T, T, T, 1.5, A, B, -0.75, C0.copy(order="F"))
    rng = np.random.default_rng(0)
    ii = rng.integers(0, T, 4096); jj = rng.integers(0, T, 4096)
    ii[:4] = [0, T - 1, 0, T - 1]; jj[:4] = [0, 0, T - 1, T - 1]
    ref = oracle.dgemm_sampled("N", "N", T, 1.5, A, B, -0.75, C0[ii, jj], ii, jj)
    mag = 1.5 * np.einsum("qk,kq->q", np.abs(A[ii, :]), np.abs(B[:, jj])) + 0.75 * np.abs(C0[ii, jj])
    assert np.all(np.abs(got[ii, jj] - ref) <= 4 * T * 2.0 ** -53 * mag)
    # timing context (not the bench number)
    dA, dB, dC = to_dev(A), to_dev(B), to_dev(C0)
    s = stream_ptr()
    for _ in range(3):
        xk.dgemm_tile_device("N", "N", T, T, T, 1.5, dA, T, dB, T, 1.0, dC, T, s)
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    e0.record()
    for _ in range(10):
        xk.dgemm_tile_device("N", "N", T, T, T, 1.5, dA, T, dB, T, 1.0, dC, T, s)
    e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / 10
    print("dgemm_tile T=2048: %.3f ms  %.2f TFLOP/s" % (ms, 2 * T ** 3 / ms / 1e9))
