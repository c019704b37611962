"""Randomised GPU parity: random routines, flags, ragged shapes, odd tile sizes, 1-3 logical
GPUs, alpha/beta special values -- every call through the C ABI against the CPU oracle under
the north_star bounds (Q13).  Seeded, so failures reproduce."""
import random

import numpy as np
import pytest

import inputs
import oracle
import paper_conf_sc_gautierl21_b200 as xk
from tests.gpu_util import device_map

pytestmark = pytest.mark.gpu
EPS = 2.0 ** -53


def tri_mask(n, lower):
    return np.tril(np.ones((n, n), bool)) if lower else np.triu(np.ones((n, n), bool))


def check(got, ref, mag, k, mask=None):
    bound = 4 * max(k, 1) * EPS * mag * 1.0000001 + 1e-300
    d = np.abs(got - ref)
    if mask is not None:
        d, bound = d[mask], bound[mask]
    assert np.all(d <= bound)


@pytest.mark.parametrize("seed", range(6))
def test_random_calls(seed):
    r = random.Random(seed)
    G = r.choice([1, 2, 3])
    T = r.choice([64, 96, 128])
    xk.init(ngpus=G, phys=device_map(G), tile=T, probe=False, topo=r.choice(["ranked", "unranked", "home"]),
            optimistic=r.random() < 0.7)
    try:
        for _ in range(8):
            routine = r.choice(["gemm", "syrk", "syr2k", "symm", "trmm", "trsm"])
            m, n, k = r.randint(1, 260), r.randint(1, 260), r.randint(1, 260)
            alpha = r.choice([1.5, -1.0, 0.0, 2.0])
            beta = r.choice([0.0, 1.0, -0.75])
            s = r.randint(0, 10 ** 6)
            if routine == "gemm":
                ta, tb = r.choice("NT"), r.choice("NT")
                A = inputs.uniform(s, *((k, m) if ta == "T" else (m, k)))
                B = inputs.uniform(s + 1, *((n, k) if tb == "T" else (k, n)))
                C0 = inputs.uniform(s + 2, m, n)
                C = C0.copy(order="F")
                assert xk.dgemm(ta, tb, m, n, k, alpha, A, A.shape[0], B, B.shape[0], beta, C, m) == 0
                ref = C0.copy(order="F")
                oracle.dgemm(ta, tb, m, n, k, alpha, A, B, beta, ref)
                bnd = oracle.gemm_bound(ta, tb, m, n, k, alpha, A, B, beta, C0) / (4 * max(k, 1) * EPS)
                check(C, ref, bnd, k)
            elif routine in ("syrk", "syr2k"):
                uplo, tr = r.choice("LU"), r.choice("NT")
                shp = (n, k) if tr == "N" else (k, n)
                A = inputs.uniform(s, *shp)
                B = inputs.uniform(s + 1, *shp)
                C0 = inputs.uniform(s + 2, n, n)
                C = C0.copy(order="F")
                opA, opB = (A, B) if tr == "N" else (A.T, B.T)
                ref = C0.copy(order="F")
                if routine == "syrk":
                    assert xk.dsyrk(uplo, tr, n, k, alpha, A, shp[0], beta, C, n) == 0
                    oracle.dsyrk(uplo, tr, n, k, alpha, A, beta, ref)
                    mag = abs(alpha) * (np.abs(opA) @ np.abs(opA).T) + abs(beta) * np.abs(C0)
                    kk = k
                else:
                    assert xk.dsyr2k(uplo, tr, n, k, alpha, A, shp[0], B, shp[0], beta, C, n) == 0
                    oracle.dsyr2k(uplo, tr, n, k, alpha, A, B, beta, ref)
                    mag = abs(alpha) * (np.abs(opA) @ np.abs(opB).T + np.abs(opB) @ np.abs(opA).T) + abs(beta) * np.abs(C0)
                    kk = 2 * k
                msk = tri_mask(n, uplo == "L")
                check(C, ref, mag, kk, msk)
                assert np.array_equal(C[~msk], C0[~msk])
            elif routine == "symm":
                side, uplo = r.choice("LR"), r.choice("LU")
                ka = m if side == "L" else n
                A = inputs.uniform(s, ka, ka)
                B = inputs.uniform(s + 1, m, n)
                C0 = inputs.uniform(s + 2, m, n)
                C = C0.copy(order="F")
                assert xk.dsymm(side, uplo, m, n, alpha, A, ka, B, m, beta, C, m) == 0
                ref = C0.copy(order="F")
                oracle.dsymm(side, uplo, m, n, alpha, A, B, beta, ref)
                S = np.where(tri_mask(ka, uplo == "L"), A, A.T)
                mag = abs(alpha) * ((np.abs(S) @ np.abs(B)) if side == "L" else (np.abs(B) @ np.abs(S))) + abs(beta) * np.abs(C0)
                check(C, ref, mag, ka)
            else:
                side, uplo, ta, dg = r.choice("LR"), r.choice("LU"), r.choice("NT"), r.choice("NU")
                ka = m if side == "L" else n
                L = inputs.tri_dd(s, ka, lower=(uplo == "L"), fill=np.nan)
                B0 = inputs.uniform(s + 1, m, n)
                X = B0.copy(order="F")
                ref = B0.copy(order="F")
                f, of = (xk.dtrmm, oracle.dtrmm) if routine == "trmm" else (xk.dtrsm, oracle.dtrsm)
                assert f(side, uplo, ta, dg, m, n, alpha, L, ka, X, m) == 0
                of(side, uplo, ta, dg, m, n, alpha, L, ref)
                if alpha == 0.0:
                    assert np.all(X == 0)
                    continue
                assert np.linalg.norm(X - ref) <= 1e-13 * max(np.linalg.norm(ref), 1e-300)
                # elementwise (Q13): TRMM vs the oracle, |alpha| 4 ka 2^-53 |op(T)||B0|;
                # TRSM: the componentwise residual of the GPU solution
                Tm = np.where(tri_mask(ka, uplo == "L"), np.nan_to_num(L, nan=0.0), 0.0)
                if dg == "U":
                    Tm[np.diag_indices(ka)] = 1.0
                opT = Tm.T if ta == "T" else Tm
                if routine == "trmm":
                    mag = (np.abs(opT) @ np.abs(B0)) if side == "L" else (np.abs(B0) @ np.abs(opT))
                    assert np.all(np.abs(X - ref) <= 4 * ka * 2.0 ** -53 * abs(alpha) * mag)
                else:
                    R = (opT @ X - alpha * B0) if side == "L" else (X @ opT - alpha * B0)
                    magr = (np.abs(opT) @ np.abs(X)) if side == "L" else (np.abs(X) @ np.abs(opT))
                    assert np.all(np.abs(R) <= 4 * ka * 2.0 ** -53 * (magr + abs(alpha) * np.abs(B0)) * 1.0000001)
    finally:
        xk.finalize()
