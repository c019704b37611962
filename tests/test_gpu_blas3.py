"""GPU parity of xk_dsyrk / xk_dsyr2k / xk_dsymm / xk_dtrmm / xk_dtrsm (SURVEY.md §8(f) rows
f1, f2, f4) against the CPU oracle, through the C ABI.

Tolerances (north_star / DESIGN.md Q13): elementwise 4*k*2^-53*(|alpha||A||B|+|beta||C|)
(SYR2K: 2k), relative Frobenius <= 1e-13; TRSM additionally the componentwise residual bound
|op(L) X - alpha B| <= 4*m*2^-53*(|op(L)||X| + |alpha||B|).  "Not referenced" rules are checked
with NaN poisoning; the untouched triangle of C (SYRK/SYR2K) must come back bit for bit.
Multi-GPU logic runs in logical-device mode (G logical GPUs on the one B200).
"""
import itertools

import numpy as np
import pytest

import inputs
import oracle
import paper_conf_sc_gautierl21_b200 as xk
from tests.gpu_util import device_map

pytestmark = pytest.mark.gpu
EPS = 2.0 ** -53


def fmat(a):
    return np.asfortranarray(a, dtype=np.float64)


def tri_mask(n, lower):
    return np.tril(np.ones((n, n), bool)) if lower else np.triu(np.ones((n, n), bool))


@pytest.fixture(params=[1, 4], ids=["G1", "G4"])
def lib(request):
    G = request.param
    xk.init(ngpus=G, phys=device_map(G), tile=128, probe=False)
    yield G
    xk.finalize()


@pytest.mark.parametrize("uplo,trans", list(itertools.product("LU", "NT")))
def test_syrk_syr2k(lib, uplo, trans):
    n, k = 300, 200
    lower = uplo == "L"
    shp = (n, k) if trans == "N" else (k, n)
    A = inputs.uniform(1, *shp); B = inputs.uniform(2, *shp)
    C0 = inputs.uniform(3, n, n)
    msk = tri_mask(n, lower)
    opA = A if trans == "N" else A.T
    opB = B if trans == "N" else B.T
    for alpha, beta in [(1.5, -0.75), (1.5, 0.0), (0.0, 0.5)]:
        C = C0.copy(order="F")
        if beta == 0.0:
            C[msk] = np.nan  # triangle not read when beta == 0
        C[~msk] = np.nan     # other triangle never read, must come back bit for bit
        Cin = C.copy(order="F")
        assert xk.dsyrk(uplo, trans, n, k, alpha, A, shp[0], beta, C, n) == 0
        ref = C0.copy(order="F")
        oracle.dsyrk(uplo, trans, n, k, alpha, A, beta, ref)
        bound = 4 * k * EPS * (abs(alpha) * (np.abs(opA) @ np.abs(opA).T) + abs(beta) * np.abs(C0))
        assert np.all(np.abs(C - ref)[msk] <= bound[msk]), (alpha, beta)
        assert np.array_equal(C[~msk], Cin[~msk], equal_nan=True)
        # SYR2K
        C = Cin.copy(order="F")
        assert xk.dsyr2k(uplo, trans, n, k, alpha, A, shp[0], B, shp[0], beta, C, n) == 0
        ref = C0.copy(order="F")
        oracle.dsyr2k(uplo, trans, n, k, alpha, A, B, beta, ref)
        mag = np.abs(opA) @ np.abs(opB).T + np.abs(opB) @ np.abs(opA).T
        bound = 4 * 2 * k * EPS * (abs(alpha) * mag + abs(beta) * np.abs(C0))
        assert np.all(np.abs(C - ref)[msk] <= bound[msk]), (alpha, beta)
        assert np.array_equal(C[~msk], Cin[~msk], equal_nan=True)


@pytest.mark.parametrize("side,uplo", list(itertools.product("LR", "LU")))
def test_symm(lib, side, uplo):
    m, n = 300, 230
    ka = m if side == "L" else n
    A = inputs.uniform(1, ka, ka)
    Ap = A.copy(order="F")
    Ap[~tri_mask(ka, uplo == "L")] = np.nan  # only the uplo triangle is read
    B = inputs.uniform(2, m, n); C0 = inputs.uniform(3, m, n)
    C = C0.copy(order="F")
    assert xk.dsymm(side, uplo, m, n, 1.5, Ap, ka, B, m, -0.75, C, m) == 0
    ref = C0.copy(order="F")
    oracle.dsymm(side, uplo, m, n, 1.5, Ap, B, -0.75, ref)
    S = np.where(tri_mask(ka, uplo == "L"), A, A.T)
    mag = (np.abs(S) @ np.abs(B)) if side == "L" else (np.abs(B) @ np.abs(S))
    assert np.all(np.abs(C - ref) <= 4 * ka * EPS * (1.5 * mag + 0.75 * np.abs(C0)))
    assert np.linalg.norm(C - ref) <= 1e-13 * np.linalg.norm(ref)


FLAGS = list(itertools.product("LR", "LU", "NT", "NU"))


def tri_of(L, lower, unit):
    T = np.where(tri_mask(L.shape[0], lower), np.nan_to_num(L, nan=0.0), 0.0)
    if unit:
        T[np.diag_indices(L.shape[0])] = 1.0
    return T


@pytest.mark.parametrize("side,uplo,ta,diag", FLAGS)
def test_trmm_trsm(lib, side, uplo, ta, diag):
    m, n = 300, 200
    ka = m if side == "L" else n
    lower, unit = uplo == "L", diag == "U"
    L = inputs.tri_dd(4, ka, lower=lower, fill=np.nan)  # Q9 factor, opposite triangle NaN
    if unit:
        L[np.diag_indices(ka)] = np.nan  # diag='U': the diagonal is not read
    B0 = inputs.uniform(2, m, n)
    T = tri_of(L, lower, unit)
    opT = T.T if ta == "T" else T
    # TRMM
    X = B0.copy(order="F")
    assert xk.dtrmm(side, uplo, ta, diag, m, n, 1.5, L, ka, X, m) == 0
    ref = B0.copy(order="F")
    oracle.dtrmm(side, uplo, ta, diag, m, n, 1.5, L, ref)
    mag = (np.abs(opT) @ np.abs(B0)) if side == "L" else (np.abs(B0) @ np.abs(opT))
    assert np.all(np.abs(X - ref) <= 4 * ka * EPS * 1.5 * mag)
    # TRSM
    X = B0.copy(order="F")
    assert xk.dtrsm(side, uplo, ta, diag, m, n, 1.5, L, ka, X, m) == 0
    ref = B0.copy(order="F")
    oracle.dtrsm(side, uplo, ta, diag, m, n, 1.5, L, ref)
    assert np.linalg.norm(X - ref) <= 1e-13 * np.linalg.norm(ref)
    R = (opT @ X - 1.5 * B0) if side == "L" else (X @ opT - 1.5 * B0)
    magr = (np.abs(opT) @ np.abs(X)) if side == "L" else (np.abs(X) @ np.abs(opT))
    assert np.all(np.abs(R) <= 4 * ka * EPS * (magr + 1.5 * np.abs(B0)) * 1.0000001)


def test_trsm_bidiagonal_exact(lib):
    """L = D(I - S), D = diag(2^p): X = alpha * prefix sums of D^-1 B exactly (bitwise)."""
    m, n = 333, 70
    p = (np.arange(m) % 5) - 2
    L = fmat(np.diag(2.0 ** p) @ (np.eye(m) - np.diag(np.ones(m - 1), -1)))
    L[np.triu_indices(m, 1)] = np.nan
    B0 = inputs.integers(7, m, n)
    X = B0.copy(order="F")
    assert xk.dtrsm("L", "L", "N", "N", m, n, 2.0, L, m, X, m) == 0
    assert np.array_equal(X, 2.0 * np.cumsum((2.0 ** -p)[:, None] * B0, axis=0))


def test_trmm_exact_integers(lib):
    m, n = 260, 190
    A = inputs.integers(3, m, m, lo=-2, span=5)
    B0 = inputs.integers(4, m, n)
    for side, uplo, ta in [("L", "L", "N"), ("L", "U", "T"), ("R", "L", "T"), ("R", "U", "N")]:
        ka = m if side == "L" else n
        Ak = A[:ka, :ka].copy(order="F")
        Bs = B0[:m, :n].copy(order="F")
        X = Bs.copy(order="F")
        assert xk.dtrmm(side, uplo, ta, "N", m, n, -2.0, Ak, ka, X, m) == 0
        ref = Bs.copy(order="F")
        oracle.dtrmm(side, uplo, ta, "N", m, n, -2.0, Ak, ref)
        assert np.array_equal(X, ref), (side, uplo, ta)


def test_trsm_gemm_composition():
    """Paper Figs. 8/9 composition: X = L^-1 B async, then C = X*D async without
    intermediate coherence; only the final C is made coherent.  Same numbers as the
    synchronous path, and no H2D of X in the second call."""
    G, T, N = 4, 128, 384
    L = inputs.tri_dd(4, N, lower=True, fill=np.nan)
    B0 = inputs.uniform(2, N, N); D = inputs.uniform(5, N, N)
    xk.init(ngpus=G, phys=device_map(G), tile=T, probe=False)
    try:
        Xs = B0.copy(order="F"); Cs = np.zeros((N, N), order="F")
        xk.dtrsm("L", "L", "N", "N", N, N, 1.5, L, N, Xs, N)
        xk.dgemm("N", "N", N, N, N, 1.0, Xs, N, D, N, 0.0, Cs, N)
        X = B0.copy(order="F"); C = np.full((N, N), -3.0, order="F")
        xk.reset_stats()
        xk.dtrsm("L", "L", "N", "N", N, N, 1.5, L, N, X, N, asynchronous=True)
        h1 = sum(xk.get_stats()["h2d_bytes"])
        xk.dgemm_async("N", "N", N, N, N, 1.0, X, N, D, N, 0.0, C, N)
        h2 = sum(xk.get_stats()["h2d_bytes"]) - h1
        assert h2 == 8 * N * N  # only D crosses PCIe; X comes from the GPUs
        xk.memory_coherent_sync(N, N, C, N)
        assert np.array_equal(C, Cs)
        xk.memory_coherent_sync(N, N, X, N)
        assert np.array_equal(X, Xs)
    finally:
        xk.finalize()
    # against the oracle: X = 1.5 L^-1 B0 (Frobenius + Q13 residual), C = X D (GEMM bound)
    refX = B0.copy(order="F")
    oracle.dtrsm("L", "L", "N", "N", N, N, 1.5, L, refX)
    Lt = tri_of(L, True, False)
    assert np.linalg.norm(X - refX) <= 1e-13 * np.linalg.norm(refX)
    R = Lt @ X - 1.5 * B0
    assert np.all(np.abs(R) <= 4 * N * EPS * (np.abs(Lt) @ np.abs(X) + 1.5 * np.abs(B0)) * 1.0000001)
    refC = np.zeros((N, N), order="F")
    oracle.dgemm("N", "N", N, N, N, 1.0, X, D, 0.0, refC)
    assert np.all(np.abs(C - refC) <= 4 * N * EPS * (np.abs(X) @ np.abs(D)))
    refC2 = np.zeros((N, N), order="F")
    oracle.dgemm("N", "N", N, N, N, 1.0, refX, D, 0.0, refC2)
    assert np.linalg.norm(C - refC2) <= 1e-13 * np.linalg.norm(refC2)


@pytest.mark.parametrize("routine", ["syrk", "syr2k"])
def test_config3_n32768_sampled(routine):
    """BASELINE configs[2] shape (N=32768, lower, NoTrans, T=2048), one GPU: sampled lower
    entries vs the oracle's dot loop (SYRK entry = GEMM entry of A*A^T)."""
    N, T = 32768, 2048
    A = inputs.uniform(1, N, N); B = inputs.uniform(2, N, N) if routine == "syr2k" else None
    C0 = inputs.uniform(3, N, N)
    C = C0.copy(order="F")
    xk.init(ngpus=1, tile=T, probe=False)
    try:
        for X in (A, B, C):
            if X is not None:
                xk.register(X)
        if routine == "syrk":
            assert xk.dsyrk("L", "N", N, N, 1.5, A, N, -0.75, C, N) == 0
        else:
            assert xk.dsyr2k("L", "N", N, N, 1.5, A, N, B, N, -0.75, C, N) == 0
    finally:
        xk.finalize()
    rng = np.random.default_rng(3)
    ii = rng.integers(0, N, 3000); jj = rng.integers(0, N, 3000)
    ii, jj = np.maximum(ii, jj), np.minimum(ii, jj)
    if routine == "syrk":
        ref = oracle.dgemm_sampled("N", "T", N, 1.5, A, A, -0.75, C0[ii, jj], ii, jj)
        mag = 1.5 * np.einsum("qk,qk->q", np.abs(A[ii, :]), np.abs(A[jj, :])) + 0.75 * np.abs(C0[ii, jj])
        kk = N
    else:
        r1 = oracle.dgemm_sampled("N", "T", N, 1.5, A, B, -0.75, C0[ii, jj], ii, jj)
        r2 = oracle.dgemm_sampled("N", "T", N, 1.5, B, A, 0.0, C0[ii, jj], ii, jj)
        ref = r1 + r2
        mag = 1.5 * (np.einsum("qk,qk->q", np.abs(A[ii, :]), np.abs(B[jj, :])) +
                     np.einsum("qk,qk->q", np.abs(B[ii, :]), np.abs(A[jj, :]))) + 0.75 * np.abs(C0[ii, jj])
        kk = 2 * N
    assert np.all(np.abs(C[ii, jj] - ref) <= 4 * kk * EPS * mag * 1.0000001)
    up = rng.integers(0, N, 2000), rng.integers(0, N, 2000)
    ui, uj = np.minimum(*up), np.maximum(*up)
    sel = ui < uj
    assert np.array_equal(C[ui[sel], uj[sel]], C0[ui[sel], uj[sel]])  # upper triangle untouched


@pytest.mark.parametrize("routine", ["trsm", "trmm"])
def test_config4_n32768_vs_oracle(routine):
    """BASELINE configs[3] (N=32768, left, lower, NoTrans, non-unit, T=2048), one GPU, against
    the oracle under the north_star bounds (no numpy reference, no widened slack).
    TRMM: L is stored with zeros above the diagonal, so the oracle's sampled dot loop
    1.5 * L(i,:) B0(:,j) is the TRMM entry by definition; elementwise bound
    4 N 2^-53 |alpha| (|L||B0|)_ij on 4096 sampled entries.
    TRSM: the oracle's solve of 8 sampled columns (it runs op(U) = U^T = L with U = L^T stored
    upper, the same forward substitution in the same order, reading L's rows contiguously);
    relative Frobenius <= 1e-13 and elementwise: both solutions satisfy the Q13 residual bound
    r = 4 N 2^-53 (|L||X| + |alpha||B0|), so |X - X_ref| <= |L^-1| (r + r_ref) <= 2 ||r||_inf
    componentwise -- for the Q9 factor (diag >= 1, |off-diag| <= 1/(2N)) the comparison
    matrix gives ||L^-1||_inf <= 1 / (1 - (N-1)/(2N)) <= 2."""
    N, T = 32768, 2048
    L = inputs.tri_dd(4, N, lower=True, fill=0.0)
    B0 = inputs.uniform(2, N, N)
    X = B0.copy(order="F")
    xk.init(ngpus=1, tile=T, probe=False)
    try:
        xk.register(L); xk.register(X)
        f = xk.dtrsm if routine == "trsm" else xk.dtrmm
        assert f("L", "L", "N", "N", N, N, 1.5, L, N, X, N) == 0
    finally:
        xk.finalize()
    rng = np.random.default_rng(4)
    if routine == "trmm":
        ii = rng.integers(0, N, 4096); jj = rng.integers(0, N, 4096)
        ii[:4] = [0, N - 1, 0, N - 1]; jj[:4] = [0, 0, N - 1, N - 1]
        ref = oracle.dgemm_sampled("N", "N", N, 1.5, L, B0, 0.0, np.zeros(len(ii)), ii, jj)
        mag = 1.5 * np.einsum("qk,kq->q", np.abs(L[ii, :]), np.abs(B0[:, jj]))
        assert np.all(np.abs(X[ii, jj] - ref) <= 4 * N * EPS * mag)
        return
    cols = np.sort(rng.choice(N, 8, replace=False))
    cols[0] = 0
    Bs = np.asfortranarray(B0[:, cols])
    U = np.asfortranarray(L.T)
    ref = Bs.copy(order="F")
    oracle.dtrsm("L", "U", "T", "N", N, len(cols), 1.5, U, ref)
    del U
    Xs = X[:, cols]
    assert np.linalg.norm(Xs - ref) <= 1e-13 * np.linalg.norm(ref)
    absL = np.abs(L)
    r = 4 * N * EPS * (absL @ np.abs(ref) + 1.5 * np.abs(Bs))
    assert np.all(np.abs(Xs - ref) <= 2 * 2 * r.max(axis=0)[None, :] * 1.0000001)
    # and the GPU solution's own residual, componentwise (Q13)
    rg = np.abs(L @ Xs - 1.5 * Bs)
    assert np.all(rg <= 4 * N * EPS * (absL @ np.abs(Xs) + 1.5 * np.abs(Bs)) * 1.0000001)


@pytest.mark.parametrize("routine", ["dsyrk", "dsyr2k", "dtrmm", "dtrsm", "dsymm"])
def test_owner_maps_do_not_change_bits(routine):
    """Readings R11-R13 (triangle round-robin for SYRK/SYR2K, TRSM/TRMM grid oriented along
    B's untouched dimension, TRMM rows snaked) only move tiles between GPUs: every tile's
    chain of operations is the same, so 8 logical GPUs (4x2 grid) give the bits of 1 GPU --
    on real-valued inputs, both sides / triangles."""
    n, k, T = 300, 170, 64
    A = inputs.uniform(1, n, n); B = inputs.uniform(2, n, n); C0 = inputs.uniform(3, n, n)
    L = inputs.tri_dd(4, n, lower=True, fill=0.0); U = np.asfortranarray(L.T)
    Ak = inputs.uniform(5, n, k); Bk = inputs.uniform(6, n, k)

    def run(G):
        xk.init(ngpus=G, phys=device_map(G), tile=T, probe=False)
        outs = []
        try:
            for side, uplo in itertools.product("LR", "LU"):
                X = C0.copy(order="F")
                if routine == "dsyrk":
                    assert xk.dsyrk(uplo, "N" if side == "L" else "T", n, k if side == "L" else n, 1.5,
                                    Ak if side == "L" else A, n, -0.75, X, n) == 0
                elif routine == "dsyr2k":
                    assert xk.dsyr2k(uplo, "N", n, k, 1.5, Ak, n, Bk, n, -0.75, X, n) == 0
                elif routine == "dsymm":
                    assert xk.dsymm(side, uplo, n, n, 1.5, A, n, B, n, -0.75, X, n) == 0
                else:
                    f = xk.dtrsm if routine == "dtrsm" else xk.dtrmm
                    tri = L if uplo == "L" else U
                    assert f(side, uplo, "N", "N", n, n, 1.5, tri, n, X, n) == 0
                outs.append(X)
        finally:
            xk.finalize()
        return outs

    for a, b in zip(run(1), run(8)):
        assert np.array_equal(a, b)


@pytest.mark.parametrize("G", [1, 8])
def test_trmm_shadow_matches_in_place(G):
    """Reading R15: host-resident DTRMM runs the shadow sweep (B's input from a per-call
    shadow, top-down), data-on-device DTRMM the in-place bottom-up sweep.  Each output tile
    sums the same terms in the same order (diagonal multiply, then contributions nearest the
    diagonal first), so the two results are bitwise equal; and the shadow sweep moves B over
    PCIe exactly once (H2D = B + the stored triangle's tiles of A)."""
    T = 128
    xk.init(ngpus=G, phys=device_map(G), tile=T, probe=False)
    try:
        m, n = 300, 260
        L = inputs.tri_dd(4, m, lower=True, fill=np.nan)
        B0 = inputs.uniform(2, m, n)
        X1 = B0.copy(order="F")
        xk.reset_stats()
        assert xk.dtrmm("L", "L", "N", "N", m, n, 1.5, L, m, X1, m) == 0
        st = xk.get_stats()
        rows = [min(T, m - i * T) for i in range(-(-m // T))]
        tri_bytes = 8 * sum(rows[i] * rows[j] for i in range(len(rows)) for j in range(i + 1))
        assert sum(st["h2d_bytes"]) == 8 * m * n + tri_bytes
        X2 = B0.copy(order="F")
        xk.memory_prefetch_async(m, n, X2, m)
        xk.memory_prefetch_async(m, m, L, m)
        xk.sync()
        assert xk.dtrmm("L", "L", "N", "N", m, n, 1.5, L, m, X2, m, asynchronous=True) == 0
        assert xk.memory_coherent_sync(m, n, X2, m) == 0
        assert np.array_equal(X1, X2)
        ref = B0.copy(order="F")
        oracle.dtrmm("L", "L", "N", "N", m, n, 1.5, L, ref)
        T_ = tri_of(L, True, False)
        assert np.all(np.abs(X1 - ref) <= 4 * m * EPS * 1.5 * (np.abs(T_) @ np.abs(B0)))
    finally:
        xk.finalize()
