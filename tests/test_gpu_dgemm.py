"""End-to-end parity of xk_dgemm / xk_dgemm_async (host-resident column-major matrices,
tile tasks on the GPU, plan-driven H2D/P2P/D2H) against the CPU oracle.

Tolerance (north_star): elementwise 4*k*2^-53*(|alpha||A||B| + |beta||C|), relative
Frobenius <= 1e-13; exact-integer inputs bitwise.  Multi-GPU logic runs in logical-device
mode (G logical GPUs mapped onto the one physical B200; peer copies become D2D copies).
"""
import numpy as np
import pytest

import inputs
import oracle
import paper_conf_sc_gautierl21_b200 as xk
from tests.gpu_util import device_map

pytestmark = pytest.mark.gpu


def shp(t, r, c):
    return (c, r) if t == "T" else (r, c)


@pytest.fixture
def lib1():
    xk.init(ngpus=1, tile=256, probe=False)
    yield
    xk.finalize()


def logical(G, **kw):
    xk.init(ngpus=G, phys=device_map(G), probe=False, **kw)


def check_bound(ta, tb, m, n, k, alpha, A, B, beta, C0, got, ref):
    bound = oracle.gemm_bound(ta, tb, m, n, k, alpha, A, B, beta, C0)
    assert np.all(np.abs(got[:m, :n] - ref[:m, :n]) <= bound)
    assert np.linalg.norm(got[:m, :n] - ref[:m, :n]) <= 1e-13 * max(np.linalg.norm(ref[:m, :n]), 1e-300)


def test_config1_n1024_t256(lib1):
    """BASELINE configs[0]: DGEMM N=1024, tile 256, 1 GPU, host-resident, vs the oracle."""
    N = 1024
    A, B, C0 = inputs.uniform(1, N, N), inputs.uniform(2, N, N), inputs.uniform(3, N, N)
    for a in (A, B, C0):
        xk.register(a)
    C = C0.copy(order="F")
    xk.register(C)
    xk.reset_stats()
    assert xk.dgemm("N", "N", N, N, N, 1.5, A, N, B, N, -0.75, C, N) == 0
    ref = C0.copy(order="F")
    oracle.dgemm("N", "N", N, N, N, 1.5, A, B, -0.75, ref)
    check_bound("N", "N", N, N, N, 1.5, A, B, -0.75, C0, C, ref)
    st = xk.get_stats()
    assert st["h2d_bytes"][0] == 3 * 8 * N * N and st["d2h_bytes"][0] == 8 * N * N
    assert st["tasks"][0] == 4 * 4 * 4 and st["p2p_in_bytes"][0] == 0


@pytest.mark.parametrize("ta,tb", [("N", "N"), ("N", "T"), ("T", "N"), ("T", "T")])
def test_ragged_transposes_padding(lib1, ta, tb):
    m, n, k = 700, 389, 513
    lda = shp(ta, m, k)[0] + 8
    ldb = shp(tb, k, n)[0] + 3
    ldc = m + 5
    A = inputs.uniform(1, *shp(ta, m, k), ld=lda)
    B = inputs.uniform(2, *shp(tb, k, n), ld=ldb)
    C0 = inputs.uniform(3, m, n, ld=ldc)
    C0[m:] = 99.0
    for alpha, beta in [(1.5, -0.75), (1.5, 0.0), (0.0, 2.0), (-1.0, 1.0)]:
        C = C0.copy(order="F")
        if beta == 0.0:
            C[:m] = np.nan  # not read
        assert xk.dgemm(ta, tb, m, n, k, alpha, A, lda, B, ldb, beta, C, ldc) == 0
        ref = C0.copy(order="F")
        oracle.dgemm(ta, tb, m, n, k, alpha, A, B, beta, ref, lda=lda, ldb=ldb, ldc=ldc)
        rows_a = shp(ta, m, k)[0]
        rows_b = shp(tb, k, n)[0]
        check_bound(ta, tb, m, n, k, alpha, A[:rows_a], B[:rows_b], beta, C0[:m], C, ref)
        assert np.all(C[m:] == 99.0)  # padding rows never written


def test_exact_integers_bitwise_all_G():
    """Exact-integer inputs: bitwise equal to the oracle for G = 1, 2, 4, 8 (logical)."""
    m, n, k = 600, 520, 700
    A, B, C0 = inputs.integers(1, m, k), inputs.integers(2, k, n), inputs.integers(3, m, n)
    ref = C0.copy(order="F")
    oracle.dgemm("N", "N", m, n, k, -2.0, A, B, 0.5, ref)
    for G in (1, 2, 4, 8):
        logical(G, tile=128)
        C = C0.copy(order="F")
        assert xk.dgemm("N", "N", m, n, k, -2.0, A, m, B, k, 0.5, C, m) == 0
        xk.finalize()
        assert np.array_equal(C, ref), G


@pytest.mark.parametrize("mode,opt", [("ranked", True), ("ranked", False), ("unranked", False), ("home", True)])
def test_heuristic_modes_same_numbers_bytes_follow_plan(mode, opt):
    """Heuristics change only where tiles come from: results are bitwise identical across
    modes and GPU counts; measured bytes equal the plan's (App. B closed forms for FULL/HOME)."""
    G, T, t = 8, 128, 4
    N = T * t
    A, B, C0 = inputs.uniform(1, N, N), inputs.uniform(2, N, N), inputs.uniform(3, N, N)
    logical(1, tile=T)
    Cref = C0.copy(order="F")
    xk.dgemm("N", "N", N, N, N, 1.5, A, N, B, N, -0.75, Cref, N)
    xk.finalize()
    logical(G, tile=T, topo=mode, optimistic=opt, grid=(4, 2))
    xk.reset_stats()
    C = C0.copy(order="F")
    xk.dgemm("N", "N", N, N, N, 1.5, A, N, B, N, -0.75, C, N)
    st = xk.get_stats()
    xk.finalize()
    assert np.array_equal(C, Cref)
    tile_b = 8 * T * T
    h2d, p2p = sum(st["h2d_bytes"]), sum(st["p2p_in_bytes"])
    L = st["link_bytes"]  # per-link matrix agrees with the per-GPU counters
    assert sum(L[G][g] for g in range(G)) == h2d and sum(L[g][G] for g in range(G)) == sum(st["d2h_bytes"])
    assert sum(L[s][d] for s in range(G) for d in range(G)) == p2p
    assert sum(st["d2h_bytes"]) == t * t * tile_b
    rA, rB = 2, 4  # min(Q, t), min(P, t)
    if mode == "home":
        assert h2d == (t * t * rA + t * t * rB + t * t) * tile_b and p2p == 0
    elif opt:
        assert h2d == (3 * t * t) * tile_b
        assert p2p == (t * t * (rA - 1) + t * t * (rB - 1)) * tile_b
    else:
        assert (3 * t * t) * tile_b <= h2d <= (t * t * rA + t * t * rB + t * t) * tile_b


def test_async_coherence_and_composition():
    """E = (A*B)*C2 with two async calls and no intermediate coherence: the
    second call reads D from the GPUs (no H2D of D); the host copy of D stays stale until
    coherence; results equal the synchronous path bitwise."""
    G, T = 4, 128
    N = 512
    A, B, C2 = inputs.uniform(1, N, N), inputs.uniform(2, N, N), inputs.uniform(6, N, N)
    logical(G, tile=T)
    Ds = np.zeros((N, N), order="F")
    Es = np.zeros((N, N), order="F")
    xk.dgemm("N", "N", N, N, N, 1.0, A, N, B, N, 0.0, Ds, N)
    xk.dgemm("N", "N", N, N, N, 1.0, Ds, N, C2, N, 0.0, Es, N)
    D = np.full((N, N), -7.0, order="F")
    E = np.full((N, N), -7.0, order="F")
    xk.reset_stats()
    xk.dgemm_async("N", "N", N, N, N, 1.0, A, N, B, N, 0.0, D, N)
    h2d_1 = sum(xk.get_stats()["h2d_bytes"])
    xk.dgemm_async("N", "N", N, N, N, 1.0, D, N, C2, N, 0.0, E, N)
    h2d_2 = sum(xk.get_stats()["h2d_bytes"]) - h2d_1
    assert h2d_2 == 8 * N * N  # only C2 crosses PCIe; D comes from the GPUs
    xk.sync()
    assert np.all(D == -7.0) and np.all(E == -7.0)  # lazy: nothing written back yet
    # partial coherence writes only the requested sub-view
    xk.memory_coherent_sync(100, 37, E[5:, 11:], N)
    assert np.array_equal(E[5:105, 11:48], Es[5:105, 11:48])
    mask = np.ones((N, N), bool); mask[5:105, 11:48] = False
    assert np.all(E[mask] == -7.0)
    xk.memory_coherent_sync(N, N, E, N)
    xk.memory_coherent_sync(N, N, D, N)
    assert np.array_equal(D, Ds) and np.array_equal(E, Es)
    xk.finalize()
    ref_D = np.zeros((N, N), order="F")
    oracle.dgemm("N", "N", N, N, N, 1.0, A, B, 0.0, ref_D)
    check_bound("N", "N", N, N, N, 1.0, A, B, 0.0, ref_D, D, ref_D)


def test_device_resident_repeat_and_invalidate():
    """Data-on-device: prefetch, then repeated async calls reuse the cached tiles (no H2D);
    C is updated on the GPU in place and made coherent once."""
    N, T = 512, 128
    A, B, C0 = inputs.uniform(1, N, N), inputs.uniform(2, N, N), inputs.uniform(3, N, N)
    logical(2, tile=T)
    C = C0.copy(order="F")
    for X in (A, B, C):
        xk.memory_prefetch_async(N, N, X, N)
    xk.sync()
    xk.reset_stats()
    for _ in range(3):
        xk.dgemm_async("N", "N", N, N, N, 1.5, A, N, B, N, -0.75, C, N)
        xk.sync()
    st = xk.get_stats()
    assert sum(st["h2d_bytes"]) == 0 and sum(st["d2h_bytes"]) == 0
    xk.memory_coherent_sync(N, N, C, N)
    ref = C0.copy(order="F")
    for _ in range(3):
        oracle.dgemm("N", "N", N, N, N, 1.5, A, B, -0.75, ref)
    assert np.linalg.norm(C - ref) <= 1e-13 * np.linalg.norm(ref)
    xk.memory_invalidate(N, N, C, N)
    xk.memory_invalidate(N, N, A, N)
    xk.finalize()


def test_full_size_n16384_exact_freivalds():
    """BASELINE configs[1] size (N=16384, T=2048), exact-integer inputs: Freivalds check
    C*x == alpha*A*(B*x) + beta*C0*x exactly (all magnitudes < 2^53)."""
    N, T = 16384, 2048
    A, B, C0 = inputs.integers(1, N, N), inputs.integers(2, N, N), inputs.integers(3, N, N)
    for X in (A, B):
        pass
    C = C0.copy(order="F")
    xk.init(ngpus=1, tile=T, probe=False)
    xk.register(A); xk.register(B); xk.register(C)
    assert xk.dgemm("N", "N", N, N, N, 2.0, A, N, B, N, -1.0, C, N) == 0
    xk.finalize()
    rng = np.random.default_rng(5)
    for _ in range(2):
        x = rng.integers(-4, 5, N).astype(np.float64)
        lhs = C @ x
        rhs = 2.0 * (A @ (B @ x)) - 1.0 * (C0 @ x)
        assert np.array_equal(lhs, rhs)


@pytest.mark.parametrize("T", [2048, 4096])
def test_eight_logical_gpus_full_tiles_exact(T):
    """8 logical GPUs (4x2 grid, the north-star layout) at the bench's tile sizes, N=16384,
    exact-integer inputs: 4096 sampled entries bitwise equal to the oracle's dot loop (every
    summation order is exact here) and an exact Freivalds check of the whole C."""
    N = 16384
    A, B, C0 = inputs.integers(1, N, N), inputs.integers(2, N, N), inputs.integers(3, N, N)
    C = C0.copy(order="F")
    logical(8, tile=T)
    try:
        xk.register(A); xk.register(B); xk.register(C)
        xk.reset_stats()
        assert xk.dgemm("N", "N", N, N, N, 2.0, A, N, B, N, -1.0, C, N) == 0
        st = xk.get_stats()
    finally:
        xk.finalize()
    t = N // T
    assert sum(st["tasks"]) == t ** 3 and all(x > 0 for x in st["tasks"])
    rng = np.random.default_rng(11)
    ii = rng.integers(0, N, 4096); jj = rng.integers(0, N, 4096)
    ref = oracle.dgemm_sampled("N", "N", N, 2.0, A, B, -1.0, C0[ii, jj], ii, jj)
    assert np.array_equal(C[ii, jj], ref)
    x = rng.integers(-4, 5, N).astype(np.float64)
    assert np.array_equal(C @ x, 2.0 * (A @ (B @ x)) - 1.0 * (C0 @ x))


@pytest.mark.parametrize("N,T", [(32768, 4096), (32768, 2048), (65536, 4096)])
def test_full_size_sampled(N, T):
    """The bench workload (N=32768, T=4096 -- bench.py's launch configuration -- and T=2048)
    and the largest BASELINE size (N=65536), G=1, uniform [-1,1): 4096 sampled entries vs the
    oracle's dot loop under the elementwise bound."""
    A, B, C = inputs.uniform(1, N, N), inputs.uniform(2, N, N), inputs.uniform(3, N, N)
    rng = np.random.default_rng(7)
    ii = rng.integers(0, N, 4096); jj = rng.integers(0, N, 4096)
    ii[:4] = [0, N - 1, 0, N - 1]; jj[:4] = [0, 0, N - 1, N - 1]
    c0 = C[ii, jj].copy()  # C is overwritten in place; keep only the sampled inputs
    xk.init(ngpus=1, tile=T, probe=False)
    try:
        xk.register(A); xk.register(B); xk.register(C)
        assert xk.dgemm("N", "N", N, N, N, 1.5, A, N, B, N, -0.75, C, N) == 0
    finally:
        xk.finalize()
    ref = oracle.dgemm_sampled("N", "N", N, 1.5, A, B, -0.75, c0, ii, jj)
    mag = 1.5 * np.einsum("qk,kq->q", np.abs(A[ii, :]), np.abs(B[:, jj])) + 0.75 * np.abs(c0)
    assert np.all(np.abs(C[ii, jj] - ref) <= 4 * N * 2.0 ** -53 * mag)


def test_empty_and_degenerate_calls(lib1):
    """m = 0, n = 0, k = 0 and alpha = 0 cases after init: no work or C <- beta*C only."""
    A = inputs.uniform(1, 64, 64)
    C0 = inputs.uniform(3, 64, 64)
    xk.reset_stats()
    C = C0.copy(order="F")
    assert xk.dgemm("N", "N", 0, 64, 64, 1.0, A, 64, A, 64, 0.0, C, 64) == 0
    assert xk.dgemm("N", "N", 64, 0, 64, 1.0, A, 64, A, 64, 0.0, C, 64) == 0
    assert xk.get_stats()["tasks"][0] == 0 and np.array_equal(C, C0)
    assert xk.dgemm("N", "N", 64, 64, 0, 1.0, A, 64, A, 64, -2.0, C, 64) == 0  # k = 0: C <- beta*C
    assert np.array_equal(C, -2.0 * C0)
    C = C0.copy(order="F")
    assert xk.dgemm("N", "N", 64, 64, 64, 0.0, A, 64, A, 64, 0.0, C, 64) == 0  # alpha = beta = 0
    assert np.all(C == 0)
    C = C0.copy(order="F")
    assert xk.dgemm("N", "N", 1, 1, 1, 1.5, A, 64, A, 64, 1.0, C, 64) == 0  # 1 x 1 x 1
    assert C[0, 0] == C0[0, 0] + 1.5 * A[0, 0] * A[0, 0]
    assert np.array_equal(C[1:], C0[1:]) and np.array_equal(C[:, 1:], C0[:, 1:])


def test_trace_timeline(tmp_path):
    """xk_trace: every copy and kernel launch appears in the Chrome trace with its bytes /
    flops; the per-kind byte totals equal the executor's counters (paper Fig. 6 breakdown)."""
    import json
    G, T, N = 2, 128, 384
    A, B, C = inputs.uniform(1, N, N), inputs.uniform(2, N, N), inputs.uniform(3, N, N)
    logical(G, tile=T)
    try:
        path = str(tmp_path / "trace.json")
        xk.reset_stats()
        xk.trace(path)
        xk.dgemm("N", "N", N, N, N, 1.5, A, N, B, N, -0.75, C, N)
        xk.trace(None)
        st = xk.get_stats()
    finally:
        xk.finalize()
    ev = json.load(open(path))["traceEvents"]
    by = {}
    for e in ev:
        by.setdefault(e["tid"], 0)
        by[e["tid"]] += e["args"].get("bytes", 0)
        assert e["dur"] >= 0
    assert by["H2D"] == sum(st["h2d_bytes"]) and by["D2H"] == sum(st["d2h_bytes"])
    assert by["P2P-in"] == sum(st["p2p_in_bytes"]) > 0
    assert any(e["tid"] == "kernels" for e in ev)
    assert st["trace_ms"]["kernel"] > 0 and st["trace_ms"]["h2d"] > 0


def test_out_of_memory_fails_cleanly():
    """No eviction: when the device tile cache cannot grow, the call returns
    XK_ERR_OOM instead of crashing, later calls refuse to run on the inconsistent cache, and
    re-initialisation recovers."""
    import torch
    N, T = 8192, 2048
    A, B, C = inputs.uniform(1, N, N), inputs.uniform(2, N, N), inputs.uniform(3, N, N)
    free, _ = torch.cuda.mem_get_info()
    hog = torch.empty(int(free - (600 << 20)) // 8, dtype=torch.float64, device="cuda")  # leave ~600 MB
    try:
        xk.init(ngpus=1, tile=T, probe=False)
        with pytest.raises(xk.XKError) as e:
            xk.dgemm("N", "N", N, N, N, 1.0, A, N, B, N, 0.0, C, N)  # needs 1.5 GB of tiles
        assert e.value.code == 3  # XK_ERR_OOM
        with pytest.raises(xk.XKError):
            xk.dgemm("N", "N", N, N, N, 1.0, A, N, B, N, 0.0, C, N)  # sticky until re-init
        xk.finalize()
    finally:
        del hog
        torch.cuda.empty_cache()
    xk.init(ngpus=1, tile=T, probe=False)
    C2 = np.zeros((N, N), order="F")
    assert xk.dgemm("N", "N", 512, 512, 512, 1.0, A, N, B, N, 0.0, C2, N) == 0
    xk.finalize()


def test_invalidate_without_coherence_then_host_rewrite():
    """The host array is authoritative after xk_memory_invalidate: results that lived only
    on the GPUs are dropped, the caller rewrites the host array, and the next call reads it."""
    N, T = 300, 128
    A, B = inputs.integers(1, N, N), inputs.integers(2, N, N)
    D = np.zeros((N, N), order="F")
    logical(2, tile=T)
    try:
        assert xk.dgemm_async("N", "N", N, N, N, 1.0, A, N, B, N, 0.0, D, N) == 0
        xk.sync()
        xk.memory_invalidate(N, N, D, N)          # D's result never reaches the host
        D[:] = inputs.integers(3, N, N)           # the caller's new contents
        E = np.zeros((N, N), order="F")
        assert xk.dgemm("N", "N", N, N, N, 1.0, D, N, B, N, 0.0, E, N) == 0
    finally:
        xk.finalize()
    ref = np.zeros((N, N), order="F")
    oracle.dgemm("N", "N", N, N, N, 1.0, np.asfortranarray(inputs.integers(3, N, N)), B, 0.0, ref)
    assert np.array_equal(E, ref)


@pytest.mark.parametrize("G", [1, 4])
def test_async_then_sync_then_coherent(G):
    """async D = A*B, then a synchronous E = D*C2 that reads D from the
    GPUs, then coherent(D): D comes back exactly (exact integers, bitwise vs the oracle) --
    the sync call must not drop D's only current copies.  Also async TRSM then sync GEMM."""
    N, T = 384, 128
    A, B, C2 = inputs.integers(1, N, N), inputs.integers(2, N, N), inputs.integers(6, N, N)
    ref_D = np.zeros((N, N), order="F")
    oracle.dgemm("N", "N", N, N, N, 1.0, A, B, 0.0, ref_D)
    ref_E = np.zeros((N, N), order="F")
    oracle.dgemm("N", "N", N, N, N, 1.0, ref_D, C2, 0.0, ref_E)
    logical(G, tile=T)
    try:
        D = np.full((N, N), -7.0, order="F")
        E = np.full((N, N), -7.0, order="F")
        assert xk.dgemm_async("N", "N", N, N, N, 1.0, A, N, B, N, 0.0, D, N) == 0
        assert xk.dgemm("N", "N", N, N, N, 1.0, D, N, C2, N, 0.0, E, N) == 0
        assert np.array_equal(E, ref_E)
        assert np.all(D == -7.0)  # not coherent yet (lazy)
        assert xk.memory_coherent_sync(N, N, D, N) == 0
        assert np.array_equal(D, ref_D)
        # TRSM (async) -> GEMM (sync) -> coherent(X): L diagonally dominant, Q13 bound on X
        L = inputs.tri_dd(4, N, lower=True)
        X = inputs.uniform(2, N, N)
        X0 = X.copy(order="F")
        F2 = np.zeros((N, N), order="F")
        assert xk.dtrsm("L", "L", "N", "N", N, N, 1.5, L, N, X, N, asynchronous=True) == 0
        assert xk.dgemm("N", "N", N, N, N, 1.0, X, N, C2, N, 0.0, F2, N) == 0
        assert np.array_equal(X, X0)
        assert xk.memory_coherent_sync(N, N, X, N) == 0
    finally:
        xk.finalize()
    refX = X0.copy(order="F")
    oracle.dtrsm("L", "L", "N", "N", N, N, 1.5, L, refX)
    assert np.linalg.norm(X - refX) <= 1e-13 * np.linalg.norm(refX)
    refF = np.zeros((N, N), order="F")
    oracle.dgemm("N", "N", N, N, N, 1.0, X, C2, 0.0, refF)
    check_bound("N", "N", N, N, N, 1.0, X, C2, 0.0, refF, F2, refF)


@pytest.mark.parametrize("grid", [(2, 4), (4, 2)])
def test_distribute_2dbc_then_dgemm(grid):
    """Data on device the paper's way (xkblas_distribute_2Dblock_cyclic_async):
    A, B, C distributed over 8 logical GPUs on a (P, Q) grid with (1, 1) blocks, then an async
    DGEMM: no byte crosses PCIe during the call (H2D = 0), every tile one H2D in the
    distribution; exact integers, bitwise vs the oracle after coherence."""
    N, T = 768, 128
    A, B, C0 = inputs.integers(1, N, N), inputs.integers(2, N, N), inputs.integers(3, N, N)
    C = C0.copy(order="F")
    ref = C0.copy(order="F")
    oracle.dgemm("N", "N", N, N, N, 2.0, A, B, -1.0, ref)
    logical(8, tile=T)
    try:
        xk.reset_stats()
        for X in (A, B, C):
            assert xk.distribute_2dbc_async(N, N, X, N, *grid) == 0
        xk.sync()
        st = xk.get_stats()
        assert sum(st["h2d_bytes"]) == 3 * 8 * N * N
        P, Q = grid
        t = N // T
        per = [0] * 8
        for bi in range(t):
            for bj in range(t):
                per[(bi % P) * Q + bj % Q] += 3 * 8 * T * T
        assert st["h2d_bytes"] == per
        xk.reset_stats()
        assert xk.dgemm_async("N", "N", N, N, N, 2.0, A, N, B, N, -1.0, C, N) == 0
        xk.sync()
        assert sum(xk.get_stats()["h2d_bytes"]) == 0
        assert xk.memory_coherent_sync(N, N, C, N) == 0
    finally:
        xk.finalize()
    assert np.array_equal(C, ref)
