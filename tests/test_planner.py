"""Planner (libxk.so, C++) vs the CPU model of the heuristics (tests/planmodel.py): the
transfer plan must be bit-exact (north_star), plus pins that come from outside both:
the paper's Fig. 2 matrix and its link classes, the heuristics'
stated preferences, and closed-form byte counts.
No GPU: G virtual GPUs with injected link matrices."""
import itertools
import os
import random

import pytest

import paper_conf_sc_gautierl21_b200 as xk
from tests import planmodel as pm

HERE = os.path.dirname(os.path.abspath(__file__))
HOST_GEN3 = 12000  # MB/s placeholder for the DGX-1 host links


def fig2():
    rows = []
    with open(os.path.join(HERE, "golden", "dgx1_fig2_bw.txt")) as f:
        for line in f:
            line = line.split("#")[0].strip()
            if line:
                rows.append([float(x) for x in line.split()])
    return rows


def with_host(gbps, host=HOST_GEN3):
    """GB/s GPU matrix -> integer MB/s (G+1)^2 matrix with a host row/column."""
    G = len(gbps)
    bw = [[int(round(gbps[s][d] * 1000)) for d in range(G)] + [host] for s in range(G)]
    bw.append([host] * G + [host * 10])
    return bw


def uniform(G, peer=700000, host=55000, local=3000000):
    bw = [[local if s == d else peer for d in range(G)] + [host] for s in range(G)]
    bw.append([host] * G + [local])
    return bw


def random_bw(G, seed):
    r = random.Random(seed)
    bw = [[r.choice([9000, 17000, 33000, 48000, 96000, 400000]) for _ in range(G + 1)] for _ in range(G + 1)]
    for i in range(G + 1):
        bw[i][i] = 1000000
    return bw


# ------------------------------------------------------------------ pins from the paper
def test_fig2_link_classes():
    bw = with_host(fig2())
    cls = pm.classes(bw)
    peer = {cls[s][d] for s in range(8) for d in range(8) if s != d}
    assert len(peer) == 3  # 2 NVLinks / 1 NVLink / PCIe
    host_cls = {cls[s][8] for s in range(8)} | {cls[8][d] for d in range(8)}
    assert host_cls == {0} and min(peer) == 1
    # every GPU has two 2-link peers, two 1-link peers and three PCIe peers (Fig. 1)
    for s in range(8):
        row = sorted(cls[s][d] for d in range(8) if d != s)
        assert row == [1, 1, 1, 2, 2, 3, 3]


def test_fig2_ranked_choice_order():
    """Destination GPU 0 with valid copies on 1 (1 NVLink), 3 (2 NVLinks), 5 (PCIe): the
    topology-aware heuristic takes 3, then 1, then 5; no heuristic takes 1."""
    bw = with_host(fig2())
    for mode, expect in [("ranked", [3, 1, 5]), ("unranked", [1, 3, 5])]:
        m = pm.Model(bw, topo=mode, grid=(4, 2), tile=4)
        t = pm.Tile(4, 4, 0, 0)
        holders = [1, 3, 5]
        got = []
        for _ in range(3):
            t.gpus = {g: pm.Copy(0, 0, -1, 1) for g in holders}
            g, st = m.choose(t, 0, 0, 10)
            assert st == pm.S_VALID
            got.append(g)
            holders.remove(g)
        assert got == expect, mode


def test_optimistic_prefers_inflight_gpu_over_host():
    """valid GPU copy first; otherwise the best GPU with the data under
    transfer instead of the host; with optimistic off, the host."""
    bw = with_host(fig2())
    t = pm.Tile(4, 4, 0, 0)
    t.gpus = {4: pm.Copy(0, 100, 7, 1), 2: pm.Copy(0, 100, 8, 1)}  # in flight until t=100
    on = pm.Model(bw, topo="ranked", optimistic=True, grid=(4, 2), tile=4)
    off = pm.Model(bw, topo="ranked", optimistic=False, grid=(4, 2), tile=4)
    assert on.choose(t, 0, 0, 50) == (4, pm.S_INFLIGHT)  # GPU 4 is 2 NVLinks from 0
    assert off.choose(t, 0, 0, 50) == (pm.HOSTID, pm.S_HOST)
    assert on.choose(t, 0, 0, 100) == (4, pm.S_VALID)  # t_done <= t -> valid
    home = pm.Model(bw, topo="home", grid=(4, 2), tile=4)
    assert home.choose(t, 0, 0, 500) == (pm.HOSTID, pm.S_HOST)


# ------------------------------------------------------------------ bit-exact equivalence
A_ADDR, B_ADDR, C_ADDR, D_ADDR, E_ADDR = 0x10000000, 0x20000000, 0x30000000, 0x40000000, 0x50000000


def both(bw, flags, calls, rate=35000000):
    s = xk.PlanSession(bw, rate, **flags)
    m = pm.Model(bw, rate, **flags)
    got, exp = [], []
    for c in calls:
        got.append(s.call(xk.make_call(**c)))
        exp.append(m.call(**c))
    s.close()
    return got, exp


def gemm(ta="N", tb="N", m=8, n=8, k=8, alpha=1.5, beta=-0.75, A=A_ADDR, B=B_ADDR, C=C_ADDR,
         sync=True, lda=None, ldb=None, ldc=None):
    lda = lda or ((k if ta == "T" else m) + 3)
    ldb = ldb or ((n if tb == "T" else k) + 1)
    ldc = ldc or m
    return dict(routine=pm.DGEMM, transA=ta, transB=tb, m=m, n=n, k=k, alpha=alpha, beta=beta,
                A=A, lda=lda, B=B, ldb=ldb, C=C, ldc=ldc, sync=sync)


TOPOS = {"uniform": uniform, "fig2": lambda G: with_host([r[:G] for r in fig2()[:G]]),
         "random": lambda G: random_bw(G, 17 * G)}


@pytest.mark.parametrize("G", [1, 2, 3, 4, 8])
@pytest.mark.parametrize("topo_name", ["uniform", "fig2", "random"])
def test_bit_exact_single_calls(G, topo_name):
    bw = TOPOS[topo_name](G)
    shapes = [(8, 8, 8), (9, 13, 5), (12, 4, 17), (1, 1, 1), (13, 13, 13)]
    for mode, opt, W in itertools.product(["ranked", "unranked", "home"], [True, False], [1, 2, 3]):
        flags = dict(topo=mode, optimistic=opt, window=W, tile=4)
        for (mm, nn, kk), (ta, tb), beta in itertools.product(shapes[:3], [("N", "N"), ("T", "N"), ("N", "T"), ("T", "T")], [0.0, -0.75]):
            got, exp = both(bw, flags, [gemm(ta, tb, mm, nn, kk, beta=beta)])
            assert got == exp, (G, topo_name, mode, opt, W, mm, nn, kk, ta, tb, beta)
    flags = dict(topo="ranked", optimistic=True, window=2, tile=4)
    for (mm, nn, kk) in shapes[3:]:
        for alpha, beta in [(0.0, 2.0), (0.0, 0.0), (1.5, 1.0), (1.0, 0.0)]:
            got, exp = both(bw, flags, [gemm(m=mm, n=nn, k=kk, alpha=alpha, beta=beta)])
            assert got == exp


@pytest.mark.parametrize("G", [2, 4, 8])
@pytest.mark.parametrize("mode", ["ranked", "unranked", "home"])
def test_bit_exact_composition_sequences(G, mode):
    """Async calls compose through the directory: D = A*B then E = D*C2 with no
    intermediate coherence; then partial coherence, sync, invalidate, prefetch, re-use."""
    bw = random_bw(G, 3) if mode != "ranked" else with_host([r[:G] for r in fig2()[:G]])
    for opt in (True, False):
        flags = dict(topo=mode, optimistic=opt, window=2, tile=4)
        calls = [
            gemm(m=12, n=12, k=12, C=D_ADDR, ldc=12, sync=False),
            gemm(m=12, n=12, k=12, A=D_ADDR, lda=12, B=C_ADDR, ldb=12, C=E_ADDR, ldc=12, sync=False, beta=0.0),
            dict(routine=pm.COHERENT, m=6, n=9, C=E_ADDR + 8 * (3 + 2 * 12), ldc=12),
            dict(routine=pm.COHERENT, m=12, n=12, C=E_ADDR, ldc=12),
            dict(routine=pm.SYNC),
            gemm(ta="T", m=12, n=12, k=12, A=D_ADDR, lda=12, B=E_ADDR, ldb=12, C=C_ADDR, ldc=12,
                 sync=False, beta=1.0),
            dict(routine=pm.COHERENT, m=12, n=12, C=C_ADDR, ldc=12),
            dict(routine=pm.INVALIDATE, m=12, n=12, C=E_ADDR, ldc=12),
            dict(routine=pm.PREFETCH, m=12, n=12, C=E_ADDR, ldc=12),
            gemm(m=12, n=12, k=12, A=E_ADDR, lda=12, B=E_ADDR, ldb=12, C=A_ADDR + 0x100000, ldc=12,
                 sync=True),
        ]
        got, exp = both(bw, flags, calls)
        for q, (g, e) in enumerate(zip(got, exp)):
            assert g == e, (G, mode, opt, q)


def test_bit_exact_random_fuzz():
    r = random.Random(1234)
    for trial in range(60):
        G = r.choice([1, 2, 3, 4, 5, 6, 8])
        bw = random_bw(G, trial)
        flags = dict(topo=r.choice(["ranked", "unranked", "home"]), optimistic=r.random() < 0.5,
                     window=r.choice([1, 2, 4]), tile=r.choice([2, 3, 4, 5]))
        calls = []
        Nt = r.randint(1, 16)  # one extent per trial: every matrix keeps one tiling (step 9)
        for _ in range(r.randint(1, 4)):
            mm, nn, kk = Nt, Nt, Nt
            ta, tb = r.choice("NT"), r.choice("NT")
            calls.append(gemm(ta, tb, mm, nn, kk, alpha=r.choice([1.5, 0.0]), beta=r.choice([0.0, 1.0, -0.75]),
                              C=r.choice([C_ADDR, D_ADDR]), ldc=16, lda=16, ldb=16, sync=r.random() < 0.5))
            if r.random() < 0.3:
                calls.append(dict(routine=pm.COHERENT, m=16, n=16, C=C_ADDR, ldc=16))
        got, exp = both(bw, flags, calls, rate=r.choice([1000, 35000000]))
        assert got == exp, trial


# ------------------------------------------------------------------ closed forms (App. B)
def byte_counts(recs):
    out = {pm.H2D: 0, pm.P2P: 0, pm.D2H: 0}
    per_gpu_h2d = {}
    for r in recs:
        if r[1] in out:
            out[r[1]] += 1
        if r[1] == pm.H2D:
            per_gpu_h2d[r[7]] = per_gpu_h2d.get(r[7], 0) + 1
    return out, per_gpu_h2d


@pytest.mark.parametrize("G,grid", [(1, (1, 1)), (2, (2, 1)), (4, (2, 2)), (8, (4, 2))])
@pytest.mark.parametrize("beta", [0.0, -0.75])
def test_closed_form_tile_counts(G, grid, beta):
    P, Q = grid
    for t in (4, 8, 6):
        T = 4
        N = t * T
        call = xk.make_call(m=N, n=N, k=N, alpha=1.5, beta=beta, A=A_ADDR, lda=N, B=B_ADDR, ldb=N,
                            C=C_ADDR, ldc=N, sync=True)
        rA = [len({(i % P) * Q + (j % Q) for j in range(t)}) for i in range(t)]
        rB = [len({(i % P) * Q + (j % Q) for i in range(t)}) for j in range(t)]
        full = xk.plan_dump(call, uniform(G), topo="ranked", optimistic=True, tile=T)
        c, _ = byte_counts(full)
        assert c[pm.H2D] == t * t + t * t + (t * t if beta else 0)
        assert c[pm.P2P] == t * sum(x - 1 for x in rA) + t * sum(x - 1 for x in rB)
        assert c[pm.D2H] == t * t
        home = xk.plan_dump(call, uniform(G), topo="home", optimistic=True, tile=T)
        c, _ = byte_counts(home)
        assert c[pm.H2D] == t * sum(rA) + t * sum(rB) + (t * t if beta else 0)
        assert c[pm.P2P] == 0
        nopt = xk.plan_dump(call, uniform(G), topo="ranked", optimistic=False, tile=T)
        c2, _ = byte_counts(nopt)
        assert t * t * 2 <= c2[pm.H2D] - (t * t if beta else 0) <= t * sum(rA) + t * sum(rB)


@pytest.mark.parametrize("G,grid", [(2, (2, 1)), (4, (2, 2)), (8, (4, 2))])
@pytest.mark.parametrize("beta", [0.0, -0.75])
def test_host_pulls_balanced_closed_form(G, grid, beta):
    """Reading R16 (balance-aware first host pull): with P | t and Q | t every GPU
    carries exactly (t_m t_k + t_k t_n + [beta != 0] t_m t_n) / G host tiles in FULL mode
    (max/mean = 1.00); the totals are App. B's FULL counts, so no byte moves to another link
    class.  HOME is untouched by R16: every requester reads its own tiles."""
    P, Q = grid
    for t in (8, 16):
        T = 4
        N = t * T
        call = xk.make_call(m=N, n=N, k=N, alpha=1.5, beta=beta, A=A_ADDR, lda=N, B=B_ADDR, ldb=N,
                            C=C_ADDR, ldc=N, sync=True)
        recs = xk.plan_dump(call, uniform(G), topo="ranked", optimistic=True, tile=T)
        _, per = byte_counts(recs)
        total = 2 * t * t + (t * t if beta else 0)
        assert [per.get(g, 0) for g in range(G)] == [total // G] * G
        # HOME: GPU g reads every A tile of its grid row's tiles and every B tile of its column
        home = xk.plan_dump(call, uniform(G), topo="home", optimistic=True, tile=T)
        _, ph = byte_counts(home)
        for g in range(G):
            pi, qj = divmod(g, Q)
            own_c = (t // P) * (t // Q)
            assert ph.get(g, 0) == (t // P) * t + t * (t // Q) + (own_c if beta else 0)


def test_host_pulls_spread_over_gpus():
    """R16 on ragged tile counts (P or Q does not divide t): per-GPU host tiles within 5% of
    the mean (max/mean <= 1.05), totals = App. B FULL."""
    for t in (9, 13, 17, 31):
        T = 4
        N = t * T
        call = xk.make_call(m=N, n=N, k=N, alpha=1.5, beta=0.0, A=A_ADDR, lda=N, B=B_ADDR, ldb=N,
                            C=C_ADDR, ldc=N, sync=True)
        recs = xk.plan_dump(call, uniform(8), topo="ranked", optimistic=True, tile=T)
        _, per = byte_counts(recs)
        vals = [per.get(g, 0) for g in range(8)]
        assert sum(vals) == 2 * t * t
        assert max(vals) <= 1.05 * sum(vals) / 8, (t, vals)


def test_composition_reuses_gpu_outputs():
    """E = D*C2 after D = A*B without intermediate coherence: no H2D of D (App. B)."""
    G, T, t = 8, 4, 8
    N = t * T
    s = xk.PlanSession(uniform(G), topo="ranked", optimistic=True, tile=T)
    s.call(xk.make_call(m=N, n=N, k=N, alpha=1.0, beta=0.0, A=A_ADDR, lda=N, B=B_ADDR, ldb=N,
                        C=D_ADDR, ldc=N, sync=False))
    recs = s.call(xk.make_call(m=N, n=N, k=N, alpha=1.0, beta=0.0, A=D_ADDR, lda=N, B=C_ADDR, ldb=N,
                               C=E_ADDR, ldc=N, sync=False))
    h2d_A = sum(1 for r in recs if r[1] == pm.H2D and r[2] == 0)
    p2p_A = sum(1 for r in recs if r[1] == pm.P2P and r[2] == 0)
    assert h2d_A == 0
    rA = [len({(i % 4) * 2 + (j % 2) for j in range(t)}) for i in range(t)]
    assert p2p_A == t * sum(x - 1 for x in rA)
    s.close()


def test_dependencies_point_backwards():
    """Every dep of a record names an earlier record (single-thread issue in plan order is
    then free of the record-before-wait hazard)."""
    call = xk.make_call(m=40, n=36, k=44, alpha=1.5, beta=-0.75, A=A_ADDR, lda=40, B=B_ADDR, ldb=44,
                        C=C_ADDR, ldc=40, sync=True)
    recs = xk.plan_dump(call, with_host(fig2()), topo="ranked", optimistic=True, tile=4)
    for r in recs:
        for d in r[14]:
            assert d < r[0]
    # each TASK waits on exactly the producers of its A, B (and C) copies on its GPU
    tasks = [r for r in recs if r[1] == pm.TASK]
    assert len(tasks) == 10 * 9 * 11
    assert all(r[14][0] >= 0 and r[14][1] >= 0 for r in tasks)


# ------------------------------------------------------------------ BLAS-3 beyond GEMM (§8(f))
def blas3_calls(routine, N, T, sync=True, alpha=1.5, beta=-0.75):
    base = dict(routine=routine, m=N, n=N, k=N, alpha=alpha, beta=beta, A=A_ADDR, lda=N + 2, B=B_ADDR,
                ldb=N + 1, C=C_ADDR, ldc=N, sync=sync)
    out = []
    if routine in (pm.DSYRK, pm.DSYR2K):
        for uplo, tr in itertools.product("LU", "NT"):
            out.append(dict(base, uplo=uplo, transA=tr))
    elif routine == pm.DSYMM:
        for side, uplo in itertools.product("LR", "LU"):
            out.append(dict(base, side=side, uplo=uplo))
    else:
        for side, uplo, tr, dg in itertools.product("LR", "LU", "NT", "NU"):
            out.append(dict(base, side=side, uplo=uplo, transA=tr, diag=dg))
    return out


@pytest.mark.parametrize("routine", [pm.DSYRK, pm.DSYR2K, pm.DSYMM, pm.DTRMM, pm.DTRSM])
@pytest.mark.parametrize("G", [1, 2, 4, 8])
def test_bit_exact_blas3(routine, G):
    for topo_name, mode, opt in [("fig2", "ranked", True), ("uniform", "ranked", False),
                                 ("random", "unranked", True), ("random", "home", False)]:
        bw = TOPOS[topo_name](G)
        flags = dict(topo=mode, optimistic=opt, window=2, tile=4)
        for N in (13, 16):
            for c in blas3_calls(routine, N, 4):
                got, exp = both(bw, flags, [c])
                assert got == exp, (routine, G, topo_name, mode, opt, N, c)
    # alpha == 0 / beta special values / async + coherence
    bw = TOPOS["fig2"](G)
    flags = dict(topo="ranked", optimistic=True, window=2, tile=4)
    for alpha, beta in [(0.0, 2.0), (0.0, 0.0), (1.5, 0.0), (1.5, 1.0)]:
        cs = blas3_calls(routine, 11, 4, alpha=alpha, beta=beta)[:2]
        got, exp = both(bw, flags, cs)
        assert got == exp, (routine, G, alpha, beta)
    cs = [dict(c, sync=False) for c in blas3_calls(routine, 12, 4)[:1]]
    cs.append(dict(routine=pm.COHERENT, m=12, n=12, C=C_ADDR, ldc=12))
    got, exp = both(bw, flags, cs)
    assert got == exp


def test_trsm_then_gemm_composition():
    """Paper Figs. 8/9: X = L^-1 B (async), then C = X * D with no
    intermediate coherence -- the GEMM reads X from the GPUs (no H2D of X)."""
    G, T, N = 8, 4, 32
    bw = TOPOS["uniform"](G)
    flags = dict(topo="ranked", optimistic=True, window=2, tile=T)
    calls = [dict(routine=pm.DTRSM, side="L", uplo="L", transA="N", diag="N", m=N, n=N, alpha=1.5,
                  A=A_ADDR, lda=N, C=B_ADDR, ldc=N, sync=False),
             dict(routine=pm.DGEMM, m=N, n=N, k=N, alpha=1.0, beta=0.0, A=B_ADDR, lda=N, B=D_ADDR, ldb=N,
                  C=E_ADDR, ldc=N, sync=False),
             dict(routine=pm.COHERENT, m=N, n=N, C=E_ADDR, ldc=N)]
    got, exp = both(bw, flags, calls)
    assert got == exp
    gemm_recs = got[1]
    assert not any(r[1] == pm.H2D and r[2] == 0 for r in gemm_recs)  # X never re-read from host
    assert any(r[1] == pm.P2P and r[2] == 0 for r in gemm_recs)


def test_triangular_task_structure():
    """Task counts of the tiled algorithms (PLASMA structure): SYRK touches only
    the t(t+1)/2 triangle tiles; TRSM has t diagonal solves per column of tiles and
    t(t-1)/2 GEMM updates per column; diagonal tiles carry the diagonal ops."""
    T, t = 4, 5
    N = T * t
    bw = uniform(4)
    syrk = xk.plan_dump(xk.make_call(routine=pm.DSYRK, uplo="L", transA="N", n=N, k=N, alpha=1.0, beta=0.5,
                                     A=A_ADDR, lda=N, C=C_ADDR, ldc=N, sync=True), bw, tile=T)
    tasks = [r for r in syrk if r[1] == pm.TASK]
    assert len(tasks) == t * (t + 1) // 2 * t
    assert all((r[15] == pm.OP_GEMM_TRI) == (r[3] == r[4]) for r in tasks)
    assert all(r[3] >= r[4] for r in tasks)  # lower triangle only
    d2h = [r for r in syrk if r[1] == pm.D2H]
    assert len(d2h) == t * (t + 1) // 2
    trsm = xk.plan_dump(xk.make_call(routine=pm.DTRSM, side="L", uplo="L", transA="N", diag="N", m=N, n=N,
                                     alpha=1.0, A=A_ADDR, lda=N, C=C_ADDR, ldc=N, sync=True), bw, tile=T)
    tasks = [r for r in trsm if r[1] == pm.TASK]
    assert sum(1 for r in tasks if r[15] == pm.OP_TRSM_DIAG) == t * t
    assert sum(1 for r in tasks if r[15] == pm.OP_GEMM) == t * t * (t - 1) // 2
    # L tiles read: only the lower triangle of A is ever copied
    a_tiles = {(r[3], r[4]) for r in trsm if r[1] in (pm.H2D, pm.P2P) and r[2] == 0}
    assert all(i >= j for (i, j) in a_tiles) and len(a_tiles) == t * (t + 1) // 2


def test_beta_deferral_structure():
    """Reading Q12'': a host-valid C tile with a chain of >= 2 tasks is not read by the first
    task (beta = 0, no C dependency); the last task adds beta*C from a shadow copy of the
    original tile (4th dependency, an H2D of operand C at version 0).  C still crosses PCIe
    exactly once per tile; a device-resident C (prefetched) is read in place, no deferral."""
    T = 4
    for G in (1, 4):
        for t in (1, 2, 5):
            N = t * T
            call = xk.make_call(m=N, n=N, k=N, alpha=1.5, beta=-0.75, A=A_ADDR, lda=N, B=B_ADDR, ldb=N,
                                C=C_ADDR, ldc=N, sync=True)
            recs = xk.plan_dump(call, uniform(G), topo="ranked", optimistic=True, tile=T)
            by_seq = {r[0]: r for r in recs}
            tasks = [r for r in recs if r[1] == pm.TASK]
            c_h2d = [r for r in recs if r[1] == pm.H2D and r[2] == 2]
            assert len(c_h2d) == t * t and all(r[6] == 0 for r in c_h2d)
            for r in tasks:
                first, last = r[5] == 0, r[5] == t - 1
                if t == 1:
                    assert r[14][2] >= 0 and r[14][3] == -1
                    continue
                assert (r[14][2] == -1) == first
                assert (r[14][3] >= 0) == last
                if last:
                    src = by_seq[r[14][3]]
                    assert src[1] == pm.H2D and src[2] == 2 and (src[3], src[4]) == (r[3], r[4])
            # the first task of every chain starts before its C tile finished crossing PCIe
            if t >= 2:
                late = sum(1 for r in tasks if r[5] == 0 and r[11] < by_seq[next(
                    x[0] for x in c_h2d if (x[3], x[4]) == (r[3], r[4]))][12])
                assert late > 0
    # data-on-device: prefetched C is read in place
    N, t = 20, 5
    s = xk.PlanSession(uniform(2), topo="ranked", optimistic=True, tile=T)
    s.call(xk.make_call(routine=pm.PREFETCH, m=N, n=N, C=C_ADDR, ldc=N, sync=False))
    recs = s.call(xk.make_call(m=N, n=N, k=N, alpha=1.5, beta=-0.75, A=A_ADDR, lda=N, B=B_ADDR, ldb=N,
                               C=C_ADDR, ldc=N, sync=False))
    assert not any(r[1] == pm.H2D and r[2] == 2 for r in recs)
    assert all(r[14][3] == -1 for r in recs if r[1] == pm.TASK)
    s.close()


@pytest.mark.parametrize("uplo", ["L", "U"])
def test_trsm_lookahead_order(uplo):
    """Readings R9 + R10 on one GPU (D = 2): at time u come the diagonal solves of step u,
    then the update of the row step u+1 solves by step u (lookahead), then the catch-up
    updates of the row solved at step u+D by every step s <= u (s ascending) -- far rows are
    updated just before they are needed, not all in step 0; every tile's chain keeps s
    ascending.  The expected sequence is written out from the rule, independently of the
    planner's sort keys."""
    T, t, D = 4, 5, 2
    N = T * t
    recs = xk.plan_dump(xk.make_call(routine=pm.DTRSM, side="L", uplo=uplo, transA="N", diag="N", m=N, n=N,
                                     alpha=1.0, A=A_ADDR, lda=N, C=C_ADDR, ldc=N, sync=True), uniform(1), tile=T)
    tasks = [r for r in recs if r[1] == pm.TASK]
    order = list(range(t)) if uplo == "L" else list(range(t - 1, -1, -1))  # row solved at step s
    expect = []
    for u in range(t):
        expect.append(("diag", order[u], u))
        if u + 1 < t:
            expect.append(("upd", order[u + 1], u))
        sr = u + D  # with D = 2 the only catch-up row at time u
        if sr < t:
            expect += [("upd", order[sr], s) for s in range(u + 1)]
    got = []
    for r in tasks:
        kind = "diag" if r[15] == pm.OP_TRSM_DIAG else "upd"
        key = (kind, r[3], r[5])
        if not got or got[-1] != key:
            got.append(key)
    assert got == expect
    assert len(tasks) == t * t + t * t * (t - 1) // 2


def test_trmm_contributions_nearest_first():
    """Reading R9 for TRMM (in place, bottom-up for left/lower): the contributions to
    B(kx, o) run nearest the diagonal first (q = kx-1, kx-2, ...), so the next step's
    diagonal multiply on row kx-1 waits only for the first contribution of each chain
    (the WAR on B(kx-1, o)), not for the whole step."""
    T, t = 4, 5
    N = T * t
    recs = xk.plan_dump(xk.make_call(routine=pm.DTRMM, side="L", uplo="L", transA="N", diag="N", m=N, n=N,
                                     alpha=1.0, A=A_ADDR, lda=N, C=C_ADDR, ldc=N, sync=True), uniform(1), tile=T)
    by_seq = {r[0]: r for r in recs}
    qs = {}
    for r in recs:
        if r[1] == pm.TASK and r[15] == pm.OP_GEMM:
            a = by_seq[r[14][0]]  # producer of the A tile read: H2D of A(kx, q)
            assert a[1] == pm.H2D and a[2] == 0 and a[3] == r[3]
            qs.setdefault((r[3], r[4]), []).append(a[4])
    assert len(qs) == t * (t - 1)
    for (kx, o), q in qs.items():
        assert q == list(range(kx - 1, -1, -1)), (kx, o, q)


def test_beta_deferral_syrk_symm():
    """Reading Q12'' extended to DSYRK/DSYR2K/DSYMM: off-diagonal SYRK tiles and SYMM tiles
    whose chain ends in a GEMM defer beta to the last task (shadow H2D of C, operand 2,
    version 0); SYRK diagonal tiles (reading R5) and SYMM chains ending in the symmetric
    diagonal op read C in place.  C still crosses PCIe once per tile."""
    T, t = 4, 3
    N = T * t
    for routine in (pm.DSYRK, pm.DSYR2K, pm.DSYMM):
        call = xk.make_call(routine=routine, uplo="L", transA="N", side="L", m=N, n=N, k=N, alpha=1.5,
                            beta=-0.75, A=A_ADDR, lda=N, B=B_ADDR, ldb=N, C=C_ADDR, ldc=N, sync=True)
        recs = xk.plan_dump(call, uniform(2), tile=T)
        by_seq = {r[0]: r for r in recs}
        chains = {}
        for r in recs:
            if r[1] == pm.TASK:
                chains.setdefault((r[3], r[4]), []).append(r)
        c_h2d = [r for r in recs if r[1] == pm.H2D and r[2] == 2]
        assert len(c_h2d) == len(chains)
        for (i, j), ch in chains.items():
            in_place = (i == j) if routine != pm.DSYMM else (i == t - 1)
            first, last = ch[0], ch[-1]
            if in_place:
                assert all(d == -1 for d in last[14][3:]) and first[14][2] >= 0
            else:
                assert first[14][2] == -1
                src = by_seq[last[14][3]]
                assert src[1] == pm.H2D and src[2] == 2 and (src[3], src[4]) == (i, j)


def test_coherent_writebacks_in_completion_order():
    """xk_memory_coherent_*: the D2H records of a view go out in the (virtual) completion order
    of their tiles, so the FIFO D2H stream never waits behind a tile whose chain ends late."""
    T, N = 4, 24
    for G in (1, 4):
        s = xk.PlanSession(uniform(G), topo="ranked", optimistic=True, tile=T)
        recs = s.call(xk.make_call(m=N, n=N, k=N, alpha=1.5, beta=-0.75, A=A_ADDR, lda=N, B=B_ADDR, ldb=N,
                                   C=C_ADDR, ldc=N, sync=False))
        by_seq = {r[0]: r for r in recs}
        wb = s.call(xk.make_call(routine=pm.COHERENT, m=N, n=N, C=C_ADDR, ldc=N))
        s.close()
        assert len(wb) == (N // T) ** 2 and all(r[1] == pm.D2H for r in wb)
        done = [by_seq[r[14][0]][12] for r in wb]
        assert done == sorted(done) and len(set(done)) > 1


@pytest.mark.parametrize("G", [1, 4, 8])
def test_trsm_window_depends_on_residency(G):
    """Reading R10 applies only when B must come from the host: with every B tile current on
    a GPU (prefetched = data-on-device, or produced by an earlier async call) the plan is the
    right-looking order; a partly resident B keeps the window.  Bit-exact vs the model in all
    three cases, for both triangles and sides."""
    bw = TOPOS["uniform"](G)
    flags = dict(topo="ranked", optimistic=True, window=2, tile=4)
    N = 24
    for side, uplo in itertools.product("LR", "LU"):
        trsm = dict(routine=pm.DTRSM, side=side, uplo=uplo, transA="N", diag="N", m=N, n=N, alpha=1.5,
                    A=A_ADDR, lda=N, C=B_ADDR, ldc=N, sync=False)
        for pre in (None, (N, N), (N // 2, N)):
            calls = []
            if pre:
                calls.append(dict(routine=pm.PREFETCH, m=pre[0], n=pre[1], C=B_ADDR, ldc=N))
            calls += [trsm, dict(routine=pm.COHERENT, m=N, n=N, C=B_ADDR, ldc=N), dict(routine=pm.SYNC)]
            got, exp = both(bw, flags, calls)
            assert got == exp, (G, side, uplo, pre)
    # on one GPU the resident case is plain right-looking: every update of step s comes
    # before the diagonal solve of step s+1 ... and the host-resident case is not
    if G == 1:
        def update_steps(recs):
            return [r[5] for r in recs if r[1] == pm.TASK]
        trsm = dict(routine=pm.DTRSM, side="L", uplo="L", transA="N", diag="N", m=N, n=N, alpha=1.5,
                    A=A_ADDR, lda=N, C=B_ADDR, ldc=N, sync=False)
        res, _ = both(bw, flags, [dict(routine=pm.PREFETCH, m=N, n=N, C=B_ADDR, ldc=N), trsm])
        host, _ = both(bw, flags, [trsm])
        assert update_steps(res[1]) == sorted(update_steps(res[1]))
        assert update_steps(host[0]) != sorted(update_steps(host[0]))


def test_invalidate_makes_host_authoritative():
    """xk_memory_invalidate drops the GPU copies and makes the host array the valid copy,
    even when the GPUs held the only current version (no coherence first): the next call
    reads the tiles from the host (H2D), never fails for want of a valid copy."""
    G = 4
    bw = TOPOS["uniform"](G)
    flags = dict(topo="ranked", optimistic=True, window=2, tile=4)
    calls = [gemm(m=12, n=12, k=12, C=D_ADDR, ldc=12, sync=False, beta=0.0),       # D only on GPUs
             dict(routine=pm.INVALIDATE, m=12, n=12, C=D_ADDR, ldc=12),          # dropped, host wins
             gemm(m=12, n=12, k=12, A=D_ADDR, lda=12, B=C_ADDR, ldb=12, C=E_ADDR, ldc=12, sync=True)]
    got, exp = both(bw, flags, calls)
    assert got == exp
    d_reads = [r for r in got[2] if r[1] == pm.H2D and r[2] == 0]
    assert len(d_reads) == 9  # every 4x4 tile of D (3 x 3 tiles) comes from the host


def test_trmm_shadow_sweep():
    """Reading R15: host-resident DTRMM reads B's input tiles from a per-call
    shadow and sweeps in the solve direction (top-down for left/lower, row 0 first), each
    B tile crossing PCIe once (the shadow's H2D; the output tile gets a device copy); the
    diagonal multiply of row kx needs only the shadow tiles of rows <= kx."""
    T, t = 4, 4
    N = T * t
    call = xk.make_call(routine=pm.DTRMM, side="L", uplo="L", transA="N", diag="N", m=N, n=N,
                        alpha=1.0, A=A_ADDR, lda=N, C=C_ADDR, ldc=N, sync=True)
    recs = xk.plan_dump(call, uniform(1), tile=T)
    by_seq = {r[0]: r for r in recs}
    diag = [r for r in recs if r[1] == pm.TASK and r[15] == pm.OP_TRMM_DIAG]
    assert [r[3] for r in diag] == sorted(r[3] for r in diag) and diag[0][3] == 0
    h2d_b = [(r[3], r[4]) for r in recs if r[1] == pm.H2D and r[2] == 2]
    assert sorted(h2d_b) == sorted(set(h2d_b)) and len(h2d_b) == t * t
    for r in diag:  # input 1 is the shadow tile's own H2D
        src = by_seq[r[14][1]]
        assert src[1] == pm.H2D and (src[3], src[4]) == (r[3], r[4])
    seen_rows = set()
    for r in recs:
        if r[1] == pm.H2D and r[2] == 2:
            seen_rows.add(r[3])
        if r[1] == pm.TASK and r[15] == pm.OP_TRMM_DIAG:
            assert seen_rows <= set(range(r[3] + 1)), (r[3], seen_rows)
    # G > 1: the same sweep; every shadow tile is read from the host at most once in every
    # source mode (later copies are forwarded), so no host read can follow the write-back of
    # the output tile that shares its host memory
    for G in (2, 4, 8):
        for mode, opt in (("ranked", True), ("ranked", False), ("home", False)):
            recs2 = xk.plan_dump(call, uniform(G), tile=T, topo=mode, optimistic=opt)
            diag2 = [r[3] for r in recs2 if r[1] == pm.TASK and r[15] == pm.OP_TRMM_DIAG]
            assert diag2[0] == 0 and sorted(diag2) == sorted(r for r in range(t) for _ in range(t))
            h2d = [(r[3], r[4]) for r in recs2 if r[1] == pm.H2D and r[2] == 2]
            assert sorted(h2d) == sorted(set(h2d)) and len(h2d) == t * t, (G, mode)
            d2h_seq = {(r[3], r[4]): r[0] for r in recs2 if r[1] == pm.D2H}
            h2d_seq = {(r[3], r[4]): r[0] for r in recs2 if r[1] == pm.H2D and r[2] == 2}
            assert all(h2d_seq[k] < d2h_seq[k] for k in d2h_seq)


@pytest.mark.parametrize("G", [1, 4])
@pytest.mark.parametrize("second", ["gemm", "trsm_then_gemm"])
def test_sync_call_keeps_gpu_dirty_inputs(G, second):
    """a synchronous call that reads a tile whose only current copy is on a
    GPU (an earlier async call's output) must not drop it: a later coherent_sync of that view
    writes every one of its tiles back, from the GPU that holds it.  Checked on the planner
    alone (not via the mirrored model): async D = A*B (or async X = TRSM), sync E = D*C,
    coherent(D) -> one D2H per tile of D, each after D's own last task."""
    T, t = 4, 3
    N = T * t
    s = xk.PlanSession(uniform(G), topo="ranked", optimistic=True, tile=T)
    if second == "gemm":
        first = s.call(xk.make_call(m=N, n=N, k=N, alpha=1.0, beta=0.0, A=A_ADDR, lda=N, B=B_ADDR,
                                    ldb=N, C=D_ADDR, ldc=N, sync=False))
    else:
        first = s.call(xk.make_call(routine=pm.DTRSM, side="L", uplo="L", transA="N", diag="N", m=N,
                                    n=N, alpha=1.0, A=A_ADDR, lda=N, C=D_ADDR, ldc=N, sync=False))
    last_task = {}
    for r in first:
        if r[1] == pm.TASK:
            last_task[(r[3], r[4])] = r[0]
    mid = s.call(xk.make_call(m=N, n=N, k=N, alpha=1.0, beta=0.0, A=D_ADDR, lda=N, B=C_ADDR, ldb=N,
                              C=E_ADDR, ldc=N, sync=True))
    assert not any(r[1] == pm.H2D and r[2] == 0 for r in mid)  # D read from the GPUs
    wb = s.call(xk.make_call(routine=pm.COHERENT, m=N, n=N, C=D_ADDR, ldc=N))
    d2h = [r for r in wb if r[1] == pm.D2H]
    assert sorted((r[3], r[4]) for r in d2h) == [(i, j) for i in range(t) for j in range(t)]
    for r in d2h:
        assert r[14][0] == -1 or r[14][0] == last_task[(r[3], r[4])]
    # a second coherent call has nothing left to write back; the next read of D is from
    # the host only if nothing on the GPUs is current any more (the GPU copies were kept)
    assert not [r for r in s.call(xk.make_call(routine=pm.COHERENT, m=N, n=N, C=D_ADDR, ldc=N))
                if r[1] == pm.D2H]
    s.close()
    # the mirrored model agrees record for record
    calls = [gemm(m=N, n=N, k=N, A=A_ADDR, lda=N, B=B_ADDR, ldb=N, C=D_ADDR, ldc=N, sync=False, beta=0.0),
             gemm(m=N, n=N, k=N, A=D_ADDR, lda=N, B=C_ADDR, ldb=N, C=E_ADDR, ldc=N, sync=True, beta=0.0),
             dict(routine=pm.COHERENT, m=N, n=N, C=D_ADDR, ldc=N)]
    got, exp = both(uniform(G), dict(topo="ranked", optimistic=True, window=2, tile=T), calls)
    assert got == exp


def _uses_shadow(routine, recs):
    if routine == "dtrmm":  # shadow sweep is top-down: row 0 multiplied first (R15)
        return next(r for r in recs if r[1] == pm.TASK and r[15] == pm.OP_TRMM_DIAG)[3] == 0
    # beta deferred: some chain's first task (tk = 0) does not read C (deps[2] == -1)
    return any(r[1] == pm.TASK and r[5] == 0 and r[15] == pm.OP_GEMM and r[14][2] == -1 for r in recs)


# per-GPU tiles of the shadow plan at G = 1, t = 4, written from the rule (DESIGN Q12'', R15):
# DGEMM A 16 + B 16 + C 16 + shadow 16; SYR2K (lower) A 16 + B 16 + C triangle 10 + shadow of
# the 6 off-diagonal tiles; SYMM (left, lower) A triangle 10 + B 16 + C 16 + shadow of the 12
# tiles whose chain ends in a GEMM (rows 0..2); TRMM A triangle 10 + B 16 + shadow 16
SHADOW_TILES_G1 = {"dgemm": 64, "dsyr2k": 48, "dsymm": 54, "dtrmm": 42}


@pytest.mark.parametrize("routine", ["dgemm", "dsyr2k", "dsymm", "dtrmm"])
@pytest.mark.parametrize("G", [1, 4])
def test_shadow_only_when_it_fits(routine, G):
    """a per-call shadow (beta deferral Q12'', TRMM R15) adds a second copy
    of C (B) to the device footprint.  With a capacity below footprint + shadow the call is
    planned without it; with room it keeps it.  G = 1: the threshold is the closed form above
    (tiles of T = 4 take 8*16*4 = 512 bytes).  G = 4: the planner's own threshold, where the
    model must agree record for record on both sides of it."""
    T, t = 4, 4
    N = T * t
    tile = 8 * 16 * T
    call = {"dgemm": gemm(m=N, n=N, k=N, lda=N, ldb=N, ldc=N),
            "dsyr2k": dict(routine=pm.DSYR2K, uplo="L", transA="N", n=N, k=N, alpha=1.5, beta=-0.75,
                           A=A_ADDR, lda=N, B=B_ADDR, ldb=N, C=C_ADDR, ldc=N, sync=True),
            "dsymm": dict(routine=pm.DSYMM, side="L", uplo="L", m=N, n=N, alpha=1.5, beta=-0.75,
                          A=A_ADDR, lda=N, B=B_ADDR, ldb=N, C=C_ADDR, ldc=N, sync=True),
            "dtrmm": dict(routine=pm.DTRMM, side="L", uplo="L", transA="N", diag="N", m=N, n=N,
                          alpha=1.5, A=A_ADDR, lda=N, C=C_ADDR, ldc=N, sync=True)}[routine]

    def plan(mem):
        return xk.plan_dump(xk.make_call(**call), uniform(G), tile=T, mem_bytes=mem)
    if G == 1:
        need = SHADOW_TILES_G1[routine] * tile
    else:
        lo, hi = 1, 1 << 30  # smallest capacity that keeps the shadow
        while lo < hi:
            mid = (lo + hi) // 2
            lo, hi = (lo, mid) if _uses_shadow(routine, plan(mid)) else (mid + 1, hi)
        need = lo
    assert _uses_shadow(routine, plan(0))  # unlimited
    for mem, expect in ((need, True), (need - 1, False)):
        got, exp = both(uniform(G), dict(topo="ranked", optimistic=True, window=2, tile=T,
                                         mem_bytes=mem), [call])
        assert got == exp
        assert _uses_shadow(routine, got[0]) == expect, (mem, need)


@pytest.mark.parametrize("grid,blk", [((2, 4), (1, 1)), ((4, 2), (1, 1)), ((2, 2), (2, 1)), ((1, 8), (1, 3))])
def test_distribute_2dbc(grid, blk):
    """xk_distribute_2dbc_async (SecIV-C): tile (bi, bj) lands on GPU
    ((bi/mb) mod P) Q + ((bj/nb) mod Q), one H2D per tile; a following async DGEMM reads no
    host tile (data on device), its operands forwarded between GPUs; bit-exact with the model."""
    G, T, t = 8, 4, 6
    N = T * t
    P, Q = grid
    mb, nb = blk
    calls = [dict(routine=pm.DISTRIBUTE, m=N, n=N, C=X, ldc=N, grid=grid, mb=mb, nb=nb) for X in (A_ADDR, B_ADDR, C_ADDR)]
    calls.append(gemm(m=N, n=N, k=N, lda=N, ldb=N, ldc=N, sync=False))
    calls.append(dict(routine=pm.COHERENT, m=N, n=N, C=C_ADDR, ldc=N))
    got, exp = both(uniform(G), dict(topo="ranked", optimistic=True, window=2, tile=T), calls)
    assert got == exp
    for recs in got[:3]:
        assert len(recs) == t * t and all(r[1] == pm.H2D for r in recs)
        for r in recs:
            assert r[7] == ((r[3] // mb) % P) * Q + (r[4] // nb) % Q
    assert not any(r[1] == pm.H2D for r in got[3])
    assert sum(1 for r in got[4] if r[1] == pm.D2H) == t * t


def test_distribute_rejects_bad_grid():
    s = xk.PlanSession(uniform(4), tile=4)
    with pytest.raises(xk.XKError):
        s.call(xk.make_call(routine=pm.DISTRIBUTE, m=8, n=8, C=A_ADDR, ldc=8, grid=(3, 2), mb=1, nb=1))
    with pytest.raises(xk.XKError):
        s.call(xk.make_call(routine=pm.DISTRIBUTE, m=8, n=8, C=A_ADDR, ldc=8, grid=(2, 2), mb=0, nb=1))
    s.close()
