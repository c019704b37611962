"""Closed-form transfer counts of every BLAS-3 plan, derived from the rules as DESIGN.md
states them -- not from tests/planmodel.py (the plan model mirrors the planner).

For a synchronous host-resident call the rules fix, per input tile, the set R of GPUs whose
tasks read it (the owner maps: 2D block-cyclic, R11 triangle round-robin, R12 snaked TRMM rows,
R13 TRSM/TRMM grid orientation).  Then:
  FULL (RANKED + optimistic): a tile valid only on the host crosses PCIe once and is forwarded
      to the other |R| - 1 requesters;
  HOME (host first): every requester reads a host-valid tile itself (|R| H2D, no P2P) --
      including a tile produced in the call once its final version has been written back
      (TRSM's solved rows); a read-once shadow (R15) is forwarded in every mode;
  D2H: every output tile once.
Counts are label-invariant, so only the sizes of the requester sets matter.  Checked against
the C++ planner for G in {1, 2, 4, 8} and tile counts t that do and do not divide evenly.
"""
import itertools

import pytest

import paper_conf_sc_gautierl21_b200 as xk
from tests import planmodel as pm  # record-kind constants only

A_ADDR, B_ADDR, C_ADDR = 0x10000000, 0x20000000, 0x30000000
GRIDS = {1: (1, 1), 2: (2, 1), 4: (2, 2), 8: (4, 2)}  # reading Q11


def links(G):
    bw = [[700000] * (G + 1) for _ in range(G + 1)]
    for g in range(G + 1):
        bw[g][G] = bw[G][g] = 55000
        bw[g][g] = 3000000
    return bw


def counts(call, G, T, mode):
    topo, opt = {"full": ("ranked", True), "home": ("home", True)}[mode]
    recs = xk.plan_dump(xk.make_call(**call), links(G), tile=T, topo=topo, optimistic=opt)
    c = {pm.H2D: 0, pm.P2P: 0, pm.D2H: 0}
    for r in recs:
        if r[1] in c:
            c[r[1]] += 1
    return c[pm.H2D], c[pm.P2P], c[pm.D2H]


# ---- owner maps restated from DESIGN.md
def block_cyclic(G):
    P, Q = GRIDS[G]
    return lambda i, j: (i % P, j % Q)


def tri_round_robin(G, t, lower=True):
    """R11: the stored triangle's tiles in column-major order dealt round-robin over G GPUs."""
    own, idx = {}, 0
    for j in range(t):
        for i in (range(j, t) if lower else range(0, j + 1)):
            own[(i, j)] = idx % G
            idx += 1
    return lambda i, j: own[(i, j)]


def trxm_owner(G, solve):
    """R13 (left side): grid rows = min(P, Q) along B's rows, columns = max(P, Q) along the
    untouched columns; R12 (TRMM only): the grid row index snakes 0..Pg-1, Pg-1..0, ..."""
    P, Q = GRIDS[G]
    Pg, Qg = min(P, Q), max(P, Q)

    def row(i):
        blk, r = divmod(i, Pg)
        return r if (solve or blk % 2 == 0) else Pg - 1 - r
    return lambda i, j: (row(i), j % Qg)


def transfer(sets, mode):
    """(H2D, P2P) for host-valid input tiles with requester sets `sets`."""
    if mode == "full":
        return len(sets), sum(len(s) - 1 for s in sets)
    return sum(len(s) for s in sets), 0


CASES = list(itertools.product([1, 2, 4, 8], [4, 5, 8], ["full", "home"]))


@pytest.mark.parametrize("G,t,mode", CASES)
@pytest.mark.parametrize("two", [False, True], ids=["syrk", "syr2k"])
@pytest.mark.parametrize("beta", [0.0, -0.75])
def test_syrk_syr2k(G, t, mode, two, beta):
    T, tk = 4, 3
    n, k = t * T, tk * T
    own = tri_round_robin(G, t)
    tiles = [(i, j) for j in range(t) for i in range(j, t)]
    # A(i, l) is op(A)_i for C tiles of row i (as the left factor) and column i (right factor)
    req = {i: {own(i, j) for j in range(i + 1)} | {own(r, i) for r in range(i, t)} for i in range(t)}
    sets = [req[i] for i in range(t) for _ in range(tk)] * (2 if two else 1)
    h2d, p2p = transfer(sets, mode)
    h2d += len(tiles) if beta else t  # C: the whole triangle, or only diagonal tiles (R5)
    call = dict(routine=pm.DSYR2K if two else pm.DSYRK, uplo="L", transA="N", n=n, k=k, alpha=1.5, beta=beta,
                A=A_ADDR, lda=n, B=B_ADDR, ldb=n, C=C_ADDR, ldc=n, sync=True)
    assert counts(call, G, T, mode) == (h2d, p2p, len(tiles))


@pytest.mark.parametrize("G,t,mode", CASES)
@pytest.mark.parametrize("beta", [0.0, -0.75])
def test_symm_left_lower(G, t, mode, beta):
    T, tn = 4, 3
    m, n = t * T, tn * T
    own = block_cyclic(G)
    # C(i, j) += sym(A)(i, l) B(l, j): stored A tile (r, q), r >= q, serves rows r and q of C
    a_sets = [{own(r, j) for j in range(tn)} | {own(q, j) for j in range(tn)}
              for q in range(t) for r in range(q, t)]
    b_sets = [{own(i, j) for i in range(t)} for l in range(t) for j in range(tn)]
    h2d, p2p = transfer(a_sets + b_sets, mode)
    h2d += t * tn if beta else 0
    call = dict(routine=pm.DSYMM, side="L", uplo="L", m=m, n=n, alpha=1.5, beta=beta, A=A_ADDR, lda=m,
                B=B_ADDR, ldb=m, C=C_ADDR, ldc=m, sync=True)
    assert counts(call, G, T, mode) == (h2d, p2p, t * tn)


@pytest.mark.parametrize("G,t,mode", CASES)
def test_trsm_left_lower(G, t, mode):
    T, tn = 4, 6
    m, n = t * T, tn * T
    own = trxm_owner(G, solve=True)
    # L(r, q), r >= q: the diagonal solve (q = r) and the updates of B's row r -> row r's owners
    l_sets = [{own(r, o) for o in range(tn)} for q in range(t) for r in range(q, t)]
    h2d, p2p = transfer(l_sets, mode)
    h2d += t * tn  # B's input tiles: read by their owners only
    # solved B(k, o) (GPU-produced) feeds the updates of B(r, o), r > k, on their owners.  It
    # is final once solved, so the synchronous call writes it back at once (D2H after its last
    # writer): FULL forwards it from its GPU, HOME (host first) re-reads the written-back copy
    solved = sum(len({own(r, o) for r in range(k + 1, t)} - {own(k, o)}) for k in range(t) for o in range(tn))
    if mode == "full":
        p2p += solved
    else:
        h2d += solved
    call = dict(routine=pm.DTRSM, side="L", uplo="L", transA="N", diag="N", m=m, n=n, alpha=1.5,
                A=A_ADDR, lda=m, C=C_ADDR, ldc=m, sync=True)
    assert counts(call, G, T, mode) == (h2d, p2p, t * tn)


@pytest.mark.parametrize("G,t,mode", CASES)
def test_trmm_left_lower(G, t, mode):
    T, tn = 4, 6
    m, n = t * T, tn * T
    own = trxm_owner(G, solve=False)
    l_sets = [{own(r, o) for o in range(tn)} for q in range(t) for r in range(q, t)]
    h2d, p2p = transfer(l_sets, mode)
    # R15 shadow of B, read from the host once per tile in every mode: shadow(q, o) feeds the
    # diagonal multiply of B(q, o) and the contributions to B(kx, o), kx > q
    sh = [{own(kx, o) for kx in range(q, t)} for q in range(t) for o in range(tn)]
    h2d += len(sh)
    p2p += sum(len(s) - 1 for s in sh)
    call = dict(routine=pm.DTRMM, side="L", uplo="L", transA="N", diag="N", m=m, n=n, alpha=1.5,
                A=A_ADDR, lda=m, C=C_ADDR, ldc=m, sync=True)
    assert counts(call, G, T, mode) == (h2d, p2p, t * tn)


@pytest.mark.parametrize("G", [2, 4, 8])
def test_owner_maps_task_balance(G):
    """R11-R13 restated: per-GPU task counts of the plans equal the counts the DESIGN formulas
    give, and their max/mean is what DESIGN.md quotes (triangle round-robin balances SYRK's
    C tiles to within one tile; TRMM's snaked rows balance its contributions)."""
    T, t = 4, 16
    N = t * T
    def per_gpu_tasks(call):
        recs = xk.plan_dump(xk.make_call(**call), links(G), tile=T)
        out = [0] * G
        for r in recs:
            if r[1] == pm.TASK:
                out[r[7]] += 1
        return out
    # SYRK (lower, N, k = N): tile (i, j) of the triangle has t_k tasks on owner_tri(i, j)
    got = per_gpu_tasks(dict(routine=pm.DSYRK, uplo="L", transA="N", n=N, k=N, alpha=1.5, beta=-0.75,
                             A=A_ADDR, lda=N, C=C_ADDR, ldc=N, sync=True))
    own = tri_round_robin(G, t)
    exp = [0] * G
    for j in range(t):
        for i in range(j, t):
            exp[own(i, j)] += t
    assert sorted(got) == sorted(exp)
    assert max(got) * G <= 1.0 * sum(got) + G * t  # within one tile's chain of the mean
    # TRMM (left, lower): B(kx, o) gets 1 diagonal multiply + kx contributions on its owner
    got = per_gpu_tasks(dict(routine=pm.DTRMM, side="L", uplo="L", transA="N", diag="N", m=N, n=N,
                             alpha=1.5, A=A_ADDR, lda=N, C=C_ADDR, ldc=N, sync=True))
    own = trxm_owner(G, solve=False)
    cells = sorted({own(i, j) for i in range(t) for j in range(t)})
    exp = {c: 0 for c in cells}
    for i in range(t):
        for j in range(t):
            exp[own(i, j)] += 1 + i
    assert sorted(got) == sorted(exp.values())
    assert max(got) * G == sum(got)  # snaked rows: exact balance when 2 Pg | t (DESIGN R12)
