"""CPU model of the two XKBlas heuristics -- the plan oracle (SURVEY.md §8(c) "Plan oracle").

Independent of the C++ planner (shares no code): a plain Python walk of the algorithm in
the order SURVEY.md §8(c) lists it, with the readings of DESIGN.md §Readings:

  1. link classes from the measured (G+1)^2 matrix (gap ratio > 1.25),
  2. per-GPU k-major task lists, k-shifted anti-diagonal order ((i+j+k) mod t, i, j),
  3. event loop on the smallest request time (end of the task W positions earlier),
  4. source selection: RANKED = topology-aware + optimistic in-flight
     source; UNRANKED = paper's "no topo"; HOME = host first,
  5. store-and-forward copy timing on per-link occupancy, integer ns,
  6. task timing and output versioning, 7. D2H after the last writer (sync calls),
  8. session rule (directory/clocks persist across async calls, reset at sync),
  9. tiles keyed in stored-matrix coordinates, 10. partial coherence.

Produces record tuples in the field order of xk_plan_rec_t:
(seq, kind, operand, bi, bj, tk, version, dst, src, src_state, depth, t_start, t_end, work, deps)
"""
H2D, P2P, TASK, D2H = 0, 1, 2, 3
S_NONE, S_VALID, S_INFLIGHT, S_HOST = 0, 1, 2, 3
RANKED, UNRANKED, HOME = 0, 1, 2
HOSTID = -1
DGEMM, DSYRK, DSYR2K, DSYMM, DTRMM, DTRSM = 0, 1, 2, 3, 4, 5
COHERENT, SYNC, INVALIDATE, PREFETCH, DISTRIBUTE = 100, 101, 102, 103, 104
OP_GEMM, OP_SCALE, OP_GEMM_TRI, OP_SYMM_DIAG, OP_TRMM_DIAG, OP_TRSM_DIAG = 0, 1, 2, 3, 4, 5


def ceil_div(a, b):
    return -(-a // b)


def classes(bw):
    n = len(bw)
    vals = sorted({bw[s][d] for s in range(n) for d in range(n) if s != d})
    cls_of, c = {}, 0
    for idx, v in enumerate(vals):
        if idx and v * 4 > vals[idx - 1] * 5:
            c += 1
        cls_of[v] = c
    return [[cls_of[bw[s][d]] if s != d else None for d in range(n)] for s in range(n)]


def near_square(G):
    q = max(c for c in range(1, G + 1) if G % c == 0 and c * c <= G)
    return G // q, q


def min_max_quotas(G, sets, count, forced):
    """R16: split count[i] tiles of requester set sets[i] over its members minimising the
    largest forced[g] + assigned[g]: binary search on that maximum, feasibility by max-flow
    (Edmonds-Karp, BFS in node order: source, sets, GPUs, sink).  Returns the flows set -> GPU."""
    nS = len(sets)
    V, src, snk = nS + G + 2, 0, nS + G + 1
    total = sum(count)

    def run(L):
        cap = [[0] * V for _ in range(V)]
        flow = [[0] * V for _ in range(V)]
        for i, S in enumerate(sets):
            cap[src][1 + i] = count[i]
            for g in S:
                cap[1 + i][1 + nS + g] = total
        for g in range(G):
            cap[1 + nS + g][snk] = max(0, L - forced[g])
        got = 0
        while True:
            par = [-1] * V
            par[src] = src
            q = [src]
            h = 0
            while h < len(q) and par[snk] < 0:
                u = q[h]
                h += 1
                for v in range(V):
                    if par[v] < 0 and cap[u][v] - flow[u][v] > 0:
                        par[v] = u
                        q.append(v)
            if par[snk] < 0:
                break
            b, v = None, snk
            while v != src:
                r = cap[par[v]][v] - flow[par[v]][v]
                b = r if b is None else min(b, r)
                v = par[v]
            v = snk
            while v != src:
                flow[par[v]][v] += b
                flow[v][par[v]] -= b
                v = par[v]
            got += b
        return got == total, flow
    lo, hi = max(max(forced), -(-(total + sum(forced)) // G)), max(forced) + total
    while lo < hi:
        mid = (lo + hi) // 2
        if run(mid)[0]:
            hi = mid
        else:
            lo = mid + 1
    flow = run(lo)[1]
    return [[max(0, flow[1 + i][1 + nS + g]) for g in range(G)] for i in range(nS)]


class Copy:
    __slots__ = ("ver", "t_done", "producer", "depth")

    def __init__(self, ver, t_done, producer, depth):
        self.ver, self.t_done, self.producer, self.depth = ver, t_done, producer, depth


class Tile:
    def __init__(self, rows, cols, bi, bj):
        self.rows, self.cols, self.bi, self.bj = rows, cols, bi, bj
        self.ver = 0
        self.host = Copy(0, 0, -1, 0)  # inputs start valid on the host
        self.gpus = {}  # g -> Copy
        self.once = False  # R15: read-once shadow


class Model:
    def __init__(self, bw, rate_mflops=35000000, topo="ranked", optimistic=True, window=4,
                 grid=(0, 0), tile=2048, mem_bytes=0):
        self.bw = [list(r) for r in bw]
        self.G = len(bw) - 1
        self.once = set()  # read-once shadow bases (R15)
        self.cls = classes(self.bw)
        self.rate = rate_mflops
        self.mode = {"ranked": RANKED, "unranked": UNRANKED, "home": HOME}[topo] if isinstance(topo, str) else topo
        self.opt = bool(optimistic)
        self.W = max(1, window)
        self.P, self.Q = grid if grid[0] > 0 else near_square(self.G)
        self.T = tile
        self.mem = mem_bytes      # per-GPU tile-cache capacity (0 = unlimited)
        self._no_shadow = False
        self.tiles = {}          # (base, ld, bi, bj) -> Tile
        self.extent = {}         # (base, ld) -> [rows, cols]
        self.link = {}           # (src_idx, dst_idx) -> free time
        self.gfree = [0] * self.G
        self.hist = [[] for _ in range(self.G)]
        self.seq = 0
        self.calls = 0

    # ------------------------------------------------------------------ helpers
    def owner(self, i, j):
        return (i % self.P) * self.Q + (j % self.Q)

    def tile(self, base, ld, bi, bj):
        key = (base, ld, bi, bj)
        if key not in self.tiles:
            rows, cols = self.extent[(base, ld)]
            self.tiles[key] = Tile(min(self.T, rows - bi * self.T), min(self.T, cols - bj * self.T), bi, bj)
            self.tiles[key].once = base in self.once
        return self.tiles[key]

    def matrix(self, base, ld, rows, cols):
        e = self.extent.get((base, ld))
        self.extent[(base, ld)] = [max(e[0], rows), max(e[1], cols)] if e else [rows, cols]

    def nsec(self, amount, rate):
        return ceil_div(amount * 1000, rate)

    def idx(self, node):
        return self.G if node == HOSTID else node

    def choose(self, t, ver, d, treq):
        valid, infl = [], []
        for g in range(self.G):
            c = t.gpus.get(g)
            if g == d or c is None or c.ver != ver:
                continue
            (valid if c.t_done <= treq else infl).append(g)
        host_ok = t.host is not None and t.host.ver == ver
        if self.mode == HOME:
            if host_ok:
                return HOSTID, S_HOST
            if valid:
                return valid[0], S_VALID
            if infl:
                return infl[0], S_INFLIGHT
            raise RuntimeError("no source")

        def best(cands):
            if self.mode == UNRANKED:
                return cands[0]
            return min(cands, key=lambda g: (-self.cls[g][d], t.gpus[g].depth, (g - d) % self.G))
        if valid:
            return best(valid), S_VALID
        if infl and (self.opt or not host_ok):
            return best(infl), S_INFLIGHT
        if host_ok:
            return HOSTID, S_HOST
        raise RuntimeError("no source")

    def copy_in(self, t, ver, d, treq, operand, out):
        src, state = self.choose(t, ver, d, treq)
        nbytes = 8 * t.rows * t.cols
        if src == HOSTID:
            ready, dep, depth = t.host.t_done, t.host.producer, 1
        else:
            c = t.gpus[src]
            ready, dep, depth = c.t_done, c.producer, c.depth + 1
        lk = (self.idx(src), d)
        start = max(treq, ready, self.link.get(lk, 0))
        end = start + self.nsec(nbytes, self.bw[self.idx(src)][d])
        self.link[lk] = end
        out.append((self.seq, H2D if src == HOSTID else P2P, operand, t.bi, t.bj, -1, ver, d, src,
                    state, depth, start, end, nbytes, (dep, -1, -1, -1), -1))
        t.gpus[d] = Copy(ver, end, self.seq, depth)
        self.seq += 1
        if src == HOSTID and t.once:  # R15: later copies are forwarded from GPUs
            t.host = None

    def copy_out(self, t, src, sub, ready, dep, out):
        r0, c0, rows, cols = sub
        nbytes = 8 * rows * cols
        lk = (src, self.G)
        start = max(ready, self.link.get(lk, 0))
        end = start + self.nsec(nbytes, self.bw[src][self.G])
        self.link[lk] = end
        out.append((self.seq, D2H, 2, t.bi, t.bj, -1, t.ver, HOSTID, src, S_VALID, 0, start, end,
                    nbytes, (dep, -1, -1, -1), -1))
        if (r0, c0, rows, cols) == (0, 0, t.rows, t.cols):
            t.host = Copy(t.ver, end, self.seq, 0)
        self.seq += 1

    # ------------------------------------------------------------------ calls
    def call(self, routine=DGEMM, transA="N", transB="N", m=0, n=0, k=0, alpha=1.0, beta=0.0,
             A=0, lda=1, B=0, ldb=1, C=0, ldc=1, sync=False, uplo="L", side="L", diag="N",
             grid=(0, 0), mb=0, nb=0):
        out = []
        ta, tb = transA.upper() in "TC", transB.upper() in "TC"
        lower, left = uplo.upper() == "L", side.upper() == "L"
        if routine in (DGEMM, DSYRK, DSYR2K, DSYMM, DTRMM, DTRSM):
            def gen():
                if routine == DGEMM:
                    return self.gen_gemm(ta, tb, m, n, k, alpha, beta, A, lda, B, ldb, C, ldc)
                if routine in (DSYRK, DSYR2K):
                    return self.gen_syrk(routine == DSYR2K, lower, ta, n, k, alpha, beta, A, lda, B, ldb, C, ldc)
                if routine == DSYMM:
                    return self.gen_symm(left, lower, m, n, alpha, beta, A, lda, B, ldb, C, ldc)
                return self.gen_trxm(routine == DTRSM, left, lower, ta, diag.upper(), m, n, alpha, A, lda, C, ldc)
            self._shadow = None
            tasks = gen()
            if tasks and self._shadow is not None and not self.fits(tasks):
                # the shadow does not fit next to the call's tiles: plan without it
                self.drop_shadow(ldc)
                self._no_shadow = True
                tasks = gen()
                self._no_shadow = False
            if tasks:
                self.run(tasks, sync, out)
            if routine in (DGEMM, DSYRK, DSYR2K, DSYMM, DTRMM):
                self.drop_shadow(ldc)
            if sync and tasks is not None:
                self.full_sync()
                if routine == DGEMM:
                    if alpha != 0 and k > 0:
                        self.release(A, (k, m) if ta else (m, k), lda)
                        self.release(B, (n, k) if tb else (k, n), ldb)
                    self.release(C, (m, n), ldc)
                elif routine in (DSYRK, DSYR2K):
                    if alpha != 0 and k > 0:
                        self.release(A, (k, n) if ta else (n, k), lda)
                        if routine == DSYR2K:
                            self.release(B, (k, n) if ta else (n, k), ldb)
                    self.release(C, (n, n), ldc)
                elif routine == DSYMM:
                    if alpha != 0:
                        ka = m if left else n
                        self.release(A, (ka, ka), lda)
                        self.release(B, (m, n), ldb)
                    self.release(C, (m, n), ldc)
                else:
                    ka = m if left else n
                    if alpha != 0:
                        self.release(A, (ka, ka), lda)
                    self.release(C, (m, n), ldc)
        elif routine == COHERENT:
            self.coherent(C, m, n, ldc, out)
        elif routine == SYNC:
            self.full_sync()
        elif routine == INVALIDATE:
            self.invalidate(C, (m, n), ldc)
        elif routine == PREFETCH:
            self.prefetch(C, m, n, ldc, out)
        elif routine == DISTRIBUTE:
            P, Q = grid
            self.prefetch(C, m, n, ldc, out, owner=lambda bi, bj: ((bi // mb) % P) * Q + (bj // nb) % Q)
        return out

    # ---- task generators: program order, symbolic versions (readings in DESIGN.md)
    def owner_trxm(self, i, j, left, solve):
        """TRSM/TRMM's B (R13, R12): the grid's larger extent along the untouched
        dimension; TRMM snakes the grid index along the triangular dimension."""
        def snake(x, n):
            blk, r = divmod(x, n)
            return r if blk % 2 == 0 else n - 1 - r
        lo, hi = min(self.P, self.Q), max(self.P, self.Q)
        Pg, Qg = (lo, hi) if left else (hi, lo)
        pi = snake(i, Pg) if (not solve and left) else i % Pg
        qj = snake(j, Qg) if (not solve and not left) else j % Qg
        return pi * Qg + qj

    def owner_tri(self, i, j, lower, t):
        """Triangular outputs (SYRK/SYR2K, R11): the stored triangle's tiles in
        column-major order, dealt round-robin over the GPUs."""
        idx = j * t - j * (j - 1) // 2 + (i - j) if lower else j * (j + 1) // 2 + i
        return idx % self.G

    def _task(self, vers, op, i, j, out, ins, skey, flops, tk, gpu=None):
        """ins = [(tile, operand)] in input order; versions read now, output bumped."""
        t = dict(gpu=self.owner(i, j) if gpu is None else gpu, op=op, out=out, tk=tk, i=i, j=j, flops=flops, skey=skey,
                 ins=[(tl, vers.get(id(tl), tl.ver), opnd) for (tl, opnd) in ins])
        vers[id(out)] = vers.get(id(out), out.ver) + 1
        t["ver"] = vers[id(out)]
        return t

    def gen_gemm(self, ta, tb, m, n, k, alpha, beta, A, lda, B, ldb, C, ldc):
        if m == 0 or n == 0 or ((alpha == 0 or k == 0) and beta == 1):
            return None
        T = self.T
        scale = alpha == 0 or k == 0
        self.matrix(C, ldc, m, n)
        if not scale:
            self.matrix(A, lda, *((k, m) if ta else (m, k)))
            self.matrix(B, ldb, *((n, k) if tb else (k, n)))
        tm, tn = ceil_div(m, T), ceil_div(n, T)
        tk = 0 if scale else ceil_div(k, T)
        tmod = max(1, tm, tn)
        # beta deferral (Q12''): a per-call shadow of C's input tiles feeds the last
        # task of each chain whose C input is valid on the host
        shadow = self.new_shadow(C, ldc) if (not scale and beta != 0 and tk >= 2) else None
        vers, tasks = {}, []
        for j in range(tn):
            for i in range(tm):
                ct = self.tile(C, ldc, i, j)
                mt, nt = min(T, m - i * T), min(T, n - j * T)
                if scale:
                    ins = [(ct, 2)] if beta != 0 else []
                    tasks.append(self._task(vers, OP_SCALE, i, j, ct, ins, (0, (i + j) % tmod, i, j, 0), mt * nt, -1))
                    continue
                defer = shadow is not None and self.host_only(ct)
                st = self.tile(shadow, ldc, i, j) if defer else None
                for kk in range(tk):
                    kt = min(T, k - kk * T)
                    at = self.tile(A, lda, kk, i) if ta else self.tile(A, lda, i, kk)
                    bt = self.tile(B, ldb, j, kk) if tb else self.tile(B, ldb, kk, j)
                    ins = [(at, 0), (bt, 1)] + ([(ct, 2)] if (kk > 0 or (beta != 0 and not defer)) else [])
                    if defer and kk == tk - 1:
                        ins.append((st, 2))
                    tasks.append(self._task(vers, OP_GEMM, i, j, ct, ins, (kk + (i + j) % tk, (i + j + kk) % tmod, i, j, 0),
                                            2 * mt * nt * kt, kk))
        self._shadow = shadow
        return tasks

    def fits(self, tasks):
        """Capacity rule of a shadow plan: on every GPU, the tiles resident now plus the
        tiles its tasks read or write, at 8 * round_up(rows, 16) * cols bytes each, fit."""
        if self.mem <= 0:
            return True
        sets = [dict() for _ in range(self.G)]
        for t in self.tiles.values():
            for g in t.gpus:
                sets[g][id(t)] = t
        for t in tasks:
            for tl in [t["out"]] + [x[0] for x in t["ins"]]:
                sets[t["gpu"]][id(tl)] = tl
        return all(sum(8 * ceil_div(tl.rows, 16) * 16 * tl.cols for tl in s.values()) <= self.mem
                   for s in sets)

    def new_shadow(self, C, ldc):
        if self._no_shadow:
            return None
        self.calls += 1
        shadow = ("shadow", self.calls, C)
        self.extent[(shadow, ldc)] = list(self.extent[(C, ldc)])
        self._shadow = shadow
        return shadow

    @staticmethod
    def host_only(ct):
        return (ct.host is not None and ct.host.ver == ct.ver
                and not any(g.ver == ct.ver for g in ct.gpus.values()))

    def drop_shadow(self, ldc):
        sh = getattr(self, "_shadow", None)
        if sh is None:
            return
        for key in [key for key in self.tiles if key[0] == sh]:
            del self.tiles[key]
        del self.extent[(sh, ldc)]
        self._shadow = None

    def gen_syrk(self, two, lower, tr, n, k, alpha, beta, A, lda, B, ldb, C, ldc):
        if n == 0 or ((alpha == 0 or k == 0) and beta == 1):
            return None
        T = self.T
        scale = alpha == 0 or k == 0
        self.matrix(C, ldc, n, n)
        if not scale:
            self.matrix(A, lda, *((k, n) if tr else (n, k)))
            if two:
                self.matrix(B, ldb, *((k, n) if tr else (n, k)))
        tn = ceil_div(n, T)
        tk = 0 if scale else ceil_div(k, T)
        tmod = max(1, tn)
        nchain = tk * (2 if two else 1)
        shadow = self.new_shadow(C, ldc) if (not scale and beta != 0 and nchain >= 2) else None
        vers, tasks = {}, []

        def opnd(X, ld, r, l):
            return self.tile(X, ld, l, r) if tr else self.tile(X, ld, r, l)
        for j in range(tn):
            for i in range(tn):
                if (i < j) if lower else (i > j):
                    continue
                dg = i == j
                ct = self.tile(C, ldc, i, j)
                mt, nt = min(T, n - i * T), min(T, n - j * T)
                if scale:
                    ins = [(ct, 2)] if (beta != 0 or dg) else []
                    tasks.append(self._task(vers, OP_SCALE, i, j, ct, ins, (0, (i + j) % tmod, i, j, 0), mt * nt, -1,
                                            gpu=self.owner_tri(i, j, lower, tn)))
                    continue
                first = True
                defer = shadow is not None and not dg and self.host_only(ct)  # diagonal: R5
                pos = 0
                for l in range(tk):
                    kt = min(T, k - l * T)
                    for s in range(2 if two else 1):
                        xa = (B, ldb, 1) if (two and s == 1) else (A, lda, 0)
                        xb = (B, ldb, 1) if (two and s == 0) else (A, lda, 0)
                        at, bt = opnd(xa[0], xa[1], i, l), opnd(xb[0], xb[1], j, l)
                        ins = [(at, xa[2]), (bt, xb[2])] + (
                            [(ct, 2)] if (not first or (beta != 0 and not defer) or dg) else [])
                        if defer and pos == nchain - 1:
                            ins.append((self.tile(shadow, ldc, i, j), 2))
                        fl = kt * nt * (nt + 1) if dg else 2 * mt * nt * kt
                        tasks.append(self._task(vers, OP_GEMM_TRI if dg else OP_GEMM, i, j, ct, ins,
                                                (2 * (l + (i + j) % tk) + s, (i + j + l) % tmod, i, j, 0), fl, l,
                                                gpu=self.owner_tri(i, j, lower, tn)))
                        first = False
                        pos += 1
        return tasks

    def gen_symm(self, left, lower, m, n, alpha, beta, A, lda, B, ldb, C, ldc):
        if m == 0 or n == 0 or (alpha == 0 and beta == 1):
            return None
        T = self.T
        scale = alpha == 0
        ka = m if left else n
        self.matrix(C, ldc, m, n)
        if not scale:
            self.matrix(A, lda, ka, ka)
            self.matrix(B, ldb, m, n)
        tm, tn, tl = ceil_div(m, T), ceil_div(n, T), ceil_div(ka, T)
        tmod = max(1, tm, tn)
        shadow = self.new_shadow(C, ldc) if (not scale and beta != 0 and tl >= 2) else None
        vers, tasks = {}, []
        for j in range(tn):
            for i in range(tm):
                ct = self.tile(C, ldc, i, j)
                mt, nt = min(T, m - i * T), min(T, n - j * T)
                if scale:
                    ins = [(ct, 2)] if beta != 0 else []
                    tasks.append(self._task(vers, OP_SCALE, i, j, ct, ins, (0, (i + j) % tmod, i, j, 0), mt * nt, -1))
                    continue
                last_diag = (i == tl - 1) if left else (j == tl - 1)  # SYMM_DIAG reads C in place
                defer = shadow is not None and not last_diag and self.host_only(ct)
                for l in range(tl):
                    kt = min(T, ka - l * T)
                    r, q = (i, l) if left else (l, j)
                    in_tri = (r >= q) if lower else (r <= q)
                    at = self.tile(A, lda, r, q) if in_tri else self.tile(A, lda, q, r)
                    bt = self.tile(B, ldb, l, j) if left else self.tile(B, ldb, i, l)
                    if r == q or left:
                        ins = [(at, 0), (bt, 1)]
                    else:
                        ins = [(bt, 1), (at, 0)]
                    if l > 0 or (beta != 0 and not defer):
                        ins.append((ct, 2))
                    if defer and l == tl - 1:
                        ins.append((self.tile(shadow, ldc, i, j), 2))
                    tasks.append(self._task(vers, OP_SYMM_DIAG if r == q else OP_GEMM, i, j, ct, ins,
                                            (l + (i + j) % tl, (i + j + l) % tmod, i, j, 0), 2 * mt * nt * kt, l))
        return tasks

    def gen_trxm(self, solve, left, lower, tr, diag, m, n, alpha, A, lda, C, ldc):
        if m == 0 or n == 0:
            return None
        T = self.T
        ka = m if left else n
        elow = lower != tr
        self.matrix(C, ldc, m, n)
        tm, tn, tk = ceil_div(m, T), ceil_div(n, T), ceil_div(ka, T)
        tmod = max(1, tm, tn)
        vers, tasks = {}, []
        if alpha == 0:
            for j in range(tn):
                for i in range(tm):
                    ct = self.tile(C, ldc, i, j)
                    mt, nt = min(T, m - i * T), min(T, n - j * T)
                    tasks.append(self._task(vers, OP_SCALE, i, j, ct, [], (0, (i + j) % tmod, i, j, 0), mt * nt, -1,
                                            gpu=self.owner_trxm(i, j, left, solve)))
            return tasks
        self.matrix(A, lda, ka, ka)

        def opA(r, q):
            return self.tile(A, lda, q, r) if tr else self.tile(A, lda, r, q)
        fwd = (left == elow) if solve else (left != elow)
        other = tn if left else tm
        # R10 window only when B must come from the host (some tile not current on a GPU)
        b_on_gpus = all(any(c.ver == tl.ver for c in tl.gpus.values())
                        for tl in (self.tile(C, ldc, i, j) for j in range(tn) for i in range(tm)))
        D = tk if b_on_gpus else 2 * (min(self.P, self.Q) if left else max(self.P, self.Q))
        # R15: TRMM from the host reads B's input tiles from a per-call shadow and
        # sweeps in the solve direction; the diagonal multiply starts from the shadow tile
        shadow = None
        if (not solve and tk >= 2
                and all(self.host_only(self.tile(C, ldc, i, j)) for j in range(tn) for i in range(tm))):
            shadow = self.new_shadow(C, ldc)
            if shadow is not None:
                self.once.add(shadow)  # read from the host at most once per tile
        Bin = shadow if shadow is not None else C
        sweep_fwd = (not fwd) if shadow is not None else fwd
        for s in range(tk):
            kx = s if sweep_fwd else tk - 1 - s
            for o in range(other):
                bi, bj = (kx, o) if left else (o, kx)
                ot = self.tile(C, ldc, bi, bj)
                mt, nt = min(T, m - bi * T), min(T, n - bj * T)
                fl = mt * mt * nt if left else mt * nt * nt
                src = self.tile(shadow, ldc, bi, bj) if shadow is not None else ot
                tasks.append(self._task(vers, OP_TRSM_DIAG if solve else OP_TRMM_DIAG, bi, bj, ot,
                                        [(opA(kx, kx), 0), (src, 2)], (s, 0, (bi + bj + s) % tmod, bi, bj), fl, s,
                                        gpu=self.owner_trxm(bi, bj, left, solve)))
                if not solve:
                    ph = 1
                    # contributions nearest the diagonal first (R9)
                    below = elow if left else not elow
                    qs = range(kx - 1, -1, -1) if below else range(kx + 1, tk)
                    for q in qs:
                        kt = min(T, ka - q * T)
                        if left:
                            ins = [(opA(kx, q), 0), (self.tile(Bin, ldc, q, bj), 2), (ot, 2)]
                        else:
                            ins = [(self.tile(Bin, ldc, bi, q), 2), (opA(q, kx), 0), (ot, 2)]
                        tasks.append(self._task(vers, OP_GEMM, bi, bj, ot, ins,
                                                (s, ph, (bi + bj + s) % tmod, bi, bj), 2 * mt * nt * kt, s,
                                                gpu=self.owner_trxm(bi, bj, left, solve)))
                        ph += 1
            if not solve:
                continue
            for r in range(tk):
                if not (r > kx if fwd else r < kx):
                    continue
                for o in range(other):
                    bi, bj = (r, o) if left else (o, r)
                    ot = self.tile(C, ldc, bi, bj)
                    mt, nt = min(T, m - bi * T), min(T, n - bj * T)
                    kt = min(T, ka - kx * T)
                    if left:
                        ins = [(opA(r, kx), 0), (self.tile(C, ldc, kx, bj), 2), (ot, 2)]
                    else:
                        ins = [(self.tile(C, ldc, bi, kx), 2), (opA(kx, r), 0), (ot, 2)]
                    # lookahead (R9): the next step's row (column) is updated first;
                    # update window (R10): row solved at step sr is updated by step s at time
                    # u = max(s, sr - D), D = 2 x grid extent along the solved dimension
                    sr = r if fwd else tk - 1 - r
                    u = max(s, sr - D)
                    ph = 1 if sr == s + 1 else 2
                    tasks.append(self._task(vers, OP_GEMM, bi, bj, ot, ins, (u, ph, sr * tk + s, (bi + bj + s) % tmod, o),
                                            2 * mt * nt * kt, s, gpu=self.owner_trxm(bi, bj, left, solve)))
        return tasks

    def run(self, tasks, sync, out):
        pending = {}
        last = {}
        for t in tasks:
            for (tl, v, _) in t["ins"]:
                pending[(id(tl), v)] = pending.get((id(tl), v), 0) + 1
            o = id(t["out"])
            if o not in last or last[o]["ver"] < t["ver"]:
                last[o] = t
        for t in last.values():
            t["last"] = True
        # R16 balance-aware first host pull (FULL mode): who carries each host-only input
        puller, lazy = {}, {}
        if self.opt and self.mode != HOME and self.G > 1:
            req, order = {}, []
            for t in tasks:
                for (tl, v, _) in t["ins"]:
                    key = (id(tl), v)
                    if key not in req:
                        req[key] = (tl, v, set())
                        order.append(key)
                    req[key][2].add(t["gpu"])
            forced = [0] * self.G
            sets, count = [], {}
            shared = []
            for key in order:
                tl, v, gs = req[key]
                if not (tl.ver == v and tl.host is not None and tl.host.ver == v
                        and not any(c.ver == v for c in tl.gpus.values())):
                    continue
                if len(gs) == 1:
                    (g,) = gs
                    puller[key] = g
                    forced[g] += 1
                    continue
                fs = frozenset(gs)
                if fs not in count:
                    sets.append(fs)
                    count[fs] = 0
                count[fs] += 1
                shared.append(key)
            if sets:
                quota = min_max_quotas(self.G, sets, [count[s] for s in sets], forced)
                for key in shared:
                    lazy[key] = quota[sets.index(frozenset(req[key][2]))]

        def designate(key, d):
            """At the first request: the requester while its quota in the set lasts, else the
            member with the most quota left (ties: lowest id)."""
            q = lazy.pop(key)
            if q[d] > 0:
                q[d] -= 1
                return d
            best = max((g for g in range(self.G) if q[g] > 0), key=lambda g: (q[g], -g))
            q[best] -= 1
            return best
        lists = [[] for _ in range(self.G)]
        for t in tasks:
            lists[t["gpu"]].append(t)
        for d in range(self.G):
            lists[d].sort(key=lambda t: t["skey"])
        pos = [0] * self.G

        def ready(t):
            if any(tl.ver != v for (tl, v, _) in t["ins"]):
                return False
            o = t["out"]
            if o.ver != t["ver"] - 1:
                return False
            p = pending.get((id(o), o.ver), 0)
            p -= sum(1 for (tl, v, _) in t["ins"] if tl is o and v == o.ver)
            return p == 0

        left = len(tasks)
        while left:
            choice = None
            for d in range(self.G):
                if pos[d] == len(lists[d]) or not ready(lists[d][pos[d]]):
                    continue
                h = self.hist[d]
                treq = h[len(h) - self.W] if len(h) >= self.W else 0
                if choice is None or treq < choice[1]:
                    choice = (d, treq)
            assert choice is not None, "deadlock"
            d, treq = choice
            t = lists[d][pos[d]]
            deps = [-1, -1, -1, -1]
            ready_at = 0
            for p, (tl, v, operand) in enumerate(t["ins"]):
                c = tl.gpus.get(d)
                if (id(tl), v) in lazy:
                    puller[(id(tl), v)] = designate((id(tl), v), d)
                pl = puller.get((id(tl), v))
                if (pl is not None and pl != d and (c is None or c.ver != v)
                        and not any(x.ver == v for x in tl.gpus.values())):
                    self.copy_in(tl, v, pl, treq, operand, out)  # first host read to its GPU
                if c is None or c.ver != v:
                    self.copy_in(tl, v, d, treq, operand, out)
                c = tl.gpus[d]
                ready_at = max(ready_at, c.t_done)
                if p < 4:
                    deps[p] = c.producer
                pending[(id(tl), v)] -= 1
            start = max(self.gfree[d], ready_at)
            end = start + self.nsec(t["flops"], self.rate)
            self.gfree[d] = end
            self.hist[d].append(end)
            o = t["out"]
            out.append((self.seq, TASK, 2, o.bi, o.bj, t["tk"], t["ver"], d, d, S_NONE, 0, start, end,
                        t["flops"], tuple(deps), t["op"]))
            o.ver = t["ver"]
            o.gpus = {d: Copy(t["ver"], end, self.seq, 0)}
            task_seq = self.seq
            self.seq += 1
            if sync and t.get("last"):
                self.copy_out(o, d, (0, 0, o.rows, o.cols), end, task_seq, out)
            pos[d] += 1
            left -= 1

    def locate(self, base, ld):
        for (b, l), (rows, cols) in self.extent.items():
            if l != ld or base < b:
                continue
            off = (base - b) // 8
            r, c = off % ld, off // ld
            if r < rows and c < cols:
                return b, r, c, rows, cols
        return None

    def coherent(self, base, m, n, ld, out):
        if m <= 0 or n <= 0:
            return
        loc = self.locate(base, ld)
        if loc is None:
            return
        b, r0, c0, rows, cols = loc
        T = self.T
        rend, cend = min(rows, r0 + m), min(cols, c0 + n)
        wb = []
        for bj in range(c0 // T, ceil_div(cend, T)):
            for bi in range(r0 // T, ceil_div(rend, T)):
                t = self.tiles.get((b, ld, bi, bj))
                if t is None or (t.host is not None and t.host.ver == t.ver):
                    continue
                holders = [g for g in range(self.G) if g in t.gpus and t.gpus[g].ver == t.ver]
                src = min(holders, key=lambda g: (t.gpus[g].t_done, g))
                tr0, tc0 = max(r0, bi * T) - bi * T, max(c0, bj * T) - bj * T
                tr1, tc1 = min(rend, bi * T + t.rows) - bi * T, min(cend, bj * T + t.cols) - bj * T
                if tr1 <= tr0 or tc1 <= tc0:
                    continue
                wb.append((t, src, (tr0, tc0, tr1 - tr0, tc1 - tc0)))
        # write-backs in completion order of their tiles (stable: column-major ties)
        wb.sort(key=lambda w: w[0].gpus[w[1]].t_done)
        for t, src, sub in wb:
            self.copy_out(t, src, sub, t.gpus[src].t_done, t.gpus[src].producer, out)

    def prefetch(self, base, m, n, ld, out, owner=None):
        if m <= 0 or n <= 0:
            return
        self.matrix(base, ld, m, n)
        T = self.T
        for bj in range(ceil_div(n, T)):
            for bi in range(ceil_div(m, T)):
                t = self.tile(base, ld, bi, bj)
                d = (owner or self.owner)(bi, bj)
                c = t.gpus.get(d)
                if c is not None and c.ver == t.ver:
                    continue
                self.copy_in(t, t.ver, d, 0, 2, out)

    def full_sync(self):
        for t in self.tiles.values():
            t.host = Copy(t.host.ver, 0, -1, t.host.depth) if t.host is not None else None
            for g in t.gpus:
                c = t.gpus[g]
                t.gpus[g] = Copy(c.ver, 0, -1, c.depth)
        self.link = {}
        self.gfree = [0] * self.G
        self.hist = [[] for _ in range(self.G)]

    def invalidate(self, base, shape, ld):
        m, n = shape
        if m <= 0 or n <= 0:
            return
        loc = self.locate(base, ld)
        if loc is None:
            return
        b, r0, c0, rows, cols = loc
        T = self.T
        rend, cend = min(rows, r0 + m), min(cols, c0 + n)
        for (bb, l, bi, bj), t in self.tiles.items():
            if (bb, l) != (b, ld):
                continue
            if bi * T >= rend or bi * T + t.rows <= r0 or bj * T >= cend or bj * T + t.cols <= c0:
                continue
            t.gpus = {}
            t.host = Copy(t.ver, 0, -1, 0)  # the host array is the valid copy from now on

    def release(self, base, shape, ld):
        """End of a sync call: drop the GPU copies of the view's tiles whose host copy is
        current; a tile valid only on a GPU (an earlier async call's output) keeps them."""
        m, n = shape
        if m <= 0 or n <= 0:
            return
        loc = self.locate(base, ld)
        if loc is None:
            return
        b, r0, c0, rows, cols = loc
        T = self.T
        rend, cend = min(rows, r0 + m), min(cols, c0 + n)
        for (bb, l, bi, bj), t in self.tiles.items():
            if (bb, l) != (b, ld):
                continue
            if bi * T >= rend or bi * T + t.rows <= r0 or bj * T >= cend or bj * T + t.cols <= c0:
                continue
            if t.host is not None and t.host.ver == t.ver:
                t.gpus = {}
