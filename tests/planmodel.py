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
DGEMM, COHERENT, SYNC, INVALIDATE, PREFETCH = 0, 100, 101, 102, 103


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


class Model:
    def __init__(self, bw, rate_mflops=35000000, topo="ranked", optimistic=True, window=2,
                 grid=(0, 0), tile=2048):
        self.bw = [list(r) for r in bw]
        self.G = len(bw) - 1
        self.cls = classes(self.bw)
        self.rate = rate_mflops
        self.mode = {"ranked": RANKED, "unranked": UNRANKED, "home": HOME}[topo] if isinstance(topo, str) else topo
        self.opt = bool(optimistic)
        self.W = max(1, window)
        self.P, self.Q = grid if grid[0] > 0 else near_square(self.G)
        self.T = tile
        self.tiles = {}          # (base, ld, bi, bj) -> Tile
        self.extent = {}         # (base, ld) -> [rows, cols]
        self.link = {}           # (src_idx, dst_idx) -> free time
        self.gfree = [0] * self.G
        self.hist = [[] for _ in range(self.G)]
        self.seq = 0

    # ------------------------------------------------------------------ helpers
    def owner(self, i, j):
        return (i % self.P) * self.Q + (j % self.Q)

    def tile(self, base, ld, bi, bj):
        key = (base, ld, bi, bj)
        if key not in self.tiles:
            rows, cols = self.extent[(base, ld)]
            self.tiles[key] = Tile(min(self.T, rows - bi * self.T), min(self.T, cols - bj * self.T), bi, bj)
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
                    state, depth, start, end, nbytes, (dep, -1, -1, -1)))
        t.gpus[d] = Copy(ver, end, self.seq, depth)
        self.seq += 1

    def copy_out(self, t, src, sub, ready, dep, out):
        r0, c0, rows, cols = sub
        nbytes = 8 * rows * cols
        lk = (src, self.G)
        start = max(ready, self.link.get(lk, 0))
        end = start + self.nsec(nbytes, self.bw[src][self.G])
        self.link[lk] = end
        out.append((self.seq, D2H, 2, t.bi, t.bj, -1, t.ver, HOSTID, src, S_VALID, 0, start, end,
                    nbytes, (dep, -1, -1, -1)))
        if (r0, c0, rows, cols) == (0, 0, t.rows, t.cols):
            t.host = Copy(t.ver, end, self.seq, 0)
        self.seq += 1

    # ------------------------------------------------------------------ calls
    def call(self, routine=DGEMM, transA="N", transB="N", m=0, n=0, k=0, alpha=1.0, beta=0.0,
             A=0, lda=1, B=0, ldb=1, C=0, ldc=1, sync=False):
        out = []
        if routine == DGEMM:
            self.gemm(transA.upper() in "TC", transB.upper() in "TC", m, n, k, alpha, beta,
                      A, lda, B, ldb, C, ldc, sync, out)
            if sync:
                self.full_sync()
                ta, tb = transA.upper() in "TC", transB.upper() in "TC"
                if alpha != 0 and k > 0:
                    self.invalidate(A, (k, m) if ta else (m, k), lda)
                    self.invalidate(B, (n, k) if tb else (k, n), ldb)
                self.invalidate(C, (m, n), ldc)
        elif routine == COHERENT:
            self.coherent(C, m, n, ldc, out)
        elif routine == SYNC:
            self.full_sync()
        elif routine == INVALIDATE:
            self.invalidate(C, (m, n), ldc)
        elif routine == PREFETCH:
            self.prefetch(C, m, n, ldc, out)
        return out

    def gemm(self, ta, tb, m, n, k, alpha, beta, A, lda, B, ldb, C, ldc, sync, out):
        if m == 0 or n == 0 or ((alpha == 0 or k == 0) and beta == 1):
            return
        T = self.T
        scale = alpha == 0 or k == 0
        self.matrix(C, ldc, m, n)
        if not scale:
            self.matrix(A, lda, *((k, m) if ta else (m, k)))
            self.matrix(B, ldb, *((n, k) if tb else (k, n)))
        tm, tn = ceil_div(m, T), ceil_div(n, T)
        tk = 0 if scale else ceil_div(k, T)
        tasks = []  # program order (j, i, kk)
        for j in range(tn):
            for i in range(tm):
                ct = self.tile(C, ldc, i, j)
                v0 = ct.ver
                mt, nt = min(T, m - i * T), min(T, n - j * T)
                if scale:
                    ins = [(ct, v0, 2)] if beta != 0 else []
                    tasks.append(dict(gpu=self.owner(i, j), out=ct, ver=v0 + 1, ins=ins, tk=-1, i=i,
                                      j=j, flops=mt * nt, last=True))
                    continue
                for kk in range(tk):
                    kt = min(T, k - kk * T)
                    at = self.tile(A, lda, kk, i) if ta else self.tile(A, lda, i, kk)
                    bt = self.tile(B, ldb, j, kk) if tb else self.tile(B, ldb, kk, j)
                    ins = [(at, at.ver, 0), (bt, bt.ver, 1)]
                    if kk > 0:
                        ins.append((ct, v0 + kk, 2))
                    elif beta != 0:
                        ins.append((ct, v0, 2))
                    tasks.append(dict(gpu=self.owner(i, j), out=ct, ver=v0 + kk + 1, ins=ins, tk=kk,
                                      i=i, j=j, flops=2 * mt * nt * kt, last=kk == tk - 1))
        self.run(tasks, sync, out)

    def run(self, tasks, sync, out):
        pending = {}
        for t in tasks:
            for (tl, v, _) in t["ins"]:
                pending[(id(tl), v)] = pending.get((id(tl), v), 0) + 1
        tmax = max([max(t["i"], t["j"]) + 1 for t in tasks] + [1])
        lists = [[] for _ in range(self.G)]
        for t in tasks:
            lists[t["gpu"]].append(t)
        for d in range(self.G):
            lists[d].sort(key=lambda t: (max(t["tk"], 0), (t["i"] + t["j"] + max(t["tk"], 0)) % tmax,
                                         t["i"], t["j"]))
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
            for (tl, v, operand) in t["ins"]:
                c = tl.gpus.get(d)
                if c is None or c.ver != v:
                    self.copy_in(tl, v, d, treq, operand, out)
                c = tl.gpus[d]
                ready_at = max(ready_at, c.t_done)
                deps[operand] = c.producer
                pending[(id(tl), v)] -= 1
            start = max(self.gfree[d], ready_at)
            end = start + self.nsec(t["flops"], self.rate)
            self.gfree[d] = end
            self.hist[d].append(end)
            o = t["out"]
            out.append((self.seq, TASK, 2, o.bi, o.bj, t["tk"], t["ver"], d, d, S_NONE, 0, start, end,
                        t["flops"], tuple(deps)))
            o.ver = t["ver"]
            o.gpus = {d: Copy(t["ver"], end, self.seq, 0)}
            task_seq = self.seq
            self.seq += 1
            if sync and t["last"]:
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
                self.copy_out(t, src, (tr0, tc0, tr1 - tr0, tc1 - tc0), t.gpus[src].t_done,
                              t.gpus[src].producer, out)

    def prefetch(self, base, m, n, ld, out):
        if m <= 0 or n <= 0:
            return
        self.matrix(base, ld, m, n)
        T = self.T
        for bj in range(ceil_div(n, T)):
            for bi in range(ceil_div(m, T)):
                t = self.tile(base, ld, bi, bj)
                d = self.owner(bi, bj)
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
