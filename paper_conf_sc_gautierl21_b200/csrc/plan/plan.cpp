// plan.cpp -- see plan.h.  Every numbered step below refers to SURVEY.md §8(c)
// "Plan oracle" (the readings are restated in DESIGN.md §Readings); the CPU model in
// tests/planmodel.py implements the same steps independently and must agree bit for bit.
#include "plan/plan.h"

#include <algorithm>
#include <cstring>
#include <map>
#include <tuple>

namespace xk {

static inline int64_t cdiv(int64_t a, int64_t b) { return (a + b - 1) / b; }

std::vector<int> link_classes(int G, const std::vector<int64_t> &bw) {
    // step 1: sort the off-diagonal bandwidths; a new class starts whenever consecutive
    // distinct values differ by a ratio > 1.25 (4*v[i] > 5*v[i-1]); higher = faster.
    const int N = G + 1;
    std::vector<int64_t> v;
    for (int s = 0; s < N; ++s)
        for (int d = 0; d < N; ++d)
            if (s != d) v.push_back(bw[(size_t)s * N + d]);
    std::sort(v.begin(), v.end());
    v.erase(std::unique(v.begin(), v.end()), v.end());
    std::map<int64_t, int> cls_of;
    int c = 0;
    for (size_t i = 0; i < v.size(); ++i) {
        if (i > 0 && 4 * v[i] > 5 * v[i - 1]) ++c;
        cls_of[v[i]] = c;
    }
    std::vector<int> cls((size_t)N * N, 1 << 20);
    for (int s = 0; s < N; ++s)
        for (int d = 0; d < N; ++d)
            if (s != d) cls[(size_t)s * N + d] = cls_of[bw[(size_t)s * N + d]];
    return cls;
}

Planner::Planner(const Topology &t, const Flags &f) : topo_(t), flags_(f) {
    cls_ = link_classes(t.G, t.bw);
    link_free_.assign((size_t)(t.G + 1) * (t.G + 1), 0);
    gpu_free_.assign(t.G, 0);
    ends_.assign(t.G, {});
}

int64_t Planner::dur(int64_t amount, int64_t rate) const {
    // copies: ceil(bytes*1000 / MBps) ns; tasks: ceil(flops*1000 / MFLOPs) ns (step 3, 5)
    return cdiv(amount * 1000, rate);
}

int Planner::find_or_add_matrix(uint64_t base, int64_t ld, int64_t rows, int64_t cols,
                                std::string &err) {
    for (size_t i = 0; i < mats_.size(); ++i) {
        Matrix &M = mats_[i];
        if (M.ld < 0 || M.shadow) continue;  // forgotten / per-call shadow
        if (M.base == base && M.ld == ld) {
            // tile extents must agree with the cached grid (step 9)
            int64_t T = flags_.T;
            auto edge_ok = [&](int64_t a, int64_t b) {
                // same ragged edge tile or both multiples beyond the shorter extent
                int64_t lo = std::min(a, b), hi = std::max(a, b);
                if (lo == hi) return true;
                return lo % T == 0 && cdiv(lo, T) <= cdiv(hi, T);
            };
            if (!edge_ok(M.rows, rows) || !edge_ok(M.cols, cols)) {
                // a clean matrix (no GPU copies, host valid) can simply be forgotten
                bool clean = true;
                for (auto &kv : keymap_) {
                    const Entry &e = entries_[kv.second];
                    if (e.mat != (int)i) continue;
                    for (auto &g : e.gpu) clean = clean && !g.present;
                    clean = clean && e.host.present && e.host.ver == e.ver;
                }
                if (!clean) {
                    err = "view of a cached matrix with a different tiling (make it coherent and invalidate first)";
                    return -1;
                }
                for (auto it = keymap_.begin(); it != keymap_.end();)
                    if (entries_[it->second].mat == (int)i) it = keymap_.erase(it); else ++it;
                M.grid.clear();
                M.gr = M.gc = 0;
                M.rows = rows;
                M.cols = cols;
                return (int)i;
            }
            M.rows = std::max(M.rows, rows);
            M.cols = std::max(M.cols, cols);
            return (int)i;
        }
    }
    // overlap with another cached matrix at a different anchor -> unsupported unless clean
    uint64_t lo = base, hi = base + (uint64_t)((cols - 1) * ld + rows) * 8;
    for (size_t i = 0; i < mats_.size(); ++i) {
        Matrix &M = mats_[i];
        if (M.ld < 0 || M.shadow) continue;
        uint64_t mlo = M.base, mhi = M.base + (uint64_t)((M.cols - 1) * M.ld + M.rows) * 8;
        if (lo < mhi && mlo < hi) {
            bool clean = true;
            for (auto &kv : keymap_) {
                const Entry &e = entries_[kv.second];
                if (e.mat != (int)i) continue;
                for (auto &g : e.gpu) clean = clean && !g.present;
                clean = clean && e.host.present && e.host.ver == e.ver;
            }
            if (!clean) {
                err = "view overlaps a cached matrix anchored elsewhere (make it coherent and invalidate first)";
                return -1;
            }
            for (auto it = keymap_.begin(); it != keymap_.end();)
                if (entries_[it->second].mat == (int)i) it = keymap_.erase(it); else ++it;
            M.grid.clear();
            M.gr = M.gc = 0;
            M.ld = -1;  // forget
        }
    }
    Matrix M;
    M.base = base;
    M.ld = ld;
    M.rows = rows;
    M.cols = cols;
    mats_.push_back(M);
    return (int)mats_.size() - 1;
}

int Planner::key_of(int mat, int64_t bi, int64_t bj) {
    Matrix &Mx = mats_[mat];
    const int64_t tr = cdiv(Mx.rows, flags_.T), tc = cdiv(Mx.cols, flags_.T);
    if (Mx.gr != tr || Mx.gc != tc) {  // (re)build the dense cache from the directory
        Mx.grid.assign((size_t)(tr * tc), -1);
        Mx.gr = tr;
        Mx.gc = tc;
        for (const auto &kv : keymap_) {
            const Entry &e = entries_[kv.second];
            if (e.mat == mat && e.bi < tr && e.bj < tc) Mx.grid[(size_t)(e.bi + e.bj * tr)] = kv.second;
        }
    }
    const bool in_grid = bi < tr && bj < tc;
    if (in_grid && Mx.grid[(size_t)(bi + bj * tr)] >= 0) return Mx.grid[(size_t)(bi + bj * tr)];
    const uint64_t k = tile_key(mat, bi, bj);
    auto it = keymap_.find(k);
    if (it != keymap_.end()) {
        if (in_grid) Mx.grid[(size_t)(bi + bj * tr)] = it->second;
        return it->second;
    }
    Entry e;
    e.mat = mat;
    e.bi = bi;
    e.bj = bj;
    const Matrix &M = mats_[mat];
    e.rows = std::min(flags_.T, M.rows - bi * flags_.T);
    e.cols = std::min(flags_.T, M.cols - bj * flags_.T);
    e.ver = 0;
    e.host.present = true;  // inputs start VALID on the host (step 4)
    e.host.ver = 0;
    e.gpu.assign(topo_.G, NodeCopy());
    entries_.push_back(e);
    int id = (int)entries_.size() - 1;
    keymap_[k] = id;
    if (in_grid) mats_[mat].grid[(size_t)(bi + bj * tr)] = id;
    return id;
}

// step 4: source selection for a tile needed on GPU d at request time treq.
int Planner::select_source(const Entry &e, int64_t ver, int d, int64_t treq, int *state) const {
    const int G = topo_.G;
    struct Small {  // G <= XK_MAX_GPUS candidates, no allocation
        int v[XK_MAX_GPUS];
        int n = 0;
        void push_back(int g) { v[n++] = g; }
        bool empty() const { return n == 0; }
        int front() const { return v[0]; }
        const int *begin() const { return v; }
        const int *end() const { return v + n; }
    } V, I;
    for (int g = 0; g < G; ++g) {
        if (g == d) continue;
        const NodeCopy &c = e.gpu[g];
        if (!c.present || c.ver != ver) continue;
        if (c.t_done <= treq) V.push_back(g); else I.push_back(g);
    }
    bool host_ok = e.host.present && e.host.ver == ver;
    auto ranked_best = [&](const Small &L) {
        int best = -1;
        std::tuple<int, int, int> bk;
        for (int g : L) {
            std::tuple<int, int, int> k(-cls_[(size_t)g * (G + 1) + d], e.gpu[g].depth,
                                        ((g - d) % G + G) % G);
            if (best < 0 || k < bk) { best = g; bk = k; }
        }
        return best;
    };
    auto lowest = [&](const Small &L) { return L.empty() ? -1 : L.front(); };
    int mode = flags_.topo;
    if (mode == XK_TOPO_HOME) {
        if (host_ok) { *state = XK_SRC_HOST; return XK_HOST; }
        if (!V.empty()) { *state = XK_SRC_VALID; return lowest(V); }
        if (!I.empty()) { *state = XK_SRC_INFLIGHT; return lowest(I); }
        *state = XK_SRC_NONE;
        return -2;
    }
    auto pick = [&](const Small &L) {
        return mode == XK_TOPO_RANKED ? ranked_best(L) : lowest(L);
    };
    if (!V.empty()) { *state = XK_SRC_VALID; return pick(V); }
    if (!I.empty() && (flags_.optimistic || !host_ok)) { *state = XK_SRC_INFLIGHT; return pick(I); }
    if (host_ok) { *state = XK_SRC_HOST; return XK_HOST; }
    *state = XK_SRC_NONE;
    return -2;
}

// step 5: copy timing, store-and-forward after the source copy completes.
bool Planner::emit_copy(int key, int64_t ver, int d, int64_t treq, int operand,
                        std::vector<Rec> &out) {
    Entry &e = entries_[key];
    const int G = topo_.G;
    int state = 0;
    int src = select_source(e, ver, d, treq, &state);
    if (src == -2) return false;  // no copy of this version anywhere (lost by invalidate)
    int sidx = (src == XK_HOST) ? G : src;
    int64_t bytes = 8 * e.rows * e.cols;
    int64_t src_ready, dep;
    int depth;
    if (src == XK_HOST) {
        src_ready = e.host.t_done;
        dep = e.host.producer;
        depth = 1;
    } else {
        src_ready = e.gpu[src].t_done;
        dep = e.gpu[src].producer;
        depth = e.gpu[src].depth + 1;
    }
    int64_t &lf = link_free_[(size_t)sidx * (G + 1) + d];
    int64_t t0 = std::max(treq, std::max(src_ready, lf));
    int64_t t1 = t0 + dur(bytes, topo_.bw_at(sidx, d));
    lf = t1;
    Rec R;
    std::memset(&R.r, 0, sizeof(R.r));
    R.r.seq = seq_++;
    R.r.kind = (src == XK_HOST) ? XK_REC_H2D : XK_REC_P2P;
    R.r.operand = operand;
    R.r.bi = e.bi;
    R.r.bj = e.bj;
    R.r.tk = -1;
    R.r.version = ver;
    R.r.dst = d;
    R.r.src = src;
    R.r.src_state = state;
    R.r.depth = depth;
    R.r.t_start = t0;
    R.r.t_end = t1;
    R.r.work = bytes;
    R.r.dep[0] = dep;
    R.r.dep[1] = R.r.dep[2] = R.r.dep[3] = -1;
    R.r.op = -1;
    R.key = key;
    R.sub_rows = e.rows;
    R.sub_cols = e.cols;
    emit(R, out);
    NodeCopy &c = e.gpu[d];
    c.present = true;
    c.ver = ver;
    c.t_done = t1;
    c.producer = R.r.seq;
    c.depth = depth;
    // R15: a read-once shadow's host memory is rewritten by the write-back of the output tile
    // it shadows, so after its one host read every other copy is forwarded from a GPU (all of
    // them descend from this H2D, which the output tile's own chain also waits on)
    if (src == XK_HOST && mats_[e.mat].host_once) e.host.present = false;
    return true;
}

void Planner::emit_d2h(int key, int src, int64_t r0, int64_t c0, int64_t rows, int64_t cols,
                       int64_t ready, int64_t dep, int operand, std::vector<Rec> &out) {
    Entry &e = entries_[key];
    const int G = topo_.G;
    int64_t bytes = 8 * rows * cols;
    int64_t &lf = link_free_[(size_t)src * (G + 1) + G];
    int64_t t0 = std::max(ready, lf);
    int64_t t1 = t0 + dur(bytes, topo_.bw_at(src, G));
    lf = t1;
    Rec R;
    std::memset(&R.r, 0, sizeof(R.r));
    R.r.seq = seq_++;
    R.r.kind = XK_REC_D2H;
    R.r.operand = operand;
    R.r.bi = e.bi;
    R.r.bj = e.bj;
    R.r.tk = -1;
    R.r.version = e.ver;
    R.r.dst = XK_HOST;
    R.r.src = src;
    R.r.src_state = XK_SRC_VALID;
    R.r.depth = 0;
    R.r.t_start = t0;
    R.r.t_end = t1;
    R.r.work = bytes;
    R.r.dep[0] = dep;
    R.r.dep[1] = R.r.dep[2] = R.r.dep[3] = -1;
    R.r.op = -1;
    R.key = key;
    R.sub_r0 = r0;
    R.sub_c0 = c0;
    R.sub_rows = rows;
    R.sub_cols = cols;
    emit(R, out);
    if (r0 == 0 && c0 == 0 && rows == e.rows && cols == e.cols) {
        e.host.present = true;
        e.host.ver = e.ver;
        e.host.t_done = t1;
        e.host.producer = R.r.seq;
        e.host.depth = 0;
    }
}

// R16 quotas: split count[S] host tiles of each shared requester set S over its members so
// that the largest per-GPU total (forced[g] + assigned) is as small as possible.  Binary
// search on that maximum L; feasibility is a max-flow (source -> set S, capacity count[S];
// S -> member g; g -> sink, capacity L - forced[g]) by Edmonds-Karp: BFS over nodes in index
// order (0 source, 1..nS sets, then GPUs, then sink), augmenting by the bottleneck.  The flow
// on S -> g is the quota (deterministic; the CPU plan model runs the same procedure).
static std::vector<std::vector<int64_t>> balance_quotas(int G, const std::vector<uint32_t> &sets,
                                                        const std::vector<int64_t> &count,
                                                        const std::vector<int64_t> &forced) {
    const int nS = (int)sets.size(), V = nS + G + 2, src = 0, snk = V - 1;
    int64_t total = 0, fmax = 0, ftot = 0;
    for (int64_t c : count) total += c;
    for (int64_t f : forced) { fmax = std::max(fmax, f); ftot += f; }
    std::vector<int64_t> cap, flow;
    auto run = [&](int64_t L) {
        cap.assign((size_t)V * V, 0);
        flow.assign((size_t)V * V, 0);
        for (int i = 0; i < nS; ++i) {
            cap[(size_t)src * V + 1 + i] = count[i];
            for (int g = 0; g < G; ++g)
                if (sets[i] >> g & 1) cap[(size_t)(1 + i) * V + 1 + nS + g] = total;
        }
        for (int g = 0; g < G; ++g) cap[(size_t)(1 + nS + g) * V + snk] = std::max<int64_t>(0, L - forced[g]);
        int64_t got = 0;
        std::vector<int> par(V);
        for (;;) {
            std::fill(par.begin(), par.end(), -1);
            par[src] = src;
            std::vector<int> q{src};
            for (size_t h = 0; h < q.size() && par[snk] < 0; ++h) {
                const int u = q[h];
                for (int v = 0; v < V; ++v)
                    if (par[v] < 0 && cap[(size_t)u * V + v] - flow[(size_t)u * V + v] > 0) {
                        par[v] = u;
                        q.push_back(v);
                    }
            }
            if (par[snk] < 0) break;
            int64_t b = INT64_MAX;
            for (int v = snk; v != src; v = par[v])
                b = std::min(b, cap[(size_t)par[v] * V + v] - flow[(size_t)par[v] * V + v]);
            for (int v = snk; v != src; v = par[v]) {
                flow[(size_t)par[v] * V + v] += b;
                flow[(size_t)v * V + par[v]] -= b;
            }
            got += b;
        }
        return got == total;
    };
    int64_t lo = std::max(fmax, (total + ftot + G - 1) / G), hi = fmax + total;
    while (lo < hi) {
        const int64_t mid = lo + (hi - lo) / 2;
        if (run(mid)) hi = mid; else lo = mid + 1;
    }
    run(lo);
    std::vector<std::vector<int64_t>> quota(nS, std::vector<int64_t>(G, 0));
    for (int i = 0; i < nS; ++i)
        for (int g = 0; g < G; ++g) quota[i][g] = std::max<int64_t>(0, flow[(size_t)(1 + i) * V + 1 + nS + g]);
    return quota;
}

// steps 2, 3, 6, 7: per-GPU lists ordered by the generator's sort key (k-major, k-shifted
// anti-diagonal), event loop on the smallest request time, task timing, output
// versioning, D2H after the last writer of each output tile.
int Planner::run_tasks(std::vector<Task> &tasks, bool sync, std::vector<Rec> &out, std::string &err) {
    const int G = topo_.G;
    const int W = std::max(1, flags_.window);
    // pending reads per (key, version) in this call, resolved once to flat counter slots.
    // Tasks are in program order and a key's versions only grow along it, so all reads of
    // (key, v) precede the write of v + 1: one (version, slot) pair per key suffices.
    std::vector<int64_t> pending;
    {
        std::vector<int64_t> last_ver(entries_.size(), -1);
        std::vector<int> last_slot(entries_.size(), -1);
        pending.reserve(tasks.size());
        for (auto &t : tasks) {
            for (auto &in : t.in) {
                if (last_slot[in.key] < 0 || last_ver[in.key] != in.ver) {
                    last_ver[in.key] = in.ver;
                    last_slot[in.key] = (int)pending.size();
                    pending.push_back(0);
                }
                in.cnt = last_slot[in.key];
                pending[in.cnt]++;
            }
            // WAR: readers of the version this task overwrites (all precede it)
            t.war = (last_slot[t.out_key] >= 0 && last_ver[t.out_key] == t.out_ver - 1) ? last_slot[t.out_key] : -1;
        }
    }
    // Balance-aware first host pull (reading R16; FULL mode only: it forwards from an in-flight
    // copy).  An input tile version valid only on the host at the start of the call crosses
    // PCIe once; which requester's link carries it is fixed here, before the event loop, so that
    // the most loaded host link carries as few tiles as possible: a tile read by one GPU goes to
    // that GPU; the tiles read by several GPUs are grouped by requester set and split by the
    // min-max quotas of balance_quotas(), then dealt inside each set in first-appearance order
    // to the member furthest below its quota.  When another requester asks first, the tile is
    // pulled to its designated GPU and forwarded from there (store-and-forward over NVLink).
    std::vector<int> puller(pending.size(), -1);
    std::vector<int> slot_set(pending.size(), -1);   // shared requester set of a host-only slot
    std::vector<std::vector<int64_t>> quota;         // per set: host tiles each member may still carry
    std::vector<uint32_t> set_mask;
    if (flags_.optimistic && flags_.topo != XK_TOPO_HOME && G > 1) {
        std::vector<uint32_t> mask(pending.size(), 0);
        std::vector<int> order;  // slots in first-appearance order
        std::vector<int> slot_key(pending.size(), -1);
        std::vector<int64_t> slot_ver(pending.size(), 0);
        for (const auto &t : tasks)
            for (const auto &in : t.in) {
                if (slot_key[in.cnt] < 0) order.push_back(in.cnt);
                mask[in.cnt] |= 1u << t.gpu;
                slot_key[in.cnt] = in.key;
                slot_ver[in.cnt] = in.ver;
            }
        auto host_only = [&](int s) {
            const Entry &e = entries_[slot_key[s]];
            if (e.ver != slot_ver[s] || !(e.host.present && e.host.ver == e.ver)) return false;
            for (const NodeCopy &g : e.gpu)
                if (g.present && g.ver == e.ver) return false;
            return true;
        };
        std::vector<int64_t> forced(G, 0);
        std::vector<uint32_t> sets;            // shared requester sets, first-appearance order
        std::vector<int64_t> count;            // host-only tiles per set
        std::unordered_map<uint32_t, int> set_id;
        for (int s : order) {
            if (!host_only(s)) continue;
            if ((mask[s] & (mask[s] - 1)) == 0) {
                int g = __builtin_ctz(mask[s]);
                puller[s] = g;
                forced[g]++;
                continue;
            }
            auto it = set_id.find(mask[s]);
            if (it == set_id.end()) {
                it = set_id.emplace(mask[s], (int)sets.size()).first;
                sets.push_back(mask[s]);
                count.push_back(0);
            }
            count[it->second]++;
        }
        if (!sets.empty()) {
            quota = balance_quotas(G, sets, count, forced);
            for (int s : order)
                if (puller[s] < 0 && host_only(s)) slot_set[s] = set_id[mask[s]];
            set_mask = sets;
        }
    }
    // the designated GPU of a shared tile is chosen at its first request (R16): the requester
    // itself while its quota in that set lasts (no extra hop), else the member with the most
    // quota left (ties: lowest id)
    auto designate = [&](int slot, int d) {
        const int id = slot_set[slot];
        auto &q = quota[id];
        if (q[d] > 0) {
            q[d]--;
            return d;
        }
        int best = -1;
        for (int g = 0; g < G; ++g)
            if ((set_mask[id] >> g & 1) && q[g] > 0 && (best < 0 || q[g] > q[best])) best = g;
        q[best]--;
        return best;
    };
    // last writer per output tile
    std::unordered_map<int, size_t> last;
    for (size_t q = 0; q < tasks.size(); ++q) {
        auto it = last.find(tasks[q].out_key);
        if (it == last.end() || tasks[it->second].out_ver < tasks[q].out_ver) last[tasks[q].out_key] = q;
    }
    for (auto &kv : last) tasks[kv.second].last_writer = true;
    out.reserve(out.size() + tasks.size() * 2);
    std::vector<std::vector<int>> lists(G);
    {
        // per-GPU order by the generator's sort key (ties: generation order), sorted on a
        // compact copy of the keys rather than through the large Task records
        struct SK { int64_t k[5]; int idx; };
        std::vector<std::vector<SK>> keys(G);
        for (size_t q = 0; q < tasks.size(); ++q) {
            SK s;
            std::copy(tasks[q].skey, tasks[q].skey + 5, s.k);
            s.idx = (int)q;
            keys[tasks[q].gpu].push_back(s);
        }
        for (int d = 0; d < G; ++d) {
            std::sort(keys[d].begin(), keys[d].end(), [](const SK &x, const SK &y) {
                for (int q = 0; q < 5; ++q)
                    if (x.k[q] != y.k[q]) return x.k[q] < y.k[q];
                return x.idx < y.idx;
            });
            lists[d].reserve(keys[d].size());
            for (const SK &s : keys[d]) lists[d].push_back(s.idx);
        }
    }
    std::vector<size_t> pos(G, 0);
    auto ready = [&](const Task &t) {
        for (auto &in : t.in)
            if (entries_[in.key].ver != in.ver) return false;
        const Entry &o = entries_[t.out_key];
        if (o.ver != t.out_ver - 1) return false;
        int64_t pend = (t.war < 0) ? 0 : pending[t.war];
        for (auto &in : t.in)
            if (in.key == t.out_key && in.ver == t.out_ver - 1) pend--;
        return pend == 0;
    };
    size_t done = 0;
    std::vector<std::pair<int64_t, int>> cand(G);
    while (done < tasks.size()) {
        // the GPU with the smallest request time whose next task is ready (ties: lower id);
        // readiness is only evaluated in (treq, d) order until the first ready one
        int nc = 0;
        for (int d = 0; d < G; ++d) {
            if (pos[d] == lists[d].size()) continue;
            const auto &h = ends_[d];
            int64_t treq = (int64_t)h.size() >= W ? h[h.size() - W] : 0;
            cand[nc++] = {treq, d};
        }
        std::sort(cand.begin(), cand.begin() + nc);
        int best = -1;
        int64_t best_treq = 0;
        for (int c = 0; c < nc; ++c) {
            if (ready(tasks[lists[cand[c].second][pos[cand[c].second]]])) {
                best = cand[c].second;
                best_treq = cand[c].first;
                break;
            }
        }
        if (best < 0) {
            err = "planner deadlock: no ready task (output aliases an input?)";
            return XK_ERR_INTERNAL;
        }
        const int d = best;
        Task &t = tasks[lists[d][pos[d]]];
        const int64_t treq = best_treq;
        int64_t in_ready = 0;
        int64_t deps[4] = {-1, -1, -1, -1};
        for (size_t p = 0; p < t.in.size(); ++p) {
            const Input &in = t.in[p];
            Entry &e = entries_[in.key];
            if (slot_set[in.cnt] >= 0 && puller[in.cnt] < 0) puller[in.cnt] = designate(in.cnt, d);
            const int pl = puller[in.cnt];
            if (pl >= 0 && pl != d && !(e.gpu[d].present && e.gpu[d].ver == in.ver)) {
                // R16: the first host read of this tile goes to its designated GPU
                bool any = false;
                for (const NodeCopy &g : e.gpu) any = any || (g.present && g.ver == in.ver);
                if (!any && !emit_copy(in.key, in.ver, pl, treq, in.operand, out)) {
                    err = "no valid copy of an input tile (invalidated without coherence?)";
                    return XK_ERR_INTERNAL;
                }
            }
            if (!(e.gpu[d].present && e.gpu[d].ver == in.ver) &&
                !emit_copy(in.key, in.ver, d, treq, in.operand, out)) {
                err = "no valid copy of an input tile (invalidated without coherence?)";
                return XK_ERR_INTERNAL;
            }
            in_ready = std::max(in_ready, e.gpu[d].t_done);
            if (p < 4) deps[p] = e.gpu[d].producer;
            pending[in.cnt]--;
        }
        int64_t t0 = std::max(gpu_free_[d], in_ready);
        int64_t t1 = t0 + dur(t.flops, topo_.rate_mflops);
        gpu_free_[d] = t1;
        ends_[d].push_back(t1);
        Entry &o = entries_[t.out_key];
        Rec R;
        std::memset(&R.r, 0, sizeof(R.r));
        R.r.seq = seq_++;
        R.r.kind = XK_REC_TASK;
        R.r.operand = 2;
        R.r.bi = o.bi;
        R.r.bj = o.bj;
        R.r.tk = t.tk;
        R.r.version = t.out_ver;
        R.r.dst = d;
        R.r.src = d;
        R.r.src_state = XK_SRC_NONE;
        R.r.depth = 0;
        R.r.op = t.op;
        R.r.t_start = t0;
        R.r.t_end = t1;
        R.r.work = t.flops;
        for (int q = 0; q < 4; ++q) R.r.dep[q] = deps[q];
        R.key = t.out_key;
        R.op = t.op;
        R.keyA = t.keyA;
        R.keyB = t.keyB;
        R.keyC2 = t.keyC2;
        R.beta2 = t.beta2;
        R.ta = t.ta;
        R.tb = t.tb;
        R.side = t.side;
        R.uplo = t.uplo;
        R.diag = t.diag;
        R.tri = t.tri;
        R.alpha = t.alpha;
        R.beta = t.beta;
        R.m = t.m;
        R.n = t.n;
        R.k = t.k;
        R.remaining = (int64_t)(lists[d].size() - pos[d]) - 1;
        emit(R, out);
        if (sink_rc_) {
            err = "issue failed";
            return sink_rc_;
        }
        o.ver = t.out_ver;
        for (int g = 0; g < G; ++g)
            if (g != d) o.gpu[g].present = false;
        o.gpu[d].present = true;
        o.gpu[d].ver = t.out_ver;
        o.gpu[d].t_done = t1;
        o.gpu[d].producer = R.r.seq;
        o.gpu[d].depth = 0;
        if (sync && t.last_writer)
            emit_d2h(t.out_key, d, 0, 0, o.rows, o.cols, t1, R.r.seq, 2, out);
        pos[d]++;
        done++;
    }
    return XK_OK;
}

static bool is_t(char c) { return c == 'T' || c == 't' || c == 'C' || c == 'c'; }
static char up(char c) { return (c >= 'a' && c <= 'z') ? (char)(c - 32) : c; }

// beta deferral (reading Q12''): when a C tile's input is valid on the host only and its
// chain has >= 2 tasks, the first task does not read C (beta = 0) and the last one adds
// beta * C_input from a per-call shadow copy of the tile -- C crosses PCIe at the end of its
// chain, when the link is idle, instead of together with the first A/B tiles.  Tiles
// already valid on some GPU (data-on-device) are read in place as before.
int Planner::add_shadow(int mc) {
    Matrix S = mats_[mc];
    S.shadow = true;
    S.grid.clear();  // its own tiles (never C's cached ids)
    S.gr = S.gc = 0;
    mats_.push_back(S);
    return (int)mats_.size() - 1;
}

bool Planner::defer_beta(int keyC) const {
    const Entry &ec = entries_[keyC];
    if (!(ec.host.present && ec.host.ver == ec.ver)) return false;
    for (const NodeCopy &g : ec.gpu)  // already resident on a GPU: nothing to defer
        if (g.present && g.ver == ec.ver) return false;
    return true;
}

// the shadow tiles were only this call's inputs: drop their GPU copies and forget them
void Planner::drop_shadow(int ms) {
    if (ms < 0) return;
    for (auto it = keymap_.begin(); it != keymap_.end();) {
        if (entries_[it->second].mat == ms) {
            for (auto &gc : entries_[it->second].gpu) gc.present = false;
            it = keymap_.erase(it);
        } else {
            ++it;
        }
    }
    mats_[ms].grid.clear();
    mats_[ms].gr = mats_[ms].gc = 0;
    mats_[ms].ld = -1;
}

// A shadow adds a second copy of C's (TRMM: B's) tiles to the device footprint, and there is
// no eviction: the shadow plan is used only if, on every GPU, the tiles resident now plus the
// tiles this call's tasks read or write there fit in the capacity (device buffers hold
// round_up(rows, 16) x cols doubles).  Otherwise the call is planned without a shadow.
bool Planner::fits(const std::vector<Task> &tasks) const {
    if (flags_.mem_bytes <= 0) return true;
    const int G = topo_.G;
    std::vector<int64_t> bytes(G, 0);
    std::vector<std::vector<char>> seen(G, std::vector<char>(entries_.size(), 0));
    auto add = [&](int g, int key) {
        if (key < 0 || seen[g][key]) return;
        seen[g][key] = 1;
        const Entry &e = entries_[key];
        bytes[g] += 8 * ((e.rows + 15) / 16 * 16) * e.cols;
    };
    for (const auto &kv : keymap_)
        for (int g = 0; g < G; ++g)
            if (entries_[kv.second].gpu[g].present) add(g, kv.second);
    for (const Task &t : tasks) {
        add(t.gpu, t.out_key);
        for (const Input &in : t.in) add(t.gpu, in.key);
    }
    for (int g = 0; g < G; ++g)
        if (bytes[g] > flags_.mem_bytes) return false;
    return true;
}

// DGEMM (PLASMA pdgemm structure): C(i,j) k-chains, beta on the first task.
int Planner::plan_gemm(const xk_call_t &c, std::vector<Rec> &out, std::string &err) {
    const int64_t m = c.m, n = c.n, k = c.k, T = flags_.T;
    const bool ta = is_t(c.transA), tb = is_t(c.transB);
    if (m == 0 || n == 0 || ((c.alpha == 0.0 || k == 0) && c.beta == 1.0)) return XK_OK;
    const bool scale_only = (c.alpha == 0.0 || k == 0);
    int mc = find_or_add_matrix(c.C, (int64_t)c.ldc, m, n, err);
    if (mc < 0) return XK_ERR_UNSUPPORTED;
    int ma = -1, mb = -1;
    if (!scale_only) {
        ma = find_or_add_matrix(c.A, (int64_t)c.lda, ta ? k : m, ta ? m : k, err);
        if (ma < 0) return XK_ERR_UNSUPPORTED;
        mb = find_or_add_matrix(c.B, (int64_t)c.ldb, tb ? n : k, tb ? k : n, err);
        if (mb < 0) return XK_ERR_UNSUPPORTED;
    }
    const int64_t tm = cdiv(m, T), tn = cdiv(n, T), tkn = scale_only ? 0 : cdiv(k, T);
    const int64_t tmod = std::max<int64_t>(1, std::max(tm, tn));
    int ms = (!scale_only && c.beta != 0.0 && tkn >= 2) ? add_shadow(mc) : -1;
    std::vector<Task> tasks;
    for (;;) {  // with the shadow if it fits (fits()), else without
        Versions V;
        V.e = &entries_;
        tasks.clear();
        tasks.reserve((size_t)(tm * tn * std::max<int64_t>(tkn, 1)));
        for (int64_t j = 0; j < tn; ++j) {
            for (int64_t i = 0; i < tm; ++i) {
                int keyC = key_of(mc, i, j);
                int64_t mt = std::min(T, m - i * T), nt = std::min(T, n - j * T);
                if (scale_only) {
                    Task t;
                    t.gpu = owner(i, j);
                    t.op = XK_OP_SCALE;
                    t.out_key = keyC;
                    if (c.beta != 0.0) t.in.push_back({keyC, V.get(keyC), 2});
                    t.out_ver = V.bump(keyC);
                    t.beta = c.beta;
                    t.tk = -1;
                    t.i = i; t.j = j;
                    t.m = mt; t.n = nt; t.k = 0;
                    t.flops = mt * nt;
                    int64_t sk[5] = {0, (i + j) % tmod, i, j, 0};
                    std::copy(sk, sk + 5, t.skey);
                    tasks.push_back(t);
                    continue;
                }
                const bool defer = ms >= 0 && defer_beta(keyC);
                const int keyS = defer ? key_of(ms, i, j) : -1;
                for (int64_t kk = 0; kk < tkn; ++kk) {
                    int64_t kt = std::min(T, k - kk * T);
                    int keyA = ta ? key_of(ma, kk, i) : key_of(ma, i, kk);
                    int keyB = tb ? key_of(mb, j, kk) : key_of(mb, kk, j);
                    Task t;
                    t.gpu = owner(i, j);
                    t.op = XK_OP_GEMM;
                    t.out_key = keyC;
                    t.in.push_back({keyA, V.get(keyA), 0});
                    t.in.push_back({keyB, V.get(keyB), 1});
                    if (kk > 0 || (c.beta != 0.0 && !defer)) t.in.push_back({keyC, V.get(keyC), 2});
                    if (defer && kk == tkn - 1) {
                        t.in.push_back({keyS, V.get(keyS), 2});
                        t.keyC2 = keyS;
                        t.beta2 = c.beta;
                    }
                    t.out_ver = V.bump(keyC);
                    t.keyA = keyA;
                    t.keyB = keyB;
                    t.ta = ta ? 'T' : 'N';
                    t.tb = tb ? 'T' : 'N';
                    t.alpha = c.alpha;
                    t.beta = (kk == 0) ? (defer ? 0.0 : c.beta) : 1.0;
                    t.tk = kk;
                    t.i = i; t.j = j;
                    t.m = mt; t.n = nt; t.k = kt;
                    t.flops = 2 * mt * nt * kt;
                    // staggered k-chains (reading Q12'): tile (i,j) starts its chain at slot
                    // (i+j) mod tk, so chains begin and end at different times and C's D2H
                    // spreads over the last tk slots instead of piling up at the end
                    int64_t sk[5] = {kk + (i + j) % tkn, (i + j + kk) % tmod, i, j, 0};
                    std::copy(sk, sk + 5, t.skey);
                    tasks.push_back(t);
                }
            }
        }
        if (ms >= 0 && !fits(tasks)) {
            drop_shadow(ms);
            ms = -1;
            continue;
        }
        break;
    }
    int rc = run_tasks(tasks, c.sync != 0, out, err);
    drop_shadow(ms);
    return rc;
}

// DSYRK / DSYR2K (PLASMA pdsyrk / pdsyr2k): tiles of the uplo triangle of C; off-diagonal
// tiles are GEMM k-chains, diagonal tiles GEMM_TRI tasks writing only the triangle.  A
// diagonal tile is always copied in (even when beta == 0) so the untouched triangle goes
// back to the host bit for bit (BLAS: it is not referenced).
int Planner::plan_syrk(const xk_call_t &c, bool two, std::vector<Rec> &out, std::string &err) {
    const int64_t n = c.n, k = c.k, T = flags_.T;
    const bool tr = is_t(c.transA), lower = up(c.uplo) == 'L';
    if (n == 0 || ((c.alpha == 0.0 || k == 0) && c.beta == 1.0)) return XK_OK;
    const bool scale_only = (c.alpha == 0.0 || k == 0);
    int mc = find_or_add_matrix(c.C, (int64_t)c.ldc, n, n, err);
    if (mc < 0) return XK_ERR_UNSUPPORTED;
    int ma = -1, mb = -1;
    if (!scale_only) {
        ma = find_or_add_matrix(c.A, (int64_t)c.lda, tr ? k : n, tr ? n : k, err);
        if (ma < 0) return XK_ERR_UNSUPPORTED;
        if (two) {
            mb = find_or_add_matrix(c.B, (int64_t)c.ldb, tr ? k : n, tr ? n : k, err);
            if (mb < 0) return XK_ERR_UNSUPPORTED;
        }
    }
    const int64_t tn = cdiv(n, T), tkn = scale_only ? 0 : cdiv(k, T);
    const int64_t tmod = std::max<int64_t>(1, tn);
    const int tri = lower ? 1 : 2;
    const int64_t nchain = tkn * (two ? 2 : 1);  // tasks per C tile
    int ms = (!scale_only && c.beta != 0.0 && nchain >= 2) ? add_shadow(mc) : -1;
    std::vector<Task> tasks;
    for (;;) {  // with the shadow if it fits (fits()), else without
        Versions V;
        V.e = &entries_;
        tasks.clear();
        auto opnd = [&](int mat, int64_t r, int64_t l) {  // tile (r, l) of op(X), X n x k
            return tr ? key_of(mat, l, r) : key_of(mat, r, l);
        };
        for (int64_t j = 0; j < tn; ++j) {
            for (int64_t i = 0; i < tn; ++i) {
                if (lower ? (i < j) : (i > j)) continue;
                const bool dg = (i == j);
                int keyC = key_of(mc, i, j);
                int64_t mt = std::min(T, n - i * T), nt = std::min(T, n - j * T);
                if (scale_only) {
                    Task t;
                    t.gpu = owner_tri(i, j, lower, tn);
                    t.op = XK_OP_SCALE;
                    t.tri = dg ? tri : 0;
                    t.out_key = keyC;
                    if (c.beta != 0.0 || dg) t.in.push_back({keyC, V.get(keyC), 2});
                    t.out_ver = V.bump(keyC);
                    t.beta = c.beta;
                    t.tk = -1;
                    t.i = i; t.j = j;
                    t.m = mt; t.n = nt;
                    t.flops = mt * nt;
                    int64_t sk[5] = {0, (i + j) % tmod, i, j, 0};
                    std::copy(sk, sk + 5, t.skey);
                    tasks.push_back(t);
                    continue;
                }
                bool first = true;
                // diagonal tiles are always read in place (reading R5), off-diagonal ones defer beta
                const bool defer = ms >= 0 && !dg && defer_beta(keyC);
                const int keyS = defer ? key_of(ms, i, j) : -1;
                int64_t pos = 0;
                for (int64_t l = 0; l < tkn; ++l) {
                    int64_t kt = std::min(T, k - l * T);
                    for (int s = 0; s < (two ? 2 : 1); ++s, ++pos) {
                        // SYRK: op(A)_i op(A)_j^T.  SYR2K: s=0 op(A)_i op(B)_j^T, s=1 op(B)_i op(A)_j^T
                        int xa = (two && s == 1) ? mb : ma, xb = (two && s == 0) ? mb : ma;
                        int keyA = opnd(xa, i, l), keyB = opnd(xb, j, l);
                        Task t;
                        t.gpu = owner_tri(i, j, lower, tn);
                        t.op = dg ? XK_OP_GEMM_TRI : XK_OP_GEMM;
                        t.tri = dg ? tri : 0;
                        t.out_key = keyC;
                        t.in.push_back({keyA, V.get(keyA), xa == ma ? 0 : 1});
                        t.in.push_back({keyB, V.get(keyB), xb == ma ? 0 : 1});
                        if (!first || (c.beta != 0.0 && !defer) || dg) t.in.push_back({keyC, V.get(keyC), 2});
                        if (defer && pos == nchain - 1) {
                            t.in.push_back({keyS, V.get(keyS), 2});
                            t.keyC2 = keyS;
                            t.beta2 = c.beta;
                        }
                        t.out_ver = V.bump(keyC);
                        t.keyA = keyA;
                        t.keyB = keyB;
                        t.ta = tr ? 'T' : 'N';  // op(A) tile = X(i,l) or X(l,i)^T
                        t.tb = tr ? 'N' : 'T';  // op(B) tile = X(j,l)^T or X(l,j)
                        t.alpha = c.alpha;
                        t.beta = first ? (defer ? 0.0 : c.beta) : 1.0;
                        t.tk = l;
                        t.i = i; t.j = j;
                        t.m = mt; t.n = nt; t.k = kt;
                        t.flops = dg ? kt * nt * (nt + 1) : 2 * mt * nt * kt;
                        // staggered chains (reading Q12'), as for DGEMM
                        int64_t sk[5] = {2 * (l + (i + j) % tkn) + s, (i + j + l) % tmod, i, j, 0};
                        std::copy(sk, sk + 5, t.skey);
                        tasks.push_back(t);
                        first = false;
                    }
                }
            }
        }
        if (ms >= 0 && !fits(tasks)) {
            drop_shadow(ms);
            ms = -1;
            continue;
        }
        break;
    }
    int rc = run_tasks(tasks, c.sync != 0, out, err);
    drop_shadow(ms);
    return rc;
}

// DSYMM (PLASMA pdsymm): C(i,j) k-chains over sym(A); the diagonal tile of A is used
// symmetrically expanded from its uplo triangle (SYMM_DIAG), off-diagonal tiles are read
// from the uplo triangle, transposed when they lie in the other one.
int Planner::plan_symm(const xk_call_t &c, std::vector<Rec> &out, std::string &err) {
    const int64_t m = c.m, n = c.n, T = flags_.T;
    const bool left = up(c.side) == 'L', lower = up(c.uplo) == 'L';
    if (m == 0 || n == 0 || (c.alpha == 0.0 && c.beta == 1.0)) return XK_OK;
    const bool scale_only = (c.alpha == 0.0);
    const int64_t ka = left ? m : n;
    int mc = find_or_add_matrix(c.C, (int64_t)c.ldc, m, n, err);
    if (mc < 0) return XK_ERR_UNSUPPORTED;
    int ma = -1, mb = -1;
    if (!scale_only) {
        ma = find_or_add_matrix(c.A, (int64_t)c.lda, ka, ka, err);
        if (ma < 0) return XK_ERR_UNSUPPORTED;
        mb = find_or_add_matrix(c.B, (int64_t)c.ldb, m, n, err);
        if (mb < 0) return XK_ERR_UNSUPPORTED;
    }
    const int64_t tm = cdiv(m, T), tn = cdiv(n, T), tl = cdiv(ka, T);
    const int64_t tmod = std::max<int64_t>(1, std::max(tm, tn));
    int ms = (!scale_only && c.beta != 0.0 && tl >= 2) ? add_shadow(mc) : -1;
    std::vector<Task> tasks;
    for (;;) {  // with the shadow if it fits (fits()), else without
        Versions V;
        V.e = &entries_;
        tasks.clear();
        for (int64_t j = 0; j < tn; ++j) {
            for (int64_t i = 0; i < tm; ++i) {
                int keyC = key_of(mc, i, j);
                int64_t mt = std::min(T, m - i * T), nt = std::min(T, n - j * T);
                if (scale_only) {
                    Task t;
                    t.gpu = owner(i, j);
                    t.op = XK_OP_SCALE;
                    t.out_key = keyC;
                    if (c.beta != 0.0) t.in.push_back({keyC, V.get(keyC), 2});
                    t.out_ver = V.bump(keyC);
                    t.beta = c.beta;
                    t.tk = -1;
                    t.i = i; t.j = j;
                    t.m = mt; t.n = nt;
                    t.flops = mt * nt;
                    int64_t sk[5] = {0, (i + j) % tmod, i, j, 0};
                    std::copy(sk, sk + 5, t.skey);
                    tasks.push_back(t);
                    continue;
                }
                // beta deferral when the chain's last task is a GEMM (SYMM_DIAG reads C in place)
                const bool last_diag = left ? (i == tl - 1) : (j == tl - 1);
                const bool defer = ms >= 0 && !last_diag && defer_beta(keyC);
                const int keyS = defer ? key_of(ms, i, j) : -1;
                for (int64_t l = 0; l < tl; ++l) {
                    int64_t kt = std::min(T, ka - l * T);
                    // sym(A) tile (r, q): stored (r, q) if it lies in the uplo triangle, else (q, r)^T
                    int64_t r = left ? i : l, q = left ? l : j;
                    bool in_tri = lower ? (r >= q) : (r <= q);
                    int keyAt = in_tri ? key_of(ma, r, q) : key_of(ma, q, r);
                    int keyBt = left ? key_of(mb, l, j) : key_of(mb, i, l);
                    Task t;
                    t.gpu = owner(i, j);
                    t.out_key = keyC;
                    t.side = left ? 'L' : 'R';
                    t.uplo = lower ? 'L' : 'U';
                    if (r == q) {
                        t.op = XK_OP_SYMM_DIAG;
                        t.keyA = keyAt;
                        t.keyB = keyBt;
                        t.in.push_back({keyAt, V.get(keyAt), 0});
                        t.in.push_back({keyBt, V.get(keyBt), 1});
                    } else if (left) {
                        t.op = XK_OP_GEMM;
                        t.keyA = keyAt;
                        t.keyB = keyBt;
                        t.ta = in_tri ? 'N' : 'T';
                        t.tb = 'N';
                        t.in.push_back({keyAt, V.get(keyAt), 0});
                        t.in.push_back({keyBt, V.get(keyBt), 1});
                    } else {
                        t.op = XK_OP_GEMM;  // C(i,j) += B(i,l) * sym(A)(l,j)
                        t.keyA = keyBt;
                        t.keyB = keyAt;
                        t.ta = 'N';
                        t.tb = in_tri ? 'N' : 'T';
                        t.in.push_back({keyBt, V.get(keyBt), 1});
                        t.in.push_back({keyAt, V.get(keyAt), 0});
                    }
                    if (l > 0 || (c.beta != 0.0 && !defer)) t.in.push_back({keyC, V.get(keyC), 2});
                    if (defer && l == tl - 1) {
                        t.in.push_back({keyS, V.get(keyS), 2});
                        t.keyC2 = keyS;
                        t.beta2 = c.beta;
                    }
                    t.out_ver = V.bump(keyC);
                    t.alpha = c.alpha;
                    t.beta = (l == 0) ? (defer ? 0.0 : c.beta) : 1.0;
                    t.tk = l;
                    t.i = i; t.j = j;
                    t.m = mt; t.n = nt; t.k = kt;
                    t.flops = 2 * mt * nt * kt;
                    // staggered chains (reading Q12'), as for DGEMM
                    int64_t sk[5] = {l + (i + j) % tl, (i + j + l) % tmod, i, j, 0};
                    std::copy(sk, sk + 5, t.skey);
                    tasks.push_back(t);
                }
            }
        }
        if (ms >= 0 && !fits(tasks)) {
            drop_shadow(ms);
            ms = -1;
            continue;
        }
        break;
    }
    int rc = run_tasks(tasks, c.sync != 0, out, err);
    drop_shadow(ms);
    return rc;
}

// DTRMM / DTRSM (PLASMA pdtrmm / pdtrsm) on the output B (passed as C).  op(A) is
// effectively lower iff (uplo == 'L') != (transA == 'T').  TRSM walks k in the solve
// direction: diagonal solve of row (col) k, then GEMM updates of the remaining rows (cols)
// with the solved tiles -- GPU-produced tiles are read by peers (the topology heuristic's
// native case inside one call).  TRMM walks rows (cols) so that every GEMM reads tiles of
// B that are still unmodified (WAR on the in-place update is enforced by the planner).
int Planner::plan_trxm(const xk_call_t &c, bool solve, std::vector<Rec> &out, std::string &err) {
    const int64_t m = c.m, n = c.n, T = flags_.T;
    const bool left = up(c.side) == 'L', lower = up(c.uplo) == 'L', tr = is_t(c.transA);
    const bool elow = (lower != tr);
    if (m == 0 || n == 0) return XK_OK;
    const int64_t ka = left ? m : n;
    int mc = find_or_add_matrix(c.C, (int64_t)c.ldc, m, n, err);
    if (mc < 0) return XK_ERR_UNSUPPORTED;
    const int64_t tm = cdiv(m, T), tn = cdiv(n, T), tk = cdiv(ka, T);
    const int64_t tmod = std::max<int64_t>(1, std::max(tm, tn));
    Versions V;
    V.e = &entries_;
    std::vector<Task> tasks;
    if (c.alpha == 0.0) {  // B <- 0, A not referenced
        for (int64_t j = 0; j < tn; ++j)
            for (int64_t i = 0; i < tm; ++i) {
                int keyC = key_of(mc, i, j);
                Task t;
                t.gpu = owner_trxm(i, j, left, solve);
                t.op = XK_OP_SCALE;
                t.out_key = keyC;
                t.out_ver = V.bump(keyC);
                t.beta = 0.0;
                t.tk = -1;
                t.i = i; t.j = j;
                t.m = std::min(T, m - i * T);
                t.n = std::min(T, n - j * T);
                t.flops = t.m * t.n;
                int64_t sk[5] = {0, (i + j) % tmod, i, j, 0};
                std::copy(sk, sk + 5, t.skey);
                tasks.push_back(t);
            }
        return run_tasks(tasks, c.sync != 0, out, err);
    }
    int ma = find_or_add_matrix(c.A, (int64_t)c.lda, ka, ka, err);
    if (ma < 0) return XK_ERR_UNSUPPORTED;
    auto opA = [&](int64_t r, int64_t q) { return tr ? key_of(ma, q, r) : key_of(ma, r, q); };
    const char tA = tr ? 'T' : 'N';
    // k order: forward when (left & lower) or (right & upper) for TRSM; TRMM the reverse
    const bool fwd = solve ? (left == elow) : (left != elow);
    const int64_t nsteps = tk;
    const int64_t other = left ? tn : tm;  // tiles along the untouched dimension
    // update window (reading R10) only when B has to come from the host: with every tile
    // of B already current on a GPU (data-on-device, composition) PCIe does not bind and the
    // plain right-looking order (window = every step) keeps more updates in flight
    bool b_on_gpus = true;
    for (int64_t j = 0; j < tn && b_on_gpus; ++j)
        for (int64_t i = 0; i < tm && b_on_gpus; ++i) {
            const Entry &e = entries_[key_of(mc, i, j)];
            bool cur = false;
            for (const NodeCopy &g : e.gpu) cur = cur || (g.present && g.ver == e.ver);
            b_on_gpus = cur;
        }
    const int64_t Dw = b_on_gpus ? nsteps : 2 * (left ? std::min(flags_.P, flags_.Q) : std::max(flags_.P, flags_.Q));
    // executor batch cap (reading R19): the R10 window turns a TRSM step's catch-up updates
    // into per-tile chains, and TRMM's contributions are per-tile chains, so consecutive
    // 16-task batches would depend on each other and could not overlap on the kernel streams
    batch_hint_ = solve ? (b_on_gpus ? 0 : 4) : 8;
    // TRMM from the host (reading R15): every step reads B's input tiles from a
    // per-call shadow, so no GEMM reads a tile the sweep overwrites and the sweep runs in the
    // solve direction (top-down for left/lower): step s needs one new row (column) of B
    // instead of the in-place order's all of B during step 0.  The diagonal multiply copies
    // its shadow tile into the output tile first (device-to-device); B crosses PCIe once.
    // The shadow is read from the host once per tile (host_once): a peer's later host read
    // could otherwise race the write-back of the output tile sharing its host memory.
    bool sh_ok = !solve && tk >= 2;
    for (int64_t j = 0; j < tn && sh_ok; ++j)
        for (int64_t i = 0; i < tm && sh_ok; ++i) sh_ok = defer_beta(key_of(mc, i, j));
    int ms = sh_ok ? add_shadow(mc) : -1;
    if (ms >= 0) mats_[ms].host_once = true;
    for (;;) {  // with the shadow if it fits (fits()), else in place
        V.cur.clear();
        tasks.clear();
        const bool sweep_fwd = ms >= 0 ? !fwd : fwd;
        for (int64_t s = 0; s < nsteps; ++s) {
            const int64_t kx = sweep_fwd ? s : nsteps - 1 - s;  // diagonal tile index of this step
            const double a_s = solve ? ((s == 0) ? c.alpha : 1.0) : c.alpha;
            for (int64_t o = 0; o < other; ++o) {
                const int64_t bi = left ? kx : o, bj = left ? o : kx;
                int keyD = opA(kx, kx), keyO = key_of(mc, bi, bj);
                const int64_t mt = std::min(T, m - bi * T), nt = std::min(T, n - bj * T);
                // diagonal task on B(kx, o) (left) / B(o, kx) (right)
                Task t;
                t.gpu = owner_trxm(bi, bj, left, solve);
                t.op = solve ? XK_OP_TRSM_DIAG : XK_OP_TRMM_DIAG;
                t.out_key = keyO;
                t.keyA = keyD;
                t.in.push_back({keyD, V.get(keyD), 0});
                if (ms >= 0) {
                    const int keyS = key_of(ms, bi, bj);
                    t.in.push_back({keyS, V.get(keyS), 2});
                    t.keyC2 = keyS;  // copied into the output tile, then multiplied in place
                } else {
                    t.in.push_back({keyO, V.get(keyO), 2});
                }
                t.out_ver = V.bump(keyO);
                t.ta = tA;
                t.side = left ? 'L' : 'R';
                t.uplo = lower ? 'L' : 'U';
                t.diag = up(c.diag);
                t.alpha = a_s;
                t.tk = s;
                t.i = bi; t.j = bj;
                t.m = mt; t.n = nt; t.k = left ? mt : nt;
                t.flops = left ? mt * mt * nt : mt * nt * nt;
                int64_t sk[5] = {s, 0, (bi + bj + s) % tmod, bi, bj};
                std::copy(sk, sk + 5, t.skey);
                tasks.push_back(t);
                // TRMM: this tile's remaining contributions (sources still unmodified)
                if (!solve) {
                    // contributions nearest the diagonal first (reading R9): the one that reads
                    // the tile the next step overwrites comes first, so that step's diagonal
                    // multiply does not wait for this step's whole chain (WAR)
                    int64_t ph = 1;
                    for (int64_t dq = 1; dq < tk; ++dq) {
                        const bool below = left ? elow : !elow;  // contributing q lie below kx
                        const int64_t q = below ? kx - dq : kx + dq;
                        if (q < 0 || q >= tk) break;
                        const int mb = ms >= 0 ? ms : mc;  // B's input tiles (shadow: R15)
                        int keyA_ = left ? opA(kx, q) : key_of(mb, bi, q);
                        int keyB_ = left ? key_of(mb, q, bj) : opA(q, kx);
                        const int64_t kt = std::min(T, ka - q * T);
                        Task g;
                        g.gpu = owner_trxm(bi, bj, left, solve);
                        g.op = XK_OP_GEMM;
                        g.out_key = keyO;
                        g.keyA = keyA_;
                        g.keyB = keyB_;
                        g.ta = left ? tA : 'N';
                        g.tb = left ? 'N' : tA;
                        g.in.push_back({keyA_, V.get(keyA_), left ? 0 : 2});
                        g.in.push_back({keyB_, V.get(keyB_), left ? 2 : 0});
                        g.in.push_back({keyO, V.get(keyO), 2});
                        g.out_ver = V.bump(keyO);
                        g.alpha = c.alpha;
                        g.beta = 1.0;
                        g.tk = s;
                        g.i = bi; g.j = bj;
                        g.m = mt; g.n = nt; g.k = kt;
                        g.flops = 2 * mt * nt * kt;
                        int64_t sk2[5] = {s, ph++, (bi + bj + s) % tmod, bi, bj};
                        std::copy(sk2, sk2 + 5, g.skey);
                        tasks.push_back(g);
                    }
                }
            }
            if (!solve) continue;
            // TRSM: update the rows (cols) still to be solved with the solved tiles of step s
            for (int64_t r = 0; r < tk; ++r) {
                const bool later = fwd ? r > kx : r < kx;
                if (!later) continue;
                for (int64_t o = 0; o < other; ++o) {
                    const int64_t bi = left ? r : o, bj = left ? o : r;
                    int keyO = key_of(mc, bi, bj);
                    int keyA_ = left ? opA(r, kx) : key_of(mc, bi, kx);
                    int keyB_ = left ? key_of(mc, kx, bj) : opA(kx, r);
                    const int64_t mt = std::min(T, m - bi * T), nt = std::min(T, n - bj * T);
                    const int64_t kt = std::min(T, ka - kx * T);
                    Task g;
                    g.gpu = owner_trxm(bi, bj, left, solve);
                    g.op = XK_OP_GEMM;
                    g.out_key = keyO;
                    g.keyA = keyA_;
                    g.keyB = keyB_;
                    g.ta = left ? tA : 'N';
                    g.tb = left ? 'N' : tA;
                    g.in.push_back({keyA_, V.get(keyA_), left ? 0 : 2});
                    g.in.push_back({keyB_, V.get(keyB_), left ? 2 : 0});
                    g.in.push_back({keyO, V.get(keyO), 2});
                    g.out_ver = V.bump(keyO);
                    g.alpha = -1.0;
                    g.beta = a_s;
                    g.tk = s;
                    g.i = bi; g.j = bj;
                    g.m = mt; g.n = nt; g.k = kt;
                    g.flops = 2 * mt * nt * kt;
                    // lookahead (reading R9): the row (col) the next step solves is updated first,
                    // so its diagonal solve can run while the other updates of this step proceed.
                    // Update window (reading R10): the row solved at step sr is updated by step s
                    // at time u = max(s, sr - D), D = 2 x the grid extent along the solved
                    // dimension; within a time, rows nearest the front first, then s ascending
                    // (every tile's chain keeps its order: results are those of right-looking)
                    const int64_t sr = fwd ? r : nsteps - 1 - r;
                    const int64_t u = std::max<int64_t>(s, sr - Dw);
                    const int64_t ph = (sr == s + 1) ? 1 : 2;
                    int64_t sk[5] = {u, ph, sr * nsteps + s, (bi + bj + s) % tmod, o};
                    std::copy(sk, sk + 5, g.skey);
                    tasks.push_back(g);
                }
            }
        }
        if (ms >= 0 && !fits(tasks)) {
            drop_shadow(ms);
            ms = -1;
            continue;
        }
        break;
    }
    int rc = run_tasks(tasks, c.sync != 0, out, err);
    drop_shadow(ms);
    return rc;
}

bool Planner::view_tiles(uint64_t base, int64_t m, int64_t n, int64_t ld, int *mat, int64_t *r0,
                         int64_t *c0) const {
    for (size_t i = 0; i < mats_.size(); ++i) {
        const Matrix &M = mats_[i];
        if (M.ld != ld || M.ld < 0 || M.shadow) continue;
        if (base < M.base) continue;
        uint64_t off = (base - M.base) / 8;
        int64_t rr = (int64_t)(off % (uint64_t)ld), cc = (int64_t)(off / (uint64_t)ld);
        if (rr < M.rows && cc < M.cols) {
            *mat = (int)i;
            *r0 = rr;
            *c0 = cc;
            (void)m; (void)n;
            return true;
        }
    }
    return false;
}

// step 10: partial coherence writes back only the stale tile intersections;
// prefetch (data-on-device) loads tiles onto their owner GPUs.
int Planner::plan_coherent(const xk_call_t &c, std::vector<Rec> &out, std::string &err,
                           bool prefetch) {
    const int64_t T = flags_.T;
    if (c.m <= 0 || c.n <= 0) return XK_OK;
    int mat;
    int64_t r0, c0;
    if (prefetch) {
        mat = find_or_add_matrix(c.C, (int64_t)c.ldc, c.m, c.n, err);
        if (mat < 0) return XK_ERR_UNSUPPORTED;
        for (int64_t bj = 0; bj < cdiv(c.n, T); ++bj)
            for (int64_t bi = 0; bi < cdiv(c.m, T); ++bi) {
                int key = key_of(mat, bi, bj);
                Entry &e = entries_[key];
                // prefetch: the owner-computes map; distribute: the caller's block-cyclic grid
                int d = owner(bi, bj);
                if (c.routine == XK_ROUTINE_DISTRIBUTE)
                    d = (int)(((bi / c.mb) % c.grid_p) * c.grid_q + ((bj / c.nb) % c.grid_q));
                if (e.gpu[d].present && e.gpu[d].ver == e.ver) continue;
                if (!emit_copy(key, e.ver, d, 0, 2, out)) {
                    err = "prefetch: no valid copy of a tile";
                    return XK_ERR_INTERNAL;
                }
            }
        return XK_OK;
    }
    if (!view_tiles(c.C, c.m, c.n, (int64_t)c.ldc, &mat, &r0, &c0)) return XK_OK;  // never cached
    const Matrix &M = mats_[mat];
    int64_t rend = std::min(M.rows, r0 + c.m), cend = std::min(M.cols, c0 + c.n);
    // write-backs go out in the (virtual) completion order of their tiles, so the FIFO D2H
    // stream is never held by a tile whose chain ends late (ties: column-major tile order)
    struct WB {
        int64_t t_done;
        int key, src;
        int64_t r0, c0, rows, cols;
    };
    std::vector<WB> wb;
    for (int64_t bj = c0 / T; bj * T < cend; ++bj) {
        for (int64_t bi = r0 / T; bi * T < rend; ++bi) {
            auto it = keymap_.find(tile_key(mat, bi, bj));
            if (it == keymap_.end()) continue;
            Entry &e = entries_[it->second];
            if (e.host.present && e.host.ver == e.ver) continue;  // host already valid
            int src = -1;
            for (int g = 0; g < topo_.G; ++g) {
                const NodeCopy &cp = e.gpu[g];
                if (!cp.present || cp.ver != e.ver) continue;
                if (src < 0 || cp.t_done < e.gpu[src].t_done) src = g;
            }
            if (src < 0) {
                err = "coherence: no valid copy of a stale tile";
                return XK_ERR_INTERNAL;
            }
            int64_t tr0 = std::max(r0, bi * T) - bi * T, tc0 = std::max(c0, bj * T) - bj * T;
            int64_t tr1 = std::min(rend, bi * T + e.rows) - bi * T;
            int64_t tc1 = std::min(cend, bj * T + e.cols) - bj * T;
            if (tr1 <= tr0 || tc1 <= tc0) continue;
            wb.push_back({e.gpu[src].t_done, it->second, src, tr0, tc0, tr1 - tr0, tc1 - tc0});
        }
    }
    std::stable_sort(wb.begin(), wb.end(), [](const WB &a, const WB &b) { return a.t_done < b.t_done; });
    for (const WB &w : wb) {
        const Entry &e = entries_[w.key];
        emit_d2h(w.key, w.src, w.r0, w.c0, w.rows, w.cols, w.t_done, e.gpu[w.src].producer, 2, out);
    }
    return XK_OK;
}

void Planner::full_sync() {
    for (auto &e : entries_) {
        e.host.t_done = 0;
        e.host.producer = -1;
        for (auto &g : e.gpu) {
            g.t_done = 0;
            g.producer = -1;
        }
    }
    std::fill(link_free_.begin(), link_free_.end(), 0);
    std::fill(gpu_free_.begin(), gpu_free_.end(), 0);
    for (auto &h : ends_) h.clear();
}

void Planner::invalidate(uint64_t base, int64_t m, int64_t n, int64_t ld) {
    int mat;
    int64_t r0, c0;
    if (m <= 0 || n <= 0) return;
    if (!view_tiles(base, m, n, ld, &mat, &r0, &c0)) return;
    const int64_t T = flags_.T;
    const Matrix &M = mats_[mat];
    int64_t rend = std::min(M.rows, r0 + m), cend = std::min(M.cols, c0 + n);
    for (auto &kv : keymap_) {
        Entry &e = entries_[kv.second];
        if (e.mat != mat) continue;
        if (e.bi * T >= rend || e.bi * T + e.rows <= r0) continue;
        if (e.bj * T >= cend || e.bj * T + e.cols <= c0) continue;
        for (auto &g : e.gpu) g.present = false;
        // the host array is the valid copy from now on (drop-in semantics: whatever the
        // caller holds there is used next; stale tiles are not written back)
        e.host.present = true;
        e.host.ver = e.ver;
        e.host.t_done = 0;
        e.host.producer = -1;
        e.host.depth = 0;
    }
}

// Drop the GPU copies of a view's tiles whose host copy is current.  A tile whose only
// current copy is on a GPU (the output of an earlier async call, not yet made coherent) is
// kept as it is: dropping it would lose the result (xk_memory_coherent_sync writes it back
// later), and marking the stale host data valid would hand it to the next reader.
void Planner::release(uint64_t base, int64_t m, int64_t n, int64_t ld) {
    int mat;
    int64_t r0, c0;
    if (m <= 0 || n <= 0) return;
    if (!view_tiles(base, m, n, ld, &mat, &r0, &c0)) return;
    const int64_t T = flags_.T;
    const Matrix &M = mats_[mat];
    int64_t rend = std::min(M.rows, r0 + m), cend = std::min(M.cols, c0 + n);
    for (auto &kv : keymap_) {
        Entry &e = entries_[kv.second];
        if (e.mat != mat) continue;
        if (e.bi * T >= rend || e.bi * T + e.rows <= r0) continue;
        if (e.bj * T >= cend || e.bj * T + e.cols <= c0) continue;
        if (!(e.host.present && e.host.ver == e.ver)) continue;  // GPU-dirty: keep
        for (auto &g : e.gpu) g.present = false;
    }
}

// After a synchronous routine: a full sync point, then the operands' device copies are
// dropped (sync routines are drop-in) -- except those of tiles whose current
// version exists only on a GPU (see release()).
void Planner::finish_call(const xk_call_t &c) {
    full_sync();
    const bool ta = is_t(c.transA), tb = is_t(c.transB);
    const bool left = up(c.side) == 'L';
    switch (c.routine) {
    case XK_ROUTINE_DGEMM:
        if (c.alpha != 0.0 && c.k > 0) {
            release(c.A, ta ? c.k : c.m, ta ? c.m : c.k, (int64_t)c.lda);
            release(c.B, tb ? c.n : c.k, tb ? c.k : c.n, (int64_t)c.ldb);
        }
        release(c.C, c.m, c.n, (int64_t)c.ldc);
        break;
    case XK_ROUTINE_DSYRK:
    case XK_ROUTINE_DSYR2K:
        if (c.alpha != 0.0 && c.k > 0) {
            release(c.A, ta ? c.k : c.n, ta ? c.n : c.k, (int64_t)c.lda);
            if (c.routine == XK_ROUTINE_DSYR2K)
                release(c.B, ta ? c.k : c.n, ta ? c.n : c.k, (int64_t)c.ldb);
        }
        release(c.C, c.n, c.n, (int64_t)c.ldc);
        break;
    case XK_ROUTINE_DSYMM:
        if (c.alpha != 0.0) {
            const int64_t ka = left ? c.m : c.n;
            release(c.A, ka, ka, (int64_t)c.lda);
            release(c.B, c.m, c.n, (int64_t)c.ldb);
        }
        release(c.C, c.m, c.n, (int64_t)c.ldc);
        break;
    default: {  // TRMM / TRSM
        const int64_t ka = left ? c.m : c.n;
        if (c.alpha != 0.0) release(c.A, ka, ka, (int64_t)c.lda);
        release(c.C, c.m, c.n, (int64_t)c.ldc);
    }
    }
}

void Planner::emit(const Rec &R, std::vector<Rec> &out) {
    if (!sink_) {
        out.push_back(R);
        return;
    }
    if (sink_rc_) return;  // an earlier record failed to issue: stop
    sink_rc_ = (*sink_)(R);
}

int Planner::plan(const xk_call_t &c, std::vector<Rec> &out, std::string &err, const Sink *sink) {
    sink_ = sink;
    sink_rc_ = 0;
    batch_hint_ = 0;
    int rc = plan_impl(c, out, err);
    sink_ = nullptr;
    if (rc == XK_OK && sink_rc_) rc = sink_rc_;
    return rc;
}

int Planner::plan_impl(const xk_call_t &c, std::vector<Rec> &out, std::string &err) {
    int rc;
    switch (c.routine) {
    case XK_ROUTINE_DGEMM:
        rc = plan_gemm(c, out, err);
        break;
    case XK_ROUTINE_DSYRK:
        rc = plan_syrk(c, false, out, err);
        break;
    case XK_ROUTINE_DSYR2K:
        rc = plan_syrk(c, true, out, err);
        break;
    case XK_ROUTINE_DSYMM:
        rc = plan_symm(c, out, err);
        break;
    case XK_ROUTINE_DTRMM:
        rc = plan_trxm(c, false, out, err);
        break;
    case XK_ROUTINE_DTRSM:
        rc = plan_trxm(c, true, out, err);
        break;
    case XK_ROUTINE_COHERENT:
        return plan_coherent(c, out, err, false);
    case XK_ROUTINE_SYNC:
        full_sync();
        return XK_OK;
    case XK_ROUTINE_INVALIDATE:
        invalidate(c.C, c.m, c.n, (int64_t)c.ldc);
        return XK_OK;
    case XK_ROUTINE_PREFETCH:
        return plan_coherent(c, out, err, true);
    case XK_ROUTINE_DISTRIBUTE:
        if (c.grid_p < 1 || c.grid_q < 1 || (int64_t)c.grid_p * c.grid_q > topo_.G || c.mb < 1 || c.nb < 1) {
            err = "distribute: need 1 <= P*Q <= ngpus and block sizes >= 1";
            return XK_ERR_CONFIG;
        }
        return plan_coherent(c, out, err, true);
    default:
        err = "unknown routine";
        return XK_ERR_CONFIG;
    }
    if (rc) return rc;
    // a quick return (BLAS: nothing to do) is not a synchronisation point
    bool quick;
    switch (c.routine) {
    case XK_ROUTINE_DGEMM:
        quick = c.m == 0 || c.n == 0 || ((c.alpha == 0.0 || c.k == 0) && c.beta == 1.0);
        break;
    case XK_ROUTINE_DSYRK:
    case XK_ROUTINE_DSYR2K:
        quick = c.n == 0 || ((c.alpha == 0.0 || c.k == 0) && c.beta == 1.0);
        break;
    case XK_ROUTINE_DSYMM:
        quick = c.m == 0 || c.n == 0 || (c.alpha == 0.0 && c.beta == 1.0);
        break;
    default:
        quick = c.m == 0 || c.n == 0;
    }
    if (c.sync && !quick) finish_call(c);
    return XK_OK;
}

}  // namespace xk
