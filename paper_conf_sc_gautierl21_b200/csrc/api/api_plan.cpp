// api_plan.cpp -- C ABI of the planner (no GPU needed): plan sessions and xk_plan_dump.
// Used by the CPU tests that compare the planner bit-exactly with tests/planmodel.py.
#include <cstring>
#include <new>
#include <string>
#include <vector>

#include "api/common.h"
#include "plan/plan.h"
#include "xk.h"

struct xk_plan_session {
    xk::Planner *p = nullptr;
};

namespace xk {

bool make_topology(const xk_topo_t *t, Topology *out, std::string &err) {
    if (!t || t->ngpus < 1 || t->ngpus > XK_MAX_GPUS) {
        err = "topology: ngpus out of range";
        return false;
    }
    out->G = t->ngpus;
    const int N = t->ngpus + 1;
    out->bw.assign((size_t)N * N, 0);
    for (int s = 0; s < N; ++s)
        for (int d = 0; d < N; ++d) {
            int64_t v = t->bw_MBps[s * N + d];
            if (v <= 0) {
                err = "topology: bandwidth entries must be > 0 MB/s";
                return false;
            }
            out->bw[(size_t)s * N + d] = v;
        }
    out->rate_mflops = t->task_rate_mflops > 0 ? t->task_rate_mflops : 35000000;
    return true;
}

void default_grid(int G, int *P, int *Q) {
    // reading Q11: P >= Q, near-square (1x1, 2x1, 2x2, 4x2)
    int q = 1;
    for (int c = 1; c * c <= G; ++c)
        if (G % c == 0) q = c;
    *Q = q;
    *P = G / q;
}

bool make_flags(const xk_flags_t *f, int G, Flags *out, std::string &err) {
    Flags F;
    if (f) {
        F.topo = f->topo;
        F.optimistic = f->optimistic;
        F.window = f->window > 0 ? f->window : 4;
        F.T = f->tile > 0 ? f->tile : 2048;
        F.P = f->grid_p;
        F.Q = f->grid_q;
        F.mem_bytes = f->mem_bytes > 0 ? f->mem_bytes : 0;
    }
    if (F.topo < XK_TOPO_RANKED || F.topo > XK_TOPO_HOME) {
        err = "flags: unknown topo mode";
        return false;
    }
    if (F.P <= 0 || F.Q <= 0) default_grid(G, &F.P, &F.Q);
    if (F.P * F.Q != G) {
        err = "flags: grid P*Q must equal the number of GPUs";
        return false;
    }
    *out = F;
    return true;
}

}  // namespace xk

extern "C" {

int xk_plan_session_create(const xk_topo_t *topo, const xk_flags_t *flags, xk_plan_session_t **out) {
    xk::Topology T;
    xk::Flags F;
    std::string err;
    if (!out || !xk::make_topology(topo, &T, err) || !xk::make_flags(flags, T.G, &F, err)) {
        xk::set_error(err.empty() ? "bad arguments" : err);
        return XK_ERR_CONFIG;
    }
    auto *s = new (std::nothrow) xk_plan_session;
    if (!s) return XK_ERR_INTERNAL;
    s->p = new xk::Planner(T, F);
    *out = s;
    return XK_OK;
}

int xk_plan_session_call(xk_plan_session_t *s, const xk_call_t *call, xk_plan_rec_t *out,
                         int64_t cap, int64_t *n_out) {
    if (!s || !call) return XK_ERR_CONFIG;
    std::vector<xk::Rec> recs;
    std::string err;
    int rc = s->p->plan(*call, recs, err);
    if (rc) {
        xk::set_error(err);
        return rc;
    }
    if (n_out) *n_out = (int64_t)recs.size();
    if ((int64_t)recs.size() > cap) return XK_ERR_CAPACITY;
    for (size_t i = 0; i < recs.size(); ++i) out[i] = recs[i].r;
    return XK_OK;
}

void xk_plan_session_destroy(xk_plan_session_t *s) {
    if (!s) return;
    delete s->p;
    delete s;
}

int xk_plan_dump(const xk_call_t *call, const xk_topo_t *topo, const xk_flags_t *flags,
                 xk_plan_rec_t *out, int64_t cap, int64_t *n_out) {
    xk_plan_session_t *s = nullptr;
    int rc = xk_plan_session_create(topo, flags, &s);
    if (rc) return rc;
    rc = xk_plan_session_call(s, call, out, cap, n_out);
    xk_plan_session_destroy(s);
    return rc;
}

}  // extern "C"
