// api.cpp -- the C ABI of libxk.so (include/xk.h): argument checking with BLAS XERBLA
// numbering, quick returns, then one planned call on the runtime.
#include <cctype>
#include <cstdlib>
#include <cstring>
#include <memory>
#include <string>

#include "api/common.h"
#include "exec/runtime.h"
#include "xk.h"

namespace xk {
static std::unique_ptr<Runtime> g_rt;
Runtime *runtime() { return g_rt.get(); }
}  // namespace xk

using xk::runtime;

namespace {

char up(char c) { return (char)std::toupper((unsigned char)c); }
bool ok_trans(char t) { t = up(t); return t == 'N' || t == 'T' || t == 'C'; }
bool is_trans(char t) { t = up(t); return t == 'T' || t == 'C'; }
bool ok_uplo(char u) { u = up(u); return u == 'L' || u == 'U'; }
bool ok_side(char s) { s = up(s); return s == 'L' || s == 'R'; }
bool ok_diag(char d) { d = up(d); return d == 'N' || d == 'U'; }
int64_t imax(int64_t a, int64_t b) { return a > b ? a : b; }

int env_int(const char *name, int dflt) {
    const char *v = std::getenv(name);
    return (v && *v) ? std::atoi(v) : dflt;
}

int need_init() {
    xk::set_error("xk_init() has not been called");
    return XK_ERR_NOT_INITIALIZED;
}

int gemm_check(char ta, char tb, int64_t m, int64_t n, int64_t k, int64_t lda, int64_t ldb,
               int64_t ldc) {
    if (!ok_trans(ta)) return -1;
    if (!ok_trans(tb)) return -2;
    if (m < 0) return -3;
    if (n < 0) return -4;
    if (k < 0) return -5;
    if (lda < imax(1, is_trans(ta) ? k : m)) return -8;
    if (ldb < imax(1, is_trans(tb) ? n : k)) return -10;
    if (ldc < imax(1, m)) return -13;
    return 0;
}

int gemm_impl(char transA, char transB, int64_t m, int64_t n, int64_t k, double alpha,
              const double *A, int64_t lda, const double *B, int64_t ldb, double beta, double *C,
              int64_t ldc, bool sync) {
    int info = gemm_check(transA, transB, m, n, k, lda, ldb, ldc);
    if (info) return info;
    if (m == 0 || n == 0 || ((alpha == 0.0 || k == 0) && beta == 1.0)) return XK_OK;
    xk::Runtime *rt = runtime();
    if (!rt) return need_init();
    xk_call_t c{};
    c.routine = XK_ROUTINE_DGEMM;
    c.transA = is_trans(transA) ? 'T' : 'N';
    c.transB = is_trans(transB) ? 'T' : 'N';
    c.uplo = 'L';
    c.side = 'L';
    c.diag = 'N';
    c.m = m;
    c.n = n;
    c.k = k;
    c.alpha = alpha;
    c.beta = beta;
    c.A = (uint64_t)(uintptr_t)A;
    c.lda = (uint64_t)lda;
    c.B = (uint64_t)(uintptr_t)B;
    c.ldb = (uint64_t)ldb;
    c.C = (uint64_t)(uintptr_t)C;
    c.ldc = (uint64_t)ldc;
    c.sync = sync ? 1 : 0;
    return rt->run(c, sync);
}

int view_call(int routine, int64_t m, int64_t n, const double *A, int64_t lda, bool wait) {
    if (m < 0) return -1;
    if (n < 0) return -2;
    if (lda < imax(1, m)) return -4;
    xk::Runtime *rt = runtime();
    if (!rt) return need_init();
    if (m == 0 || n == 0) return XK_OK;
    xk_call_t c{};
    c.routine = routine;
    c.m = m;
    c.n = n;
    c.C = (uint64_t)(uintptr_t)A;
    c.ldc = (uint64_t)lda;
    return rt->run(c, wait);
}


}  // namespace

extern "C" {

void xk_config_default(xk_config_t *cfg) {
    if (!cfg) return;
    std::memset(cfg, 0, sizeof(*cfg));
    cfg->ngpus = env_int("XK_NGPUS", 0);
    const char *t = std::getenv("XK_TILE");
    cfg->tile = (t && *t) ? std::atoll(t) : 2048;
    const char *topo = std::getenv("XK_TOPO");
    cfg->topo = XK_TOPO_RANKED;
    if (topo && !std::strcmp(topo, "unranked")) cfg->topo = XK_TOPO_UNRANKED;
    if (topo && !std::strcmp(topo, "home")) cfg->topo = XK_TOPO_HOME;
    cfg->optimistic = env_int("XK_OPTIMISTIC", 1);
    cfg->window = env_int("XK_WINDOW", 4);
    cfg->kstreams = env_int("XK_KSTREAMS", 2);
    cfg->probe = env_int("XK_PROBE", 1);
    const char *rate = std::getenv("XK_TASK_RATE");  // planner task rate in MFLOP/s (0 = measured)
    cfg->task_rate_mflops = (rate && *rate) ? std::atoll(rate) : 0;
}

int xk_init(const xk_config_t *cfg) {
    xk_config_t c;
    if (cfg) c = *cfg; else xk_config_default(&c);
    if (xk::g_rt) xk_finalize();
    std::unique_ptr<xk::Runtime> rt(new xk::Runtime());
    int rc = rt->init(c);
    if (rc) {
        rt->finalize();
        return rc;
    }
    xk::g_rt = std::move(rt);
    return XK_OK;
}

int xk_finalize(void) {
    if (!xk::g_rt) return XK_OK;
    int rc = xk::g_rt->finalize();
    xk::g_rt.reset();
    return rc;
}

int xk_register(void *p, size_t bytes) {
    if (!runtime()) return need_init();
    return runtime()->register_host(p, bytes);
}

int xk_unregister(void *p) {
    if (!runtime()) return need_init();
    return runtime()->unregister_host(p);
}

int xk_dgemm(char transA, char transB, int64_t m, int64_t n, int64_t k, double alpha,
             const double *A, int64_t lda, const double *B, int64_t ldb, double beta, double *C,
             int64_t ldc) {
    return gemm_impl(transA, transB, m, n, k, alpha, A, lda, B, ldb, beta, C, ldc, true);
}

int xk_dgemm_async(char transA, char transB, int64_t m, int64_t n, int64_t k, double alpha,
                   const double *A, int64_t lda, const double *B, int64_t ldb, double beta,
                   double *C, int64_t ldc) {
    return gemm_impl(transA, transB, m, n, k, alpha, A, lda, B, ldb, beta, C, ldc, false);
}

// ---- other BLAS-3: tile algorithms of PLASMA structure
static int syrk_check(char uplo, char trans, int64_t n, int64_t k, int64_t lda, int64_t ldc) {
    if (!ok_uplo(uplo)) return -1;
    if (!ok_trans(trans)) return -2;
    if (n < 0) return -3;
    if (k < 0) return -4;
    if (lda < imax(1, is_trans(trans) ? k : n)) return -7;
    if (ldc < imax(1, n)) return -10;
    return 0;
}
static int syr2k_check(char uplo, char trans, int64_t n, int64_t k, int64_t lda, int64_t ldb,
                       int64_t ldc) {
    if (!ok_uplo(uplo)) return -1;
    if (!ok_trans(trans)) return -2;
    if (n < 0) return -3;
    if (k < 0) return -4;
    int64_t nr = is_trans(trans) ? k : n;
    if (lda < imax(1, nr)) return -7;
    if (ldb < imax(1, nr)) return -9;
    if (ldc < imax(1, n)) return -12;
    return 0;
}
static int symm_check(char side, char uplo, int64_t m, int64_t n, int64_t lda, int64_t ldb,
                      int64_t ldc) {
    if (!ok_side(side)) return -1;
    if (!ok_uplo(uplo)) return -2;
    if (m < 0) return -3;
    if (n < 0) return -4;
    if (lda < imax(1, up(side) == 'L' ? m : n)) return -7;
    if (ldb < imax(1, m)) return -9;
    if (ldc < imax(1, m)) return -12;
    return 0;
}
static int tr_check(char side, char uplo, char ta, char diag, int64_t m, int64_t n, int64_t lda,
                    int64_t ldb) {
    if (!ok_side(side)) return -1;
    if (!ok_uplo(uplo)) return -2;
    if (!ok_trans(ta)) return -3;
    if (!ok_diag(diag)) return -4;
    if (m < 0) return -5;
    if (n < 0) return -6;
    if (lda < imax(1, up(side) == 'L' ? m : n)) return -9;
    if (ldb < imax(1, m)) return -11;
    return 0;
}

static int run_call(xk_call_t &c, bool sync) {
    xk::Runtime *rt = runtime();
    if (!rt) return need_init();
    c.sync = sync ? 1 : 0;
    return rt->run(c, sync);
}

static int syrk_impl(bool two, char uplo, char trans, int64_t n, int64_t k, double alpha,
                     const double *A, int64_t lda, const double *B, int64_t ldb, double beta,
                     double *C, int64_t ldc, bool sync) {
    int info = two ? syr2k_check(uplo, trans, n, k, lda, ldb, ldc) : syrk_check(uplo, trans, n, k, lda, ldc);
    if (info) return info;
    if (n == 0 || ((alpha == 0.0 || k == 0) && beta == 1.0)) return XK_OK;
    xk_call_t c{};
    c.routine = two ? XK_ROUTINE_DSYR2K : XK_ROUTINE_DSYRK;
    c.uplo = up(uplo);
    c.transA = is_trans(trans) ? 'T' : 'N';
    c.transB = 'N';
    c.side = 'L';
    c.diag = 'N';
    c.m = n;
    c.n = n;
    c.k = k;
    c.alpha = alpha;
    c.beta = beta;
    c.A = (uint64_t)(uintptr_t)A;
    c.lda = (uint64_t)lda;
    c.B = (uint64_t)(uintptr_t)B;
    c.ldb = (uint64_t)(two ? ldb : 1);
    c.C = (uint64_t)(uintptr_t)C;
    c.ldc = (uint64_t)ldc;
    return run_call(c, sync);
}

static int symm_impl(char side, char uplo, int64_t m, int64_t n, double alpha, const double *A,
                     int64_t lda, const double *B, int64_t ldb, double beta, double *C, int64_t ldc,
                     bool sync) {
    int info = symm_check(side, uplo, m, n, lda, ldb, ldc);
    if (info) return info;
    if (m == 0 || n == 0 || (alpha == 0.0 && beta == 1.0)) return XK_OK;
    xk_call_t c{};
    c.routine = XK_ROUTINE_DSYMM;
    c.side = up(side);
    c.uplo = up(uplo);
    c.transA = c.transB = 'N';
    c.diag = 'N';
    c.m = m;
    c.n = n;
    c.k = up(side) == 'L' ? m : n;
    c.alpha = alpha;
    c.beta = beta;
    c.A = (uint64_t)(uintptr_t)A;
    c.lda = (uint64_t)lda;
    c.B = (uint64_t)(uintptr_t)B;
    c.ldb = (uint64_t)ldb;
    c.C = (uint64_t)(uintptr_t)C;
    c.ldc = (uint64_t)ldc;
    return run_call(c, sync);
}

static int trxm_impl(bool solve, char side, char uplo, char transA, char diag, int64_t m, int64_t n,
                     double alpha, const double *A, int64_t lda, double *B, int64_t ldb, bool sync) {
    int info = tr_check(side, uplo, transA, diag, m, n, lda, ldb);
    if (info) return info;
    if (m == 0 || n == 0) return XK_OK;
    xk_call_t c{};
    c.routine = solve ? XK_ROUTINE_DTRSM : XK_ROUTINE_DTRMM;
    c.side = up(side);
    c.uplo = up(uplo);
    c.transA = is_trans(transA) ? 'T' : 'N';
    c.transB = 'N';
    c.diag = up(diag);
    c.m = m;
    c.n = n;
    c.k = up(side) == 'L' ? m : n;
    c.alpha = alpha;
    c.beta = 0.0;
    c.A = (uint64_t)(uintptr_t)A;
    c.lda = (uint64_t)lda;
    c.C = (uint64_t)(uintptr_t)B;  // the output matrix of TRMM/TRSM travels as C (xk.h)
    c.ldc = (uint64_t)ldb;
    return run_call(c, sync);
}

int xk_dsyrk(char uplo, char trans, int64_t n, int64_t k, double alpha, const double *A,
             int64_t lda, double beta, double *C, int64_t ldc) {
    return syrk_impl(false, uplo, trans, n, k, alpha, A, lda, nullptr, 1, beta, C, ldc, true);
}
int xk_dsyrk_async(char uplo, char trans, int64_t n, int64_t k, double alpha, const double *A,
                   int64_t lda, double beta, double *C, int64_t ldc) {
    return syrk_impl(false, uplo, trans, n, k, alpha, A, lda, nullptr, 1, beta, C, ldc, false);
}
int xk_dsyr2k(char uplo, char trans, int64_t n, int64_t k, double alpha, const double *A,
              int64_t lda, const double *B, int64_t ldb, double beta, double *C, int64_t ldc) {
    return syrk_impl(true, uplo, trans, n, k, alpha, A, lda, B, ldb, beta, C, ldc, true);
}
int xk_dsyr2k_async(char uplo, char trans, int64_t n, int64_t k, double alpha, const double *A,
                    int64_t lda, const double *B, int64_t ldb, double beta, double *C, int64_t ldc) {
    return syrk_impl(true, uplo, trans, n, k, alpha, A, lda, B, ldb, beta, C, ldc, false);
}
int xk_dsymm(char side, char uplo, int64_t m, int64_t n, double alpha, const double *A,
             int64_t lda, const double *B, int64_t ldb, double beta, double *C, int64_t ldc) {
    return symm_impl(side, uplo, m, n, alpha, A, lda, B, ldb, beta, C, ldc, true);
}
int xk_dsymm_async(char side, char uplo, int64_t m, int64_t n, double alpha, const double *A,
                   int64_t lda, const double *B, int64_t ldb, double beta, double *C, int64_t ldc) {
    return symm_impl(side, uplo, m, n, alpha, A, lda, B, ldb, beta, C, ldc, false);
}
int xk_dtrmm(char side, char uplo, char transA, char diag, int64_t m, int64_t n, double alpha,
             const double *A, int64_t lda, double *B, int64_t ldb) {
    return trxm_impl(false, side, uplo, transA, diag, m, n, alpha, A, lda, B, ldb, true);
}
int xk_dtrmm_async(char side, char uplo, char transA, char diag, int64_t m, int64_t n, double alpha,
                   const double *A, int64_t lda, double *B, int64_t ldb) {
    return trxm_impl(false, side, uplo, transA, diag, m, n, alpha, A, lda, B, ldb, false);
}
int xk_dtrsm(char side, char uplo, char transA, char diag, int64_t m, int64_t n, double alpha,
             const double *A, int64_t lda, double *B, int64_t ldb) {
    return trxm_impl(true, side, uplo, transA, diag, m, n, alpha, A, lda, B, ldb, true);
}
int xk_dtrsm_async(char side, char uplo, char transA, char diag, int64_t m, int64_t n, double alpha,
                   const double *A, int64_t lda, double *B, int64_t ldb) {
    return trxm_impl(true, side, uplo, transA, diag, m, n, alpha, A, lda, B, ldb, false);
}

// ---- coherence / sync
int xk_memory_coherent_sync(int64_t m, int64_t n, double *A, int64_t lda) {
    return view_call(XK_ROUTINE_COHERENT, m, n, A, lda, true);
}
int xk_memory_coherent_async(int64_t m, int64_t n, double *A, int64_t lda) {
    return view_call(XK_ROUTINE_COHERENT, m, n, A, lda, false);
}
int xk_memory_prefetch_async(int64_t m, int64_t n, const double *A, int64_t lda) {
    return view_call(XK_ROUTINE_PREFETCH, m, n, A, lda, false);
}
int xk_distribute_2dbc_async(int64_t m, int64_t n, const double *A, int64_t lda, int P, int Q,
                             int64_t mb, int64_t nb) {
    if (m < 0) return -1;
    if (n < 0) return -2;
    if (lda < imax(1, m)) return -4;
    if (P < 1) return -5;
    xk::Runtime *rt = runtime();
    if (Q < 1 || (rt && (int64_t)P * Q > rt->topo.G)) return -6;
    if (mb < 1) return -7;
    if (nb < 1) return -8;
    if (!rt) return need_init();
    if (m == 0 || n == 0) return XK_OK;
    xk_call_t c{};
    c.routine = XK_ROUTINE_DISTRIBUTE;
    c.m = m;
    c.n = n;
    c.C = (uint64_t)(uintptr_t)A;
    c.ldc = (uint64_t)lda;
    c.grid_p = P;
    c.grid_q = Q;
    c.mb = mb;
    c.nb = nb;
    return rt->run(c, false);
}
int xk_sync(void) {
    xk::Runtime *rt = runtime();
    if (!rt) return need_init();
    std::lock_guard<std::recursive_mutex> lk(rt->mu);
    int rc = rt->sync_all();
    if (rc) return rc;
    xk_call_t c{};
    c.routine = XK_ROUTINE_SYNC;
    return rt->run(c, false);
}
int xk_memory_invalidate(int64_t m, int64_t n, const double *A, int64_t lda) {
    if (m < 0) return -1;
    if (n < 0) return -2;
    if (lda < imax(1, m)) return -4;
    xk::Runtime *rt = runtime();
    if (!rt) return need_init();
    return rt->invalidate((uint64_t)(uintptr_t)A, m, n, lda);
}

// ---- observability
int xk_get_stats(xk_stats_t *out) {
    xk::Runtime *rt = runtime();
    if (!rt) return need_init();
    if (!out) return XK_ERR_CONFIG;
    std::lock_guard<std::recursive_mutex> lk(rt->mu);
    *out = rt->stats;
    return XK_OK;
}
int xk_reset_stats(void) {
    xk::Runtime *rt = runtime();
    if (!rt) return need_init();
    std::lock_guard<std::recursive_mutex> lk(rt->mu);
    int G = rt->stats.ngpus;
    std::memset(&rt->stats, 0, sizeof(rt->stats));
    rt->stats.ngpus = G;
    return XK_OK;
}
int xk_set_kernel_timing(int on) {
    xk::Runtime *rt = runtime();
    if (!rt) return need_init();
    rt->kernel_timing = on != 0;
    return XK_OK;
}
int xk_trace(const char *path) {
    xk::Runtime *rt = runtime();
    if (!rt) return need_init();
    if (path) return rt->trace_start(path);
    return rt->trace_stop();
}

int xk_get_topology(xk_topo_t *out) {
    xk::Runtime *rt = runtime();
    if (!rt) return need_init();
    if (!out) return XK_ERR_CONFIG;
    std::memset(out, 0, sizeof(*out));
    const int G = rt->topo.G;
    out->ngpus = G;
    for (int s = 0; s <= G; ++s)
        for (int d = 0; d <= G; ++d) out->bw_MBps[s * (G + 1) + d] = rt->topo.bw_at(s, d);
    for (int s = 0; s < G; ++s)
        for (int d = 0; d < G; ++d) out->perf_rank[s * G + d] = rt->perf_rank[(size_t)s * G + d];
    out->task_rate_mflops = rt->topo.rate_mflops;
    for (int q = 0; q < 3; ++q) out->host_all_MBps[q] = rt->host_all_MBps[q];
    out->host_probe_bytes = rt->host_probe_bytes;
    return XK_OK;
}

int xk_probe_host_links(int64_t bytes_per_gpu) {
    xk::Runtime *rt = runtime();
    if (!rt) return need_init();
    if (bytes_per_gpu <= 0) return XK_ERR_CONFIG;
    return rt->probe_host_links(bytes_per_gpu);
}

}  // extern "C"
