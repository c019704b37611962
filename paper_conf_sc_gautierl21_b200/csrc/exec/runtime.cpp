// runtime.cpp -- executor of plan records (see runtime.h).
//
// Ordering is enforced with CUDA events, never by the virtual-time model: every record
// waits on the events of the records it depends on (plan deps = RAW), and a buffer that is
// overwritten first waits on the reads of its previous contents (WAR) and its previous
// write (WAW).  Records are issued by one host thread in plan order, and every dependency
// names an earlier record, so no cudaStreamWaitEvent is ever issued before the matching
// cudaEventRecord (the issue-order hazard of SURVEY.md §0.1).
#include "exec/runtime.h"

#include <algorithm>
#include <cstdlib>
#include <cstdio>
#include <cstring>
#include <chrono>
#include <thread>

#include "api/common.h"
#include "kernels/kernels.h"

namespace xk {

#define XK_CK(call)                                        \
    do {                                                   \
        cudaError_t _e = (call);                           \
        if (_e != cudaSuccess) return cuda_fail(_e, #call); \
    } while (0)

static inline int64_t round_up(int64_t a, int64_t b) { return (a + b - 1) / b * b; }

int Runtime::cuda_fail(cudaError_t e, const char *what) {
    set_error(std::string(what) + ": " + cudaGetErrorString(e));
    return XK_ERR_CUDA;
}

int Runtime::set_dev(int g) {
    int p = devs_[g].phys;
    if (p != cur_dev_) {
        XK_CK(cudaSetDevice(p));
        cur_dev_ = p;
    }
    return XK_OK;
}

Runtime::~Runtime() {}

int Runtime::init(const xk_config_t &cfg) {
    cfg_ = cfg;
    int ndev = 0;
    cudaError_t e = cudaGetDeviceCount(&ndev);
    if (e != cudaSuccess || ndev == 0) {
        set_error(std::string("no CUDA device: ") + cudaGetErrorString(e));
        return XK_ERR_NO_DEVICE;
    }
    rank_mode_ = cfg.world > 1;
    if (rank_mode_ && (cfg.rank < 0 || cfg.rank >= cfg.world || (cfg.ngpus > 0 && cfg.ngpus != cfg.world))) {
        set_error("config: rank mode needs 0 <= rank < world and ngpus in {0, world}");
        return XK_ERR_CONFIG;
    }
    rank_ = rank_mode_ ? cfg.rank : 0;
    int G = rank_mode_ ? cfg.world : cfg.ngpus > 0 ? cfg.ngpus : ndev;
    if (G > XK_MAX_GPUS) {
        set_error("ngpus > XK_MAX_GPUS");
        return XK_ERR_CONFIG;
    }
    devs_.assign(G, Device());
    for (int g = 0; g < G; ++g) {
        if (rank_mode_ && g != rank_) {  // a peer process's GPU: no streams here
            devs_[g].local = false;
            devs_[g].phys = -1;
            continue;
        }
        int p = cfg.map_devices ? cfg.phys[g] : g % ndev;
        if (p < 0 || p >= ndev) {
            set_error("logical->physical device map out of range");
            return XK_ERR_CONFIG;
        }
        devs_[g].phys = p;
    }
    int ks = cfg.kstreams > 0 ? std::min(cfg.kstreams, kMaxKStreams) : 2;
    cfg_.kstreams = ks;
    {
        const char *dv = getenv("XK_DEFER_D2H");
        defer_d2h_ = !(dv && dv[0] == '0');
        const char *rv = getenv("XK_RAMP");  // grouped launches per batch-size doubling
        ramp_div_ = rv ? std::max(1, atoi(rv)) : ramp_div_;
    }
    nks_ = std::max(ks, 4);  // streams created: batches use the first ks, diagonal ops all
    // peer access between distinct physical devices (NVLink / NVSwitch)
    for (int a = 0; a < G; ++a)
        for (int b = 0; b < G; ++b) {
            int pa = devs_[a].phys, pb = devs_[b].phys;
            if (pa == pb || !devs_[a].local || !devs_[b].local) continue;
            int can = 0;
            XK_CK(cudaDeviceCanAccessPeer(&can, pa, pb));
            if (!can) continue;
            XK_CK(cudaSetDevice(pa));
            cudaError_t pe = cudaDeviceEnablePeerAccess(pb, 0);
            if (pe != cudaSuccess && pe != cudaErrorPeerAccessAlreadyEnabled) return cuda_fail(pe, "cudaDeviceEnablePeerAccess");
            cudaGetLastError();
        }
    for (int g = 0; g < G; ++g) {
        Device &d = devs_[g];
        if (!d.local) continue;
        XK_CK(cudaSetDevice(d.phys));
        XK_CK(cudaStreamCreateWithFlags(&d.h2d, cudaStreamNonBlocking));
        XK_CK(cudaStreamCreateWithFlags(&d.d2h, cudaStreamNonBlocking));
        XK_CK(cudaStreamCreateWithFlags(&d.p2p, cudaStreamNonBlocking));
        for (int k = 0; k < nks_; ++k) XK_CK(cudaStreamCreateWithFlags(&d.ks[k], cudaStreamNonBlocking));
        int lo = 0, hi = 0;
        XK_CK(cudaDeviceGetStreamPriorityRange(&lo, &hi));
        XK_CK(cudaStreamCreateWithPriority(&d.kdiag, cudaStreamNonBlocking, hi));
    }
    cur_dev_ = -1;
    ev_pool_.assign(G, {});
    ev_used_.assign(G, {});
    batch_.assign(G, PendingBatch());
    batch_count_.assign(G, 0);
    batches_in_call_.assign(G, 0);
    {
        const char *eb = std::getenv("XK_BATCH");
        int mb = (eb && *eb) ? std::atoi(eb) : 16;
        max_batch_ = std::max(1, std::min(kMaxBatch, mb));
    }
    // flags
    flags_.topo = cfg.topo;
    flags_.optimistic = cfg.optimistic;
    flags_.window = cfg.window > 0 ? cfg.window : 4;
    flags_.T = cfg.tile > 0 ? cfg.tile : 2048;
    flags_.P = cfg.grid_p;
    flags_.Q = cfg.grid_q;
    if (flags_.P <= 0 || flags_.Q <= 0) default_grid(G, &flags_.P, &flags_.Q);
    if (flags_.P * flags_.Q != G || flags_.topo < 0 || flags_.topo > 2) {
        set_error("config: grid P*Q must equal ngpus; topo in {0,1,2}");
        return XK_ERR_CONFIG;
    }
    if (rank_mode_) {
        int rc = init_rank_mode(cfg);
        if (rc) {
            if (sess_) sess_->abort();
            return rc;
        }
    }
    // same physical device (logical-device mode, or ranks sharing a GPU)
    auto same_dev = [&](int s, int d) {
        return rank_mode_ ? devs_[s].pci == devs_[d].pci : devs_[s].phys == devs_[d].phys;
    };
    // topology (a1): defaults, then the measured matrix when probing
    topo.G = G;
    topo.bw.assign((size_t)(G + 1) * (G + 1), 0);
    for (int s = 0; s <= G; ++s)
        for (int d = 0; d <= G; ++d) {
            int64_t v;
            if (s == G || d == G) v = (s == d) ? 3000000 : 55000;
            else if (s == d) v = 3000000;
            else v = same_dev(s, d) ? 1500000 : 700000;
            topo.bw[(size_t)s * (G + 1) + d] = v;
        }
    topo.rate_mflops = cfg.task_rate_mflops > 0 ? cfg.task_rate_mflops : 35000000;
    perf_rank.assign((size_t)G * G, 0);
    for (int s = 0; s < G; ++s)
        for (int d = 0; d < G; ++d) {
            int ps = devs_[s].phys, pd = devs_[d].phys;
            if (ps == pd || !devs_[s].local || !devs_[d].local) continue;
            int v = 0;
            if (cudaDeviceGetP2PAttribute(&v, cudaDevP2PAttrPerformanceRank, ps, pd) == cudaSuccess)
                perf_rank[(size_t)s * G + d] = v;
            cudaGetLastError();
        }
    if (cfg.probe) {
        int rc = rank_mode_ ? probe_topology_rank() : probe_topology();
        if (rc) {
            if (sess_) sess_->abort();
            return rc;
        }
    }
    // tile-cache capacity the planner plans against (shadow plans only when they fit)
    if (cfg.mem_bytes > 0) {
        flags_.mem_bytes = cfg.mem_bytes;
    } else if (rank_mode_) {
        flags_.mem_bytes = devs_[rank_].arena_bytes;  // the same on every rank
    } else {
        int64_t cap = INT64_MAX;
        for (int g = 0; g < G; ++g) {
            int share = 0;
            for (int h = 0; h < G; ++h) share += devs_[h].phys == devs_[g].phys;
            size_t fr = 0, tot = 0;
            XK_CK(cudaSetDevice(devs_[g].phys));
            XK_CK(cudaMemGetInfo(&fr, &tot));
            cap = std::min(cap, (int64_t)((double)fr * 0.9) / share);
        }
        cur_dev_ = -1;
        flags_.mem_bytes = cap;
    }
    planner_.reset(new Planner(topo, flags_));
    std::memset(&stats, 0, sizeof(stats));
    stats.ngpus = G;
    const char *tp = std::getenv("XK_TRACE");
    if (tp && *tp) return trace_start(tp);
    return XK_OK;
}

// a1: time pinned H2D/D2H per GPU and CE copies for every ordered GPU pair; the FP64
// tile rate from one T x T x T tile GEMM.  Untimed by the API ("store the
// performance of link during the library initialization").
int Runtime::probe_topology() {
    const int G = (int)devs_.size();
    const size_t bytes = (size_t)64 << 20;
    void *host = nullptr;
    XK_CK(cudaMallocHost(&host, bytes));
    std::memset(host, 1, bytes);
    std::vector<void *> dbuf(G, nullptr), dbuf2(G, nullptr);
    for (int g = 0; g < G; ++g) {
        XK_CK(cudaSetDevice(devs_[g].phys));
        XK_CK(cudaMalloc(&dbuf[g], bytes));
        XK_CK(cudaMalloc(&dbuf2[g], bytes));
    }
    auto timed = [&](int g, cudaStream_t s, auto fn, float *ms_out) -> int {
        XK_CK(cudaSetDevice(devs_[g].phys));
        cudaEvent_t a, b;
        XK_CK(cudaEventCreate(&a));
        XK_CK(cudaEventCreate(&b));
        float best = 1e30f;
        for (int rep = 0; rep < 3; ++rep) {
            XK_CK(cudaEventRecord(a, s));
            XK_CK(fn());
            XK_CK(cudaEventRecord(b, s));
            XK_CK(cudaEventSynchronize(b));
            float ms = 0;
            XK_CK(cudaEventElapsedTime(&ms, a, b));
            if (rep > 0) best = std::min(best, ms);
        }
        cudaEventDestroy(a);
        cudaEventDestroy(b);
        *ms_out = best;
        return XK_OK;
    };
    auto mbps = [&](float ms) { return (int64_t)((double)bytes / (ms * 1e-3) / 1e6); };
    const int N = G + 1;
    for (int g = 0; g < G; ++g) {
        float ms;
        int rc = timed(g, devs_[g].h2d, [&] { return cudaMemcpyAsync(dbuf[g], host, bytes, cudaMemcpyHostToDevice, devs_[g].h2d); }, &ms);
        if (rc) return rc;
        topo.bw[(size_t)G * N + g] = mbps(ms);
        rc = timed(g, devs_[g].d2h, [&] { return cudaMemcpyAsync(host, dbuf[g], bytes, cudaMemcpyDeviceToHost, devs_[g].d2h); }, &ms);
        if (rc) return rc;
        topo.bw[(size_t)g * N + G] = mbps(ms);
        rc = timed(g, devs_[g].p2p, [&] { return cudaMemcpyAsync(dbuf2[g], dbuf[g], bytes, cudaMemcpyDeviceToDevice, devs_[g].p2p); }, &ms);
        if (rc) return rc;
        topo.bw[(size_t)g * N + g] = mbps(ms);
    }
    for (int s = 0; s < G; ++s)
        for (int d = 0; d < G; ++d) {
            if (s == d) continue;
            float ms;
            int rc = timed(d, devs_[d].p2p, [&] { return cudaMemcpyAsync(dbuf[d], dbuf[s], bytes, cudaMemcpyDeviceToDevice, devs_[d].p2p); }, &ms);
            if (rc) return rc;
            topo.bw[(size_t)s * N + d] = mbps(ms);
        }
    topo.bw[(size_t)G * N + G] = topo.bw[0];
    // FP64 tile-task rate on GPU 0: one grouped launch of kRateTasks T x T x T tile GEMMs
    // (T <= 2048), the form the executor launches them in -- a lone tile launch leaves part
    // of the last wave idle and under-states the rate the planner's virtual time should use
    if (cfg_.task_rate_mflops <= 0) {
        constexpr int kRateTasks = 8;
        int64_t T = std::min<int64_t>(flags_.T, 2048);
        size_t tb = (size_t)T * T * 8;
        double *a = nullptr, *b = nullptr, *c = nullptr;
        XK_CK(cudaSetDevice(devs_[0].phys));
        XK_CK(cudaMalloc(&a, tb));
        XK_CK(cudaMalloc(&b, tb));
        XK_CK(cudaMalloc(&c, tb * kRateTasks));
        XK_CK(cudaMemsetAsync(a, 0, tb, devs_[0].ks[0]));
        XK_CK(cudaMemsetAsync(b, 0, tb, devs_[0].ks[0]));
        XK_CK(cudaMemsetAsync(c, 0, tb * kRateTasks, devs_[0].ks[0]));
        TileBatch batch;
        batch.n = kRateTasks;
        for (int q = 0; q < kRateTasks; ++q)
            batch.t[q] = TileTask{a, b, c + (size_t)q * T * T, T, T, T, T, T, T, 1.0, 1.0, 0, nullptr, 0, 0.0};
        float ms;
        int rc = timed(0, devs_[0].ks[0], [&] { return launch_dgemm_batch(false, false, batch, devs_[0].ks[0]); }, &ms);
        cudaFree(a);
        cudaFree(b);
        cudaFree(c);
        if (rc) return rc;
        topo.rate_mflops = std::max<int64_t>(1, (int64_t)(2.0 * T * T * T * kRateTasks / (ms * 1e3)));
    }
    for (int g = 0; g < G; ++g) {
        cudaSetDevice(devs_[g].phys);
        cudaFree(dbuf[g]);
        cudaFree(dbuf2[g]);
    }
    cudaFreeHost(host);
    cur_dev_ = -1;
    return XK_OK;
}

// Rank mode set-up: open the session file, map its flag array into this
// GPU's address space, agree on one arena size, allocate this GPU's tile arena and map
// every peer's arena through CUDA IPC.  Collective: every rank runs it in xk_init.
int Runtime::init_rank_mode(const xk_config_t &cfg) {
    const int G = (int)devs_.size();
    if (!stream_memops_available()) {
        set_error("rank mode: cuStreamWaitValue32/cuStreamWriteValue32 unavailable");
        return XK_ERR_CUDA;
    }
    std::string path(cfg.session, strnlen(cfg.session, sizeof cfg.session));
    if (path.empty()) {
        set_error("config: rank mode needs xk_config_t.session (a unique file path)");
        return XK_ERR_CONFIG;
    }
    sess_.reset(new Session());
    std::string err;
    int rc = sess_->open(path, rank_, G, 300.0, err);
    if (rc) {
        set_error(err);
        sess_.reset();
        return rc;
    }
    SessionHeader *h = sess_->hdr();
    SessionRank &me = h->rank[rank_];
    Device &d = devs_[rank_];
    XK_CK(cudaSetDevice(d.phys));
    XK_CK(cudaHostRegister(sess_->flags(), sess_->flags_bytes(), cudaHostRegisterPortable | cudaHostRegisterMapped));
    XK_CK(cudaHostGetDevicePointer((void **)&dflags_, sess_->flags(), 0));
    int dom = 0, bus = 0, dv = 0;
    XK_CK(cudaDeviceGetAttribute(&dom, cudaDevAttrPciDomainId, d.phys));
    XK_CK(cudaDeviceGetAttribute(&bus, cudaDevAttrPciBusId, d.phys));
    XK_CK(cudaDeviceGetAttribute(&dv, cudaDevAttrPciDeviceId, d.phys));
    me.pci = (dom << 16) | (bus << 8) | dv;
    // everything that shapes the plan must agree, or the processes would execute different
    // plans (FNV-1a over the fields; kstreams and the like only change local issue)
    uint64_t hcfg = 1469598103934665603ull;
    for (int64_t v : {(int64_t)cfg.tile, (int64_t)cfg.topo, (int64_t)cfg.optimistic, (int64_t)cfg.window,
                      (int64_t)cfg.grid_p, (int64_t)cfg.grid_q, (int64_t)cfg.probe, cfg.task_rate_mflops,
                      cfg.mem_bytes}) {
        hcfg ^= (uint64_t)v;
        hcfg *= 1099511628211ull;
    }
    me.plan_cfg = hcfg;
    auto bar = [&](const char *what) {
        if (sess_->barrier(300.0)) return XK_OK;
        set_error(std::string("rank mode: a peer failed or timed out during ") + what);
        return XK_ERR_CUDA;
    };
    if ((rc = bar("init (device ids)"))) return rc;
    for (int g = 0; g < G; ++g)
        if (h->rank[g].plan_cfg != me.plan_cfg) {
            set_error("config: rank mode needs the same tile/topo/optimistic/window/grid/probe/task rate on every rank");
            return XK_ERR_CONFIG;
        }
    int share = 0;
    for (int g = 0; g < G; ++g) {
        devs_[g].pci = h->rank[g].pci;
        share += h->rank[g].pci == me.pci;
    }
    size_t fr = 0, tot = 0;
    XK_CK(cudaMemGetInfo(&fr, &tot));
    me.arena_proposed = cfg.arena_bytes > 0 ? cfg.arena_bytes : (int64_t)((double)fr * 0.85) / std::max(1, share);
    if ((rc = bar("init (arena size)"))) return rc;
    int64_t ab = h->rank[0].arena_proposed;
    for (int g = 1; g < G; ++g) ab = std::min(ab, h->rank[g].arena_proposed);
    ab = ab / (2 << 20) * (2 << 20);
    if (ab < ((int64_t)256 << 20)) {
        set_error("rank mode: arena smaller than 256 MiB");
        return XK_ERR_OOM;
    }
    void *arena = nullptr;
    cudaError_t e = cudaMalloc(&arena, (size_t)ab);
    if (e != cudaSuccess) {
        cudaGetLastError();
        set_error("rank mode: cannot allocate the device tile arena");
        return XK_ERR_OOM;
    }
    d.arena = static_cast<char *>(arena);
    d.arena_bytes = ab;
    XK_CK(cudaIpcGetMemHandle(&me.arena, arena));
    me.arena_bytes = ab;
    if ((rc = bar("init (arena handles)"))) return rc;
    for (int g = 0; g < G; ++g) {
        if (g == rank_) continue;
        void *p = nullptr;
        XK_CK(cudaIpcOpenMemHandle(&p, h->rank[g].arena, cudaIpcMemLazyEnablePeerAccess));
        devs_[g].arena = static_cast<char *>(p);
        devs_[g].arena_bytes = h->rank[g].arena_bytes;
    }
    cur_dev_ = -1;
    return bar("init (arena mappings)");
}

// a1 in rank mode: each process times its own host links and local copies, then pulls
// 64 MiB from every peer's arena in G-1 barrier-separated rounds (round j: rank r pulls
// from rank r-j, a permutation, so no two pulls share a source); the rows meet in the
// session file and every process builds the identical matrix the planner needs.
int Runtime::probe_topology_rank() {
    const int G = (int)devs_.size(), N = G + 1;
    const size_t bytes = (size_t)64 << 20;
    Device &d = devs_[rank_];
    SessionHeader *h = sess_->hdr();
    SessionRank &me = h->rank[rank_];
    int rc;
    if ((rc = set_dev(rank_))) return rc;
    void *host = nullptr;
    XK_CK(cudaMallocHost(&host, bytes));
    std::memset(host, 1, bytes);
    char *src0 = d.arena, *dst = d.arena + bytes;
    auto timed = [&](cudaStream_t s, auto fn, float *ms_out) -> int {
        cudaEvent_t a, b;
        XK_CK(cudaEventCreate(&a));
        XK_CK(cudaEventCreate(&b));
        float best = 1e30f;
        for (int rep = 0; rep < 3; ++rep) {
            XK_CK(cudaEventRecord(a, s));
            XK_CK(fn());
            XK_CK(cudaEventRecord(b, s));
            XK_CK(cudaEventSynchronize(b));
            float ms = 0;
            XK_CK(cudaEventElapsedTime(&ms, a, b));
            if (rep > 0) best = std::min(best, ms);
        }
        cudaEventDestroy(a);
        cudaEventDestroy(b);
        *ms_out = best;
        return XK_OK;
    };
    auto mbps = [&](float ms) { return (int64_t)((double)bytes / (ms * 1e-3) / 1e6); };
    float ms;
    if ((rc = timed(d.h2d, [&] { return cudaMemcpyAsync(src0, host, bytes, cudaMemcpyHostToDevice, d.h2d); }, &ms))) return rc;
    me.bw_in[G] = mbps(ms);
    if ((rc = timed(d.d2h, [&] { return cudaMemcpyAsync(host, src0, bytes, cudaMemcpyDeviceToHost, d.d2h); }, &ms))) return rc;
    me.bw_to_host = mbps(ms);
    if ((rc = timed(d.p2p, [&] { return cudaMemcpyAsync(dst, src0, bytes, cudaMemcpyDeviceToDevice, d.p2p); }, &ms))) return rc;
    me.bw_local = mbps(ms);
    cudaFreeHost(host);
    for (int j = 1; j < G; ++j) {
        if (!sess_->barrier(300.0)) {
            set_error("rank mode: a peer failed during the topology probe");
            return XK_ERR_CUDA;
        }
        const int s = (rank_ - j + G) % G;
        const char *src = devs_[s].arena;
        if ((rc = timed(d.p2p, [&] { return cudaMemcpyAsync(dst, src, bytes, cudaMemcpyDeviceToDevice, d.p2p); }, &ms))) return rc;
        me.bw_in[s] = mbps(ms);
    }
    // FP64 tile-task rate, measured by rank 0 for everyone (T <= 2048, in its arena)
    me.rate_mflops = 0;
    if (rank_ == 0 && cfg_.task_rate_mflops <= 0) {
        // one grouped launch of up to 8 tile tasks, as in the single-process probe
        const int64_t T = std::min<int64_t>(flags_.T, 2048);
        const size_t tb = (size_t)T * T * 8;
        const int nt = (int)std::min<int64_t>(8, d.arena_bytes / (int64_t)tb - 2);
        if (nt >= 1) {
            double *a = reinterpret_cast<double *>(d.arena), *b = a + (size_t)T * T, *c = b + (size_t)T * T;
            XK_CK(cudaMemsetAsync(d.arena, 0, (2 + nt) * tb, d.ks[0]));
            TileBatch batch;
            batch.n = nt;
            for (int q = 0; q < nt; ++q)
                batch.t[q] = TileTask{a, b, c + (size_t)q * T * T, T, T, T, T, T, T, 1.0, 1.0, 0, nullptr, 0, 0.0};
            if ((rc = timed(d.ks[0], [&] { return launch_dgemm_batch(false, false, batch, d.ks[0]); }, &ms))) return rc;
            me.rate_mflops = std::max<int64_t>(1, (int64_t)(2.0 * T * T * T * nt / (ms * 1e3)));
        }
    }
    if (!sess_->barrier(300.0)) {
        set_error("rank mode: a peer failed during the topology probe");
        return XK_ERR_CUDA;
    }
    for (int g = 0; g < G; ++g) {
        const SessionRank &sr = h->rank[g];
        for (int s = 0; s < G; ++s)
            if (s != g) topo.bw[(size_t)s * N + g] = sr.bw_in[s];
        topo.bw[(size_t)G * N + g] = sr.bw_in[G];
        topo.bw[(size_t)g * N + G] = sr.bw_to_host;
        topo.bw[(size_t)g * N + g] = sr.bw_local;
    }
    topo.bw[(size_t)G * N + G] = topo.bw[0];
    if (cfg_.task_rate_mflops <= 0 && h->rank[0].rate_mflops > 0) topo.rate_mflops = h->rank[0].rate_mflops;
    cur_dev_ = -1;
    // nobody reuses its arena (tile allocations start at offset 0) before every pull is done
    if (!sess_->barrier(300.0)) {
        set_error("rank mode: a peer failed during the topology probe");
        return XK_ERR_CUDA;
    }
    return XK_OK;
}

cudaEvent_t Runtime::new_event(int g) {
    auto &pool = ev_pool_[g];
    cudaEvent_t e = nullptr;
    if (!pool.empty()) {
        e = pool.back();
        pool.pop_back();
    } else if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess) {
        return nullptr;
    }
    ev_used_[g].push_back(e);
    return e;
}

int Runtime::record(cudaStream_t s, int g, Ev *out) {
    cudaEvent_t e = new_event(g);
    if (!e) return cuda_fail(cudaGetLastError(), "cudaEventCreate");
    XK_CK(cudaEventRecord(e, s));
    out->e = e;
    out->s = s;
    out->c = ++rec_count_[s];
    return XK_OK;
}

int Runtime::wait_on(cudaStream_t s, const Ev &ev) {
    if (ev.rseq >= 0) {  // executed by a peer process: its completion flag
        if (ev.rseq < epoch_seq_) return XK_OK;
        XK_CK(stream_wait_flag(s, dflags_ + (uint64_t)ev.rseq % kFlagCap, (uint32_t)(ev.rseq + 1)));
        return XK_OK;
    }
    if (!ev.e || ev.s == s) return XK_OK;  // same stream: already ordered
    if (ev.c) {  // already waited for this event or a later one of its stream: implied
        uint64_t &w = waited_[std::make_pair(s, ev.s)];
        if (ev.c <= w) {
            ++waits_skipped_;
            return XK_OK;
        }
        w = ev.c;
    }
    XK_CK(cudaStreamWaitEvent(s, ev.e, 0));
    return XK_OK;
}

int Runtime::wait_dep(cudaStream_t s, int64_t seq) {
    if (seq < 0) return XK_OK;
    auto it = seq_ev_.find(seq);
    if (it != seq_ev_.end()) return wait_on(s, it->second);
    // not issued here since the last full sync: completed before it, or (rank mode)
    // executed by a peer process -- local records are always issued before a dependant
    if (rank_mode_ && seq >= epoch_seq_) return wait_on(s, Ev::remote(seq));
    return XK_OK;
}

int Runtime::signal(cudaStream_t s, int64_t seq) {
    if (!rank_mode_) return XK_OK;
    XK_CK(stream_write_flag(s, dflags_ + (uint64_t)seq % kFlagCap, (uint32_t)(seq + 1)));
    return XK_OK;
}

static void add_reader(Buffer &b, const Ev &ev) {
    for (auto &r : b.readers)
        if (ev.rseq < 0 && r.rseq < 0 && r.s == ev.s) {  // in-order stream: the newer event subsumes the older one
            r = ev;
            return;
        }
    b.readers.push_back(ev);
}

double *Runtime::alloc(int g, size_t bytes, int *rc) {
    Device &d = devs_[g];
    auto it = d.free_bufs.find(bytes);
    if (it != d.free_bufs.end() && !it->second.empty()) {
        double *p = it->second.back();
        it->second.pop_back();
        d.bytes_in_use += bytes;
        return p;
    }
    if (rank_mode_) {
        // every process runs this allocator for EVERY GPU in plan order, so all agree on
        // where each tile lives in each arena without exchanging a message
        const int64_t off = round_up(d.arena_top, 1024);
        if (off + (int64_t)bytes > d.arena_bytes) {
            set_error("rank mode: device tile arena full (no eviction): raise xk_config_t.arena_bytes");
            *rc = XK_ERR_OOM;
            return nullptr;
        }
        d.arena_top = off + (int64_t)bytes;
        d.bytes_in_use += bytes;
        return reinterpret_cast<double *>(d.arena + off);
    }
    if ((*rc = set_dev(g))) return nullptr;
    const auto t_alloc = std::chrono::steady_clock::now();
    struct AllocTimer {  // counts the new buffer and its host time on every exit path
        xk_stats_t &st;
        std::chrono::steady_clock::time_point t0;
        ~AllocTimer() {
            st.device_allocs++;
            st.device_alloc_ms += std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
        }
    } alloc_timer{stats, t_alloc};
    double *p = nullptr;
    cudaError_t e = cudaMalloc(&p, bytes);
    if (e != cudaSuccess) {
        cudaGetLastError();
        // give cached free buffers of this device back and retry once
        for (auto &kv : d.free_bufs)
            for (double *q : kv.second) {
                cudaFree(q);
                for (auto a = d.all_bufs.begin(); a != d.all_bufs.end(); ++a)
                    if (a->first == q) { d.all_bufs.erase(a); break; }
            }
        d.free_bufs.clear();
        e = cudaMalloc(&p, bytes);
        if (e != cudaSuccess) {
            cudaGetLastError();
            set_error("device tile cache full (no eviction): cudaMalloc failed");
            *rc = XK_ERR_OOM;
            return nullptr;
        }
    }
    d.all_bufs.push_back({p, bytes});
    d.bytes_in_use += bytes;
    return p;
}

void Runtime::free_buf(int g, double *p, size_t bytes) {
    devs_[g].free_bufs[bytes].push_back(p);
    devs_[g].bytes_in_use -= bytes;
}

Buffer *Runtime::buf(int key, int g, bool create, int *rc) {
    int64_t id = (int64_t)key * XK_MAX_GPUS + g;
    auto it = bufs_.find(id);
    if (it != bufs_.end()) return &it->second;
    if (!create) {
        set_error("internal: missing device tile");
        *rc = XK_ERR_INTERNAL;
        return nullptr;
    }
    const Entry &e = planner_->entry(key);
    Buffer b;
    b.ld = round_up(e.rows, 16);
    b.bytes = (size_t)b.ld * e.cols * 8;
    b.p = alloc(g, b.bytes, rc);
    if (!b.p) return nullptr;
    return &(bufs_[id] = b);
}

int Runtime::issue(const Rec &R) {
    const xk_plan_rec_t &r = R.r;
    const Entry &e = planner_->entry(R.key);
    const Matrix &M = planner_->matrix(e.mat);
    const int64_t T = flags_.T;
    int rc = XK_OK;
    // a record that depends on a deferred write-back: launch that batch (which issues it)
    for (int q = 0; q < 4 && !deferred_seq_.empty(); ++q) {
        auto it = r.dep[q] >= 0 ? deferred_seq_.find(r.dep[q]) : deferred_seq_.end();
        if (it != deferred_seq_.end() && (rc = flush_batch(it->second))) return rc;
    }
    // the D2H of a tile whose last writer is still in this GPU's pending batch waits for the
    // batch instead of launching it early (a step's diagonal ops / GEMMs stay one launch) --
    // except in the GPU's last tasks of the call, where the write-back is the tail
    if (rank_mode_ && r.seq - epoch_seq_ >= (int64_t)(kFlagCap / 2)) {
        set_error("rank mode: more plan records in flight than the completion-flag ring holds");
        return XK_ERR_UNSUPPORTED;
    }
    const int max_batch = planner_->batch_hint() > 0 ? std::min(max_batch_, planner_->batch_hint()) : max_batch_;
    if (defer_d2h_ && here(r) && r.kind == XK_REC_D2H && r.dep[0] >= 0 && batch_[r.src].contains_seq(r.dep[0]) &&
        batch_[r.src].recs.back().remaining >= max_batch) {
        PendingBatch &bt = batch_[r.src];
        bt.deferred.push_back(R);
        bt.in_ids.push_back((int64_t)R.key * XK_MAX_GPUS + r.src);
        deferred_seq_[r.seq] = r.src;
        return XK_OK;
    }
    if (r.kind != XK_REC_TASK && (rc = flush_for(R))) return rc;
    if (!here(r)) return issue_remote(R);
    switch (r.kind) {
    case XK_REC_H2D: {
        const int g = r.dst;
        if ((rc = set_dev(g))) return rc;
        Buffer *B = buf(R.key, g, true, &rc);
        if (!B) return rc;
        cudaStream_t s = devs_[g].h2d;
        if ((rc = wait_dep(s, r.dep[0]))) return rc;
        for (auto &rd : B->readers)
            if ((rc = wait_on(s, rd))) return rc;
        if ((rc = wait_on(s, B->writer))) return rc;
        const char *host = (const char *)(uintptr_t)M.base + (e.bi * T + e.bj * T * M.ld) * 8;
        cudaEvent_t ta = nullptr;
        if (tracing_ && (rc = trace_begin(g, s, &ta))) return rc;
        if ((rc = copy_host(true, B->p, B->ld, (char *)host, M.ld, e.rows, e.cols, s))) return rc;
        if (tracing_) trace_end(g, s, ta, 0, "H2D", r.work);
        Ev ev;
        if ((rc = record(s, g, &ev))) return rc;
        if ((rc = signal(s, r.seq))) return rc;
        seq_ev_[r.seq] = ev;
        B->writer = ev;
        B->readers.clear();
        stats.h2d_bytes[g] += r.work;
        stats.link_bytes[(size_t)devs_.size() * (devs_.size() + 1) + g] += r.work;
        return XK_OK;
    }
    case XK_REC_P2P: {
        const int g = r.dst, gs = r.src;
        Buffer *S = buf(R.key, gs, false, &rc);
        if (!S) return rc;
        if ((rc = set_dev(g))) return rc;
        Buffer *D = buf(R.key, g, true, &rc);
        if (!D) return rc;
        S = buf(R.key, gs, false, &rc);  // rehash may have moved it
        cudaStream_t s = devs_[g].p2p;
        if ((rc = wait_dep(s, r.dep[0]))) return rc;
        if ((rc = wait_on(s, S->writer))) return rc;
        for (auto &rd : D->readers)
            if ((rc = wait_on(s, rd))) return rc;
        if ((rc = wait_on(s, D->writer))) return rc;
        // store-and-forward of a whole compact tile over NVLink (copy engine, SMs stay free)
        cudaEvent_t ta = nullptr;
        if (tracing_ && (rc = trace_begin(g, s, &ta))) return rc;
        XK_CK(cudaMemcpyAsync(D->p, S->p, S->bytes, cudaMemcpyDeviceToDevice, s));
        if (tracing_) trace_end(g, s, ta, 1, r.src_state == XK_SRC_INFLIGHT ? "P2P fwd-inflight" : "P2P", r.work);
        Ev ev;
        if ((rc = record(s, g, &ev))) return rc;
        if ((rc = signal(s, r.seq))) return rc;
        seq_ev_[r.seq] = ev;
        D->writer = ev;
        D->readers.clear();
        add_reader(*S, ev);
        stats.p2p_in_bytes[g] += r.work;
        stats.p2p_out_bytes[gs] += r.work;
        stats.link_bytes[(size_t)gs * (devs_.size() + 1) + g] += r.work;
        if (r.src_state == XK_SRC_INFLIGHT) stats.forwards_inflight++;
        else stats.forwards_valid++;
        return XK_OK;
    }
    case XK_REC_TASK: {
        const int g = r.dst;
        if ((rc = set_dev(g))) return rc;
        Buffer *O = buf(R.key, g, true, &rc);
        if (!O) return rc;
        const int64_t idO = (int64_t)R.key * XK_MAX_GPUS + g;
        if (R.op == XK_OP_TRSM_DIAG || R.op == XK_OP_TRMM_DIAG) {
            // diagonal solves/multiplies of one step share the diagonal tile of A: grouped
            // into one recursion over all their B tiles (grouped GEMMs, one base launch)
            if (!buf(R.keyA, g, false, &rc)) return rc;
            if (R.keyC2 >= 0 && !buf(R.keyC2, g, false, &rc)) return rc;
            const int64_t idA = (int64_t)R.keyA * XK_MAX_GPUS + g;
            const int64_t idC2 = R.keyC2 >= 0 ? (int64_t)R.keyC2 * XK_MAX_GPUS + g : -1;
            PendingBatch &bt = batch_[g];
            bool conflict = !bt.recs.empty() &&
                            (bt.op != R.op || bt.recs[0].keyA != R.keyA || bt.recs[0].alpha != R.alpha ||
                             bt.recs[0].side != R.side || bt.recs[0].uplo != R.uplo || bt.recs[0].ta != R.ta ||
                             bt.recs[0].diag != R.diag ||
                             (R.side == 'L' ? bt.recs[0].m != R.m : bt.recs[0].n != R.n));
            conflict = conflict || (int)bt.recs.size() >= max_batch || bt.touches(idO, true) ||
                       bt.touches(idA, false) || (idC2 >= 0 && bt.touches(idC2, false));
            for (int q = 0; q < 4 && !conflict; ++q)
                if (r.dep[q] >= 0 && bt.contains_seq(r.dep[q])) conflict = true;
            if (conflict && (rc = flush_batch(g))) return rc;
            bt.recs.push_back(R);
            bt.out_ids.push_back(idO);
            bt.in_ids.push_back(idA);
            if (idC2 >= 0) bt.in_ids.push_back(idC2);
            bt.op = R.op;
            return XK_OK;
        }
        if (R.op != XK_OP_GEMM && R.op != XK_OP_GEMM_TRI) {
            // scale / diagonal-tile ops are launched directly, after this GPU's pending batch
            if ((rc = flush_batch(g))) return rc;
            // independent scale / SYMM-diagonal ops spread over all kernel streams
            const uint64_t h = (uint64_t)(e.bi * 7919 + e.bj * 104729);
            cudaStream_t s = devs_[g].ks[h % (uint64_t)nks_];
            for (int q = 0; q < 4; ++q)
                if ((rc = wait_dep(s, r.dep[q]))) return rc;
            for (auto &rd : O->readers)
                if ((rc = wait_on(s, rd))) return rc;
            if ((rc = wait_on(s, O->writer))) return rc;
            Buffer *A = nullptr, *B = nullptr;
            if (R.keyA >= 0 && !(A = buf(R.keyA, g, false, &rc))) return rc;
            if (R.keyB >= 0 && !(B = buf(R.keyB, g, false, &rc))) return rc;
            O = buf(R.key, g, false, &rc);
            cudaError_t ke = cudaSuccess;
            cudaEvent_t ta = nullptr;
            if (tracing_ && (rc = trace_begin(g, s, &ta))) return rc;
            if (R.op == XK_OP_SCALE) {
                ke = launch_scale_tri(R.m, R.n, R.beta, O->p, O->ld, R.tri, s);
            } else if (R.op == XK_OP_SYMM_DIAG) {
                // expand the diagonal tile of A symmetrically into a scratch tile, then GEMM
                const int64_t ka = (R.side == 'L') ? R.m : R.n;
                const int64_t lds = (ka + 15) / 16 * 16;
                double *S = alloc(g, (size_t)lds * ka * 8, &rc);
                if (!S) return rc;
                scratch_.push_back({g, {S, (size_t)lds * ka * 8}});
                ke = launch_symm_expand(ka, A->p, A->ld, R.uplo, S, lds, s);
                if (ke == cudaSuccess) {
                    if (R.side == 'L')
                        ke = launch_dgemm_tile(false, false, R.m, R.n, R.k, R.alpha, S, lds, B->p, B->ld, R.beta,
                                               O->p, O->ld, s);
                    else
                        ke = launch_dgemm_tile(false, false, R.m, R.n, R.k, R.alpha, B->p, B->ld, S, lds, R.beta,
                                               O->p, O->ld, s);
                }
            } else {
                set_error("internal: unknown tile op");
                return XK_ERR_INTERNAL;
            }
            if (ke != cudaSuccess) return cuda_fail(ke, "tile kernel launch");
            if (tracing_) {
                static const char *nm[] = {"gemm", "scale", "gemm_tri", "symm_diag", "trmm_diag", "trsm_diag"};
                trace_end(g, s, ta, 2, nm[R.op], r.work);
            }
            Ev ev;
            if ((rc = record(s, g, &ev))) return rc;
            if ((rc = signal(s, r.seq))) return rc;
            seq_ev_[r.seq] = ev;
            O->writer = ev;
            O->readers.clear();
            if (A) add_reader(*A, ev);
            if (B) add_reader(*B, ev);
            stats.tasks[g]++;
            stats.flops[g] += r.work;
            stats.kernel_launches++;
            return XK_OK;
        }
        if (!buf(R.keyA, g, false, &rc) || !buf(R.keyB, g, false, &rc)) return rc;
        if (R.keyC2 >= 0 && !buf(R.keyC2, g, false, &rc)) return rc;
        const int64_t idA = (int64_t)R.keyA * XK_MAX_GPUS + g, idB = (int64_t)R.keyB * XK_MAX_GPUS + g;
        const int64_t idC2 = R.keyC2 >= 0 ? (int64_t)R.keyC2 * XK_MAX_GPUS + g : -1;
        PendingBatch &bt = batch_[g];
        // batch size ramps 1, 2, 4, ... (ramp_div_ launches per size, XK_RAMP) up to max_batch_
        // at the start of each call, so the
        // first kernels start as soon as their own inputs have landed instead of waiting
        // for a whole batch worth of tiles to cross PCIe
        // ... and ramps down (half of the GPU's remaining tasks) at the end, so the write-back
        // of the last C tiles does not wait for one large final batch
        const int64_t left0 = (bt.recs.empty() ? R.remaining : bt.recs[0].remaining) + 1;
        const int cap = (int)std::min<int64_t>(std::min<int64_t>(max_batch, std::max<int64_t>(1, (left0 + 1) / 2)),
                                               (int64_t)1 << std::min<int64_t>(batches_in_call_[g] / ramp_div_, 5));
        bool conflict = (int)bt.recs.size() >= cap ||
                        (!bt.recs.empty() && (bt.op == XK_OP_TRSM_DIAG || bt.op == XK_OP_TRMM_DIAG)) ||
                        (!bt.recs.empty() && (bt.ta != R.ta || bt.tb != R.tb)) ||
                        bt.touches(idO, true) || bt.touches(idA, false) || bt.touches(idB, false) ||
                        (idC2 >= 0 && bt.touches(idC2, false));
        for (int q = 0; q < 4 && !conflict; ++q)
            if (r.dep[q] >= 0 && bt.contains_seq(r.dep[q])) conflict = true;
        if (conflict && (rc = flush_batch(g))) return rc;
        bt.recs.push_back(R);
        bt.out_ids.push_back(idO);
        bt.in_ids.push_back(idA);
        bt.in_ids.push_back(idB);
        if (idC2 >= 0) bt.in_ids.push_back(idC2);
        bt.ta = R.ta;
        bt.tb = R.tb;
        bt.op = XK_OP_GEMM;
        return XK_OK;
    }
    case XK_REC_D2H: {
        const int gs = r.src;
        if ((rc = set_dev(gs))) return rc;
        Buffer *S = buf(R.key, gs, false, &rc);
        if (!S) return rc;
        cudaStream_t s = devs_[gs].d2h;
        if ((rc = wait_dep(s, r.dep[0]))) return rc;
        if ((rc = wait_on(s, S->writer))) return rc;
        char *host = (char *)(uintptr_t)M.base +
                     ((e.bi * T + R.sub_r0) + (e.bj * T + R.sub_c0) * M.ld) * 8;
        const double *src = S->p + R.sub_r0 + R.sub_c0 * S->ld;
        cudaEvent_t ta = nullptr;
        if (tracing_ && (rc = trace_begin(gs, s, &ta))) return rc;
        if ((rc = copy_host(false, (double *)src, S->ld, host, M.ld, R.sub_rows, R.sub_cols, s))) return rc;
        if (tracing_) trace_end(gs, s, ta, 3, "D2H", r.work);
        Ev ev;
        if ((rc = record(s, gs, &ev))) return rc;
        if ((rc = signal(s, r.seq))) return rc;
        seq_ev_[r.seq] = ev;
        add_reader(*S, ev);
        pending_d2h_.push_back(ev);
        stats.d2h_bytes[gs] += r.work;
        stats.link_bytes[(size_t)gs * (devs_.size() + 1) + devs_.size()] += r.work;
        return XK_OK;
    }
    default:
        set_error("internal: unknown record kind");
        return XK_ERR_INTERNAL;
    }
}

// Rank mode: a record another process executes.  Nothing is enqueued here; the directory
// of buffers is kept identical on every process (same allocations, in plan order), the
// peer's output is known only by its completion flag, and a P2P that pulls one of OUR
// tiles becomes a remote reader of it (a later overwrite waits for the pull's flag).
int Runtime::issue_remote(const Rec &R) {
    const xk_plan_rec_t &r = R.r;
    int rc = XK_OK;
    switch (r.kind) {
    case XK_REC_H2D:
    case XK_REC_P2P: {
        Buffer *D = buf(R.key, r.dst, true, &rc);
        if (!D) return rc;
        D->writer = Ev::remote(r.seq);
        D->readers.clear();
        if (r.kind == XK_REC_P2P && r.src == rank_) {
            Buffer *S = buf(R.key, r.src, false, &rc);
            if (!S) return rc;
            add_reader(*S, Ev::remote(r.seq));
            stats.p2p_out_bytes[rank_] += r.work;  // pulled by the peer, counted at the source too
        }
        return XK_OK;
    }
    case XK_REC_TASK: {
        Buffer *O = buf(R.key, r.dst, true, &rc);
        if (!O) return rc;
        O->writer = Ev::remote(r.seq);
        O->readers.clear();
        if (R.op == XK_OP_SYMM_DIAG) {  // the owner's scratch tile, same size and order
            const int64_t ka = (R.side == 'L') ? R.m : R.n;
            const size_t sb = (size_t)((ka + 15) / 16 * 16) * ka * 8;
            double *S = alloc(r.dst, sb, &rc);
            if (!S) return rc;
            scratch_.push_back({r.dst, {S, sb}});
        }
        return XK_OK;
    }
    case XK_REC_D2H:
        return XK_OK;
    default:
        set_error("internal: unknown record kind");
        return XK_ERR_INTERNAL;
    }
}

// Launch the pending tile tasks of GPU g as one grouped kernel on the next kernel stream.
int Runtime::flush_batch(int g) {
    PendingBatch &bt = batch_[g];
    if (bt.recs.empty()) return XK_OK;
    int rc;
    if ((rc = set_dev(g))) return rc;
    const Device &d = devs_[g];
    // kernel timing serialises the grouped launches on one stream so that each launch's
    // event-timed duration is its own (no overlap with a concurrent launch)
    const bool diag = bt.op == XK_OP_TRSM_DIAG || bt.op == XK_OP_TRMM_DIAG;
    // diagonal-tile ops go to the high-priority stream: with the planner's lookahead (R9) a
    // TRSM step's solve overlaps the previous step's trailing updates instead of queueing
    // behind them
    cudaStream_t s = kernel_timing ? d.ks[0] : diag ? d.kdiag : d.ks[batch_count_[g]++ % cfg_.kstreams];
    if (diag) {
        const Rec &R0 = bt.recs[0];
        Buffer *A = buf(R0.keyA, g, false, &rc);
        if (!A) return rc;
        double *Bp[kMaxBatch];
        int64_t ldb[kMaxBatch], other[kMaxBatch];
        int64_t flops = 0;
        const int nb = (int)bt.recs.size();
        for (int q = 0; q < nb; ++q) {
            const Rec &R = bt.recs[q];
            for (int j = 0; j < 4; ++j)
                if ((rc = wait_dep(s, R.r.dep[j]))) return rc;
            Buffer *O = buf(R.key, g, false, &rc);
            if (!O) return rc;
            for (auto &rd : O->readers)
                if ((rc = wait_on(s, rd))) return rc;
            if ((rc = wait_on(s, O->writer))) return rc;
            Bp[q] = O->p;
            ldb[q] = O->ld;
            other[q] = (R.side == 'L') ? R.n : R.m;
            flops += R.r.work;
        }
        cudaEvent_t ta = nullptr;
        if (tracing_ && (rc = trace_begin(g, s, &ta))) return rc;
        // TRMM from a shadow (reading R15): the input tile is copied into the output tile,
        // then multiplied in place with the others of the group
        for (int q = 0; q < nb; ++q) {
            const Rec &R = bt.recs[q];
            if (R.keyC2 < 0) continue;
            Buffer *S = buf(R.keyC2, g, false, &rc);
            if (!S) return rc;
            cudaError_t ce = cudaMemcpy2DAsync(Bp[q], (size_t)ldb[q] * 8, S->p, (size_t)S->ld * 8,
                                               (size_t)R.m * 8, (size_t)R.n, cudaMemcpyDeviceToDevice, s);
            if (ce != cudaSuccess) return cuda_fail(ce, "shadow tile copy");
        }
        cudaError_t ke = launch_trxm_batch(bt.op == XK_OP_TRSM_DIAG, R0.side, R0.uplo, R0.ta, R0.diag,
                                           R0.side == 'L' ? R0.m : R0.n, R0.alpha, A->p, A->ld, nb, Bp,
                                           ldb, other, s);
        if (ke != cudaSuccess) return cuda_fail(ke, "diagonal-tile kernel launch");
        if (tracing_)
            trace_end(g, s, ta, 2, std::string(bt.op == XK_OP_TRSM_DIAG ? "trsm_diag x" : "trmm_diag x") +
                                       std::to_string(nb), flops);
        Ev ev;
        if ((rc = record(s, g, &ev))) return rc;
        for (int q = 0; q < nb; ++q) {
            const Rec &R = bt.recs[q];
            if ((rc = signal(s, R.r.seq))) return rc;
            seq_ev_[R.r.seq] = ev;
            Buffer *O = buf(R.key, g, false, &rc);
            O->writer = ev;
            O->readers.clear();
            if (R.keyC2 >= 0) add_reader(*buf(R.keyC2, g, false, &rc), ev);
            stats.tasks[g]++;
            stats.flops[g] += R.r.work;
        }
        add_reader(*A, ev);
        stats.kernel_launches++;
        bt.recs.clear();
        bt.out_ids.clear();
        bt.in_ids.clear();
        return issue_deferred(g);
    }
    TileBatch tb;
    tb.n = (int)bt.recs.size();
    int64_t flops = 0;
    for (int q = 0; q < tb.n; ++q) {
        const Rec &R = bt.recs[q];
        for (int j = 0; j < 4; ++j)
            if ((rc = wait_dep(s, R.r.dep[j]))) return rc;
        Buffer *O = buf(R.key, g, false, &rc);
        Buffer *A = buf(R.keyA, g, false, &rc);
        Buffer *B = buf(R.keyB, g, false, &rc);
        if (!O || !A || !B) return rc;
        for (auto &rd : O->readers)
            if ((rc = wait_on(s, rd))) return rc;
        if ((rc = wait_on(s, O->writer))) return rc;
        Buffer *C2 = nullptr;
        if (R.keyC2 >= 0 && !(C2 = buf(R.keyC2, g, false, &rc))) return rc;
        tb.t[q] = TileTask{A->p, B->p, O->p, A->ld, B->ld, O->ld, R.m, R.n, R.k, R.alpha, R.beta, R.tri,
                           C2 ? C2->p : nullptr, C2 ? C2->ld : 0, C2 ? R.beta2 : 0.0};
        flops += R.r.work;
    }
    cudaEvent_t t0 = nullptr, t1 = nullptr;
    if (kernel_timing) {
        XK_CK(cudaEventCreate(&t0));
        XK_CK(cudaEventCreate(&t1));
        XK_CK(cudaEventRecord(t0, s));
    }
    cudaEvent_t tra = nullptr;
    if (tracing_ && (rc = trace_begin(g, s, &tra))) return rc;
    cudaError_t ke = launch_dgemm_batch(bt.ta == 'T', bt.tb == 'T', tb, s);
    if (ke != cudaSuccess) return cuda_fail(ke, "tile kernel launch");
    if (tracing_) trace_end(g, s, tra, 2, "gemm batch x" + std::to_string(tb.n), flops);
    if (kernel_timing) {
        XK_CK(cudaEventRecord(t1, s));
        ktimers_.push_back({t0, t1});
        ktimer_flops_.push_back(flops);
    }
    Ev ev;
    if ((rc = record(s, g, &ev))) return rc;
    for (int q = 0; q < tb.n; ++q) {
        const Rec &R = bt.recs[q];
        if ((rc = signal(s, R.r.seq))) return rc;
        seq_ev_[R.r.seq] = ev;
        Buffer *O = buf(R.key, g, false, &rc);
        O->writer = ev;
        O->readers.clear();
        add_reader(*buf(R.keyA, g, false, &rc), ev);
        add_reader(*buf(R.keyB, g, false, &rc), ev);
        if (R.keyC2 >= 0) add_reader(*buf(R.keyC2, g, false, &rc), ev);
        stats.tasks[g]++;
        stats.flops[g] += R.r.work;
    }
    stats.kernel_launches++;
    batches_in_call_[g]++;
    bt.recs.clear();
    bt.out_ids.clear();
    bt.in_ids.clear();
    return issue_deferred(g);
}

// Issue the write-backs that waited for GPU g's batch (now launched, so their last writer
// has an event).
int Runtime::issue_deferred(int g) {
    if (batch_[g].deferred.empty()) return XK_OK;
    std::vector<Rec> d;
    d.swap(batch_[g].deferred);
    for (const Rec &R : d) deferred_seq_.erase(R.r.seq);
    for (const Rec &R : d) {
        int rc = issue(R);
        if (rc) return rc;
    }
    return XK_OK;
}

// Before a copy record is issued: launch any pending batch it depends on or whose
// buffers it overwrites.
int Runtime::flush_for(const Rec &R) {
    const xk_plan_rec_t &r = R.r;
    for (size_t g = 0; g < batch_.size(); ++g) {
        PendingBatch &bt = batch_[g];
        if (bt.recs.empty()) continue;
        bool need = r.dep[0] >= 0 && bt.contains_seq(r.dep[0]);
        if (!need && r.kind != XK_REC_D2H && r.dst == (int)g)
            need = bt.touches((int64_t)R.key * XK_MAX_GPUS + g, true);
        if (!need && (r.kind == XK_REC_P2P || r.kind == XK_REC_D2H) && r.src == (int)g)
            need = bt.touches((int64_t)R.key * XK_MAX_GPUS + g, false);
        if (need) {
            int rc = flush_batch((int)g);
            if (rc) return rc;
        }
    }
    return XK_OK;
}

// ---------------------------------------------------------------- timeline tracing
int Runtime::trace_begin(int g, cudaStream_t s, cudaEvent_t *a) {
    XK_CK(cudaEventCreate(a));
    XK_CK(cudaEventRecord(*a, s));
    (void)g;
    return XK_OK;
}

void Runtime::trace_end(int g, cudaStream_t s, cudaEvent_t a, int kind, std::string name, int64_t work) {
    cudaEvent_t b = nullptr;
    if (cudaEventCreate(&b) != cudaSuccess || cudaEventRecord(b, s) != cudaSuccess) {
        cudaGetLastError();
        return;
    }
    trace_ops_.push_back({g, kind, a, b, std::move(name), work});
}

// After a full sync: turn the recorded event pairs into Chrome-trace events.
void Runtime::trace_collect() {
    static const char *tid[] = {"H2D", "P2P-in", "kernels", "D2H"};
    for (auto &op : trace_ops_) {
        float t0 = 0, t1 = 0;
        if (cudaEventElapsedTime(&t0, trace_base_[op.g], op.a) == cudaSuccess &&
            cudaEventElapsedTime(&t1, trace_base_[op.g], op.b) == cudaSuccess) {
            char buf[256];
            snprintf(buf, sizeof buf,
                     "{\"name\":\"%s\",\"ph\":\"X\",\"ts\":%.3f,\"dur\":%.3f,\"pid\":\"GPU %d\",\"tid\":\"%s\",\"args\":{\"%s\":%lld}}",
                     op.name.c_str(), t0 * 1e3, (t1 - t0) * 1e3, op.g, tid[op.kind],
                     op.kind == 2 ? "flops" : "bytes", (long long)op.work);
            trace_json_.push_back(buf);
            stats.trace_ms[op.kind] += (t1 - t0);
        }
        cudaEventDestroy(op.a);
        cudaEventDestroy(op.b);
    }
    cudaGetLastError();
    trace_ops_.clear();
}

int Runtime::trace_start(const std::string &path) {
    std::lock_guard<std::recursive_mutex> lk(mu);
    int rc = sync_all();
    if (rc) return rc;
    trace_path_ = path;
    trace_json_.clear();
    trace_base_.assign(devs_.size(), nullptr);
    for (size_t g = 0; g < devs_.size(); ++g) {
        if (!devs_[g].local) continue;
        XK_CK(cudaSetDevice(devs_[g].phys));
        XK_CK(cudaEventCreate(&trace_base_[g]));
        XK_CK(cudaEventRecord(trace_base_[g], devs_[g].h2d));
    }
    cur_dev_ = -1;
    tracing_ = true;
    return XK_OK;
}

int Runtime::trace_stop() {
    std::lock_guard<std::recursive_mutex> lk(mu);
    if (!tracing_) return XK_OK;
    int rc = sync_all();  // collects the remaining ops
    tracing_ = false;
    FILE *f = fopen(trace_path_.c_str(), "w");
    if (f) {
        fprintf(f, "{\"traceEvents\":[\n");
        for (size_t i = 0; i < trace_json_.size(); ++i)
            fprintf(f, "%s%s\n", trace_json_[i].c_str(), i + 1 < trace_json_.size() ? "," : "");
        fprintf(f, "],\"displayTimeUnit\":\"ms\"}\n");
        fclose(f);
    } else if (!rc) {
        set_error("xk_trace: cannot write " + trace_path_);
        rc = XK_ERR_CONFIG;
    }
    for (cudaEvent_t e : trace_base_) cudaEventDestroy(e);
    trace_base_.clear();
    trace_json_.clear();
    return rc;
}

// Boundaries of host registrations strictly inside [lo, hi): a pinned copy must not
// straddle two registrations (the driver rejects it), so copy_host splits there.
std::vector<uintptr_t> Runtime::reg_cuts(uintptr_t lo, uintptr_t hi) const {
    const uintptr_t page = 4096;
    std::vector<uintptr_t> cuts;
    auto scan = [&](const std::map<uintptr_t, size_t> &m) {
        for (auto &kv : m) {
            uintptr_t a = kv.first / page * page, b = (kv.first + kv.second + page - 1) / page * page;
            if (lo < a && a < hi) cuts.push_back(a);
            if (lo < b && b < hi) cuts.push_back(b);
        }
    };
    scan(internal_reg_);
    scan(registered_);
    std::sort(cuts.begin(), cuts.end());
    cuts.erase(std::unique(cuts.begin(), cuts.end()), cuts.end());
    return cuts;
}

// 2D copy between a device tile (ld = dld) and a host view (ld = hld), split so that no
// single copy crosses a host registration boundary.
int Runtime::copy_host(bool h2d, double *dev, int64_t dld, char *host, int64_t hld, int64_t rows,
                       int64_t cols, cudaStream_t s) {
    const cudaMemcpyKind kind = h2d ? cudaMemcpyHostToDevice : cudaMemcpyDeviceToHost;
    const uintptr_t lo = (uintptr_t)host;
    const uintptr_t hi = lo + (uintptr_t)(((cols - 1) * hld + rows) * 8);
    std::vector<uintptr_t> cuts = reg_cuts(lo, hi);
    auto cp2d = [&](int64_t c0, int64_t ncol) -> int {
        char *h = host + c0 * hld * 8;
        double *d = dev + c0 * dld;
        cudaError_t e = h2d ? cudaMemcpy2DAsync(d, dld * 8, h, hld * 8, rows * 8, ncol, kind, s)
                            : cudaMemcpy2DAsync(h, hld * 8, d, dld * 8, rows * 8, ncol, kind, s);
        if (e != cudaSuccess) return cuda_fail(e, "cudaMemcpy2DAsync (tile)");
        return XK_OK;
    };
    if (cuts.empty()) return cp2d(0, cols);
    auto segment = [&](uintptr_t a) {  // index of the registration segment holding address a
        return (int64_t)(std::upper_bound(cuts.begin(), cuts.end(), a) - cuts.begin());
    };
    int64_t c = 0;
    while (c < cols) {
        uintptr_t cl = lo + (uintptr_t)(c * hld * 8), ch = cl + (uintptr_t)(rows * 8);
        if (segment(cl) != segment(ch - 1)) {
            // this column straddles a boundary: 1D pieces
            uintptr_t a = cl;
            while (a < ch) {
                auto it = std::upper_bound(cuts.begin(), cuts.end(), a);
                uintptr_t b = (it == cuts.end() || *it > ch) ? ch : *it;
                char *h = (char *)a;
                char *d = (char *)(dev + c * dld) + (a - cl);
                cudaError_t e = h2d ? cudaMemcpyAsync(d, h, b - a, kind, s) : cudaMemcpyAsync(h, d, b - a, kind, s);
                if (e != cudaSuccess) return cuda_fail(e, "cudaMemcpyAsync (tile piece)");
                a = b;
            }
            ++c;
            continue;
        }
        int64_t seg = segment(cl), c2 = c + 1;
        while (c2 < cols) {
            uintptr_t l2 = lo + (uintptr_t)(c2 * hld * 8), h2 = l2 + (uintptr_t)(rows * 8);
            if (segment(l2) != seg || segment(h2 - 1) != seg) break;
            ++c2;
        }
        int rc = cp2d(c, c2 - c);
        if (rc) return rc;
        c = c2;
    }
    return XK_OK;
}

static bool host_pinned(uintptr_t addr) {
    cudaPointerAttributes a{};
    bool ok = cudaPointerGetAttributes(&a, (void *)addr) == cudaSuccess && a.type == cudaMemoryTypeHost;
    cudaGetLastError();
    return ok;
}

// Page-lock a host view for the duration of the call (or of the async epoch).  Memory the
// caller registered (xk_register, cudaHostRegister, cudaMallocHost, torch pin_memory) is
// used as is; otherwise the page range is registered internally -- skipping a boundary
// page that a neighbouring allocation already pinned -- and counted in the stats.  Internal
// registrations are dropped at the next full synchronisation point, so a registration
// never outlives the caller's buffer (the async contract keeps buffers alive until then).
int Runtime::ensure_pinned(uint64_t base, int64_t rows, int64_t cols, int64_t ld) {
    if (rows <= 0 || cols <= 0) return XK_OK;
    uintptr_t lo = (uintptr_t)base, hi = lo + (uintptr_t)(((cols - 1) * ld + rows) * 8);
    auto covered = [&](const std::map<uintptr_t, size_t> &m) {
        auto it = m.upper_bound(lo);
        if (it == m.begin()) return false;
        --it;
        return it->first <= lo && hi <= it->first + it->second;
    };
    if (covered(registered_) || covered(internal_reg_)) return XK_OK;
    const uintptr_t page = 4096;
    bool lo_p = host_pinned(lo), hi_p = host_pinned(hi - 1);
    if (lo_p && hi_p && host_pinned(lo + (hi - lo) / 2)) return XK_OK;  // pinned elsewhere
    uintptr_t plo = lo_p ? ((lo / page) + 1) * page : (lo / page) * page;
    uintptr_t phi = hi_p ? ((hi - 1) / page) * page : ((hi + page - 1) / page) * page;
    if (phi <= plo) return XK_OK;
    cudaError_t e = cudaHostRegister((void *)plo, phi - plo, cudaHostRegisterPortable);
    if (e == cudaErrorHostMemoryAlreadyRegistered) {
        cudaGetLastError();
        return XK_OK;
    }
    if (e != cudaSuccess) return cuda_fail(e, "cudaHostRegister (internal)");
    internal_reg_[plo] = phi - plo;
    stats.host_registrations++;
    return XK_OK;
}

void Runtime::release_internal_pins() {
    for (auto &kv : internal_reg_) cudaHostUnregister((void *)kv.first);
    cudaGetLastError();
    internal_reg_.clear();
}

// BW_h2d(G), BW_d2h(G) and full duplex with every GPU copying at once
// from its own pinned host region (host DRAM and root complexes are shared).
int Runtime::probe_host_links(int64_t bytes_per_gpu) {
    std::lock_guard<std::recursive_mutex> lk(mu);
    int rc = sync_all();
    if (rc) return rc;
    const int G = (int)devs_.size();
    std::vector<int> mine;
    for (int g = 0; g < G; ++g)
        if (devs_[g].local) mine.push_back(g);
    const size_t n = mine.size();
    std::vector<void *> hin(n, nullptr), hout(n, nullptr), din(n, nullptr), dout(n, nullptr);
    size_t bytes = (size_t)bytes_per_gpu;
    // rank mode: the device side of the probe lives in the free top of this rank's tile arena
    // (the arena holds most of the device memory; a cudaMalloc next to it may not fit)
    const bool in_arena = rank_mode_;
    auto release = [&]() {
        for (size_t q = 0; q < n; ++q) {
            if (hin[q]) cudaFreeHost(hin[q]);
            if (hout[q]) cudaFreeHost(hout[q]);
            cudaSetDevice(devs_[mine[q]].phys);
            if (!in_arena && din[q]) cudaFree(din[q]);
            if (!in_arena && dout[q]) cudaFree(dout[q]);
            hin[q] = hout[q] = din[q] = dout[q] = nullptr;
        }
        cudaGetLastError();
        cur_dev_ = -1;
    };
    // allocate, halving on failure down to 64 MiB; rank mode: collectively (every rank must
    // probe the same size): each posts whether it could allocate, all halve if one could not
    for (;;) {
        bool ok = true;
        for (size_t q = 0; q < n && ok; ++q) {
            ok = cudaHostAlloc(&hin[q], bytes, cudaHostAllocPortable) == cudaSuccess &&
                 cudaHostAlloc(&hout[q], bytes, cudaHostAllocPortable) == cudaSuccess &&
                 cudaSetDevice(devs_[mine[q]].phys) == cudaSuccess;
            if (ok && in_arena) {
                const Device &d = devs_[mine[q]];
                const int64_t top = d.arena_bytes - 2 * (int64_t)bytes;
                ok = top >= round_up(d.arena_top, 1024);
                if (ok) {
                    din[q] = d.arena + top;
                    dout[q] = d.arena + top + bytes;
                }
            } else if (ok) {
                ok = cudaMalloc(&din[q], bytes) == cudaSuccess && cudaMalloc(&dout[q], bytes) == cudaSuccess;
            }
        }
        if (rank_mode_) {
            SessionRank &me = sess_->hdr()->rank[rank_];
            me.host_probe_bytes = ok ? (int64_t)bytes : 0;
            if (!sess_->barrier(300.0)) {
                release();
                set_error("rank mode: a peer failed during the host-link probe");
                return XK_ERR_CUDA;
            }
            for (int g = 0; g < G; ++g) ok = ok && sess_->hdr()->rank[g].host_probe_bytes == (int64_t)bytes;
            if (!sess_->barrier(300.0)) {  // everyone has read the flags before they change
                release();
                set_error("rank mode: a peer failed during the host-link probe");
                return XK_ERR_CUDA;
            }
        }
        if (ok) break;
        release();
        if (bytes / 2 < ((size_t)64 << 20)) {
            set_error("xk_probe_host_links: cannot allocate the probe buffers");
            return XK_ERR_OOM;
        }
        bytes /= 2;
    }
    // the measurement; on any failure the buffers are still released below
    auto measure = [&]() -> int {
        for (size_t q = 0; q < n; ++q) {  // touch the pages (first-touch cost outside the timing)
            std::memset(hin[q], 1, bytes);
            std::memset(hout[q], 0, bytes);
            cudaSetDevice(devs_[mine[q]].phys);
            cudaMemset(din[q], 0, bytes);
            cudaMemset(dout[q], 0, bytes);
        }
        auto sync_mine = [&]() -> int {
            for (size_t q = 0; q < n; ++q) {
                Device &d = devs_[mine[q]];
                XK_CK(cudaStreamSynchronize(d.h2d));
                XK_CK(cudaStreamSynchronize(d.d2h));
            }
            return XK_OK;
        };
        for (size_t q = 0; q < n; ++q) {
            XK_CK(cudaSetDevice(devs_[mine[q]].phys));
            XK_CK(cudaDeviceSynchronize());
        }
        for (int pat = 0; pat < 3; ++pat) {  // 0 H2D, 1 D2H, 2 both
            double best = 1e300;
            for (int rep = 0; rep < 3; ++rep) {
                if (rank_mode_ && !sess_->barrier(300.0)) {
                    set_error("rank mode: a peer failed during the host-link probe");
                    return XK_ERR_CUDA;
                }
                auto t0 = std::chrono::steady_clock::now();
                for (size_t q = 0; q < n; ++q) {
                    Device &d = devs_[mine[q]];
                    XK_CK(cudaSetDevice(d.phys));
                    if (pat != 1) XK_CK(cudaMemcpyAsync(din[q], hin[q], bytes, cudaMemcpyHostToDevice, d.h2d));
                    if (pat != 0) XK_CK(cudaMemcpyAsync(hout[q], dout[q], bytes, cudaMemcpyDeviceToHost, d.d2h));
                }
                if ((rc = sync_mine())) return rc;
                double ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
                if (rep > 0) best = std::min(best, ms);
            }
            double tot_bytes = (double)bytes * (pat == 2 ? 2 : 1) * (double)n, tmax = best;
            if (rank_mode_) {  // aggregate over ranks: all bytes / the slowest rank's time
                SessionRank &me = sess_->hdr()->rank[rank_];
                me.host_probe_ms = best;
                me.host_probe_bytes = (int64_t)bytes;
                if (!sess_->barrier(300.0)) {
                    set_error("rank mode: a peer failed during the host-link probe");
                    return XK_ERR_CUDA;
                }
                tot_bytes = 0;
                tmax = 0;
                for (int g = 0; g < G; ++g) {
                    const SessionRank &r = sess_->hdr()->rank[g];
                    tot_bytes += (double)r.host_probe_bytes * (pat == 2 ? 2 : 1);
                    tmax = std::max(tmax, r.host_probe_ms);
                }
            }
            host_all_MBps[pat] = (int64_t)(tot_bytes / (tmax * 1e-3) / 1e6);
        }
        return XK_OK;
    };
    rc = measure();
    if (rc) {
        release();
        return rc;
    }
    host_probe_bytes = (int64_t)bytes;
    release();
    if (rank_mode_ && !sess_->barrier(300.0)) {
        set_error("rank mode: a peer failed during the host-link probe");
        return XK_ERR_CUDA;
    }
    return XK_OK;
}

int Runtime::register_host(void *p, size_t bytes) {
    std::lock_guard<std::recursive_mutex> lk(mu);
    if (!p || bytes == 0) return XK_OK;
    cudaError_t e = cudaHostRegister(p, bytes, cudaHostRegisterPortable);
    if (e == cudaErrorHostMemoryAlreadyRegistered) {
        cudaGetLastError();
        return XK_OK;
    }
    if (e != cudaSuccess) return cuda_fail(e, "cudaHostRegister");
    registered_[(uintptr_t)p] = bytes;
    return XK_OK;
}

int Runtime::unregister_host(void *p) {
    std::lock_guard<std::recursive_mutex> lk(mu);
    auto it = registered_.find((uintptr_t)p);
    if (it == registered_.end()) return XK_OK;
    int rc = sync_all();
    if (rc) return rc;
    registered_.erase(it);
    XK_CK(cudaHostUnregister(p));
    return XK_OK;
}

void Runtime::release_invalid() {
    // in id order: the free lists (and so every later placement) come out the same in
    // every process of rank mode
    std::vector<int64_t> ids;
    for (auto &kv : bufs_) {
        int key = (int)(kv.first / XK_MAX_GPUS), g = (int)(kv.first % XK_MAX_GPUS);
        if (!planner_->entry(key).gpu[g].present) ids.push_back(kv.first);
    }
    std::sort(ids.begin(), ids.end());
    for (int64_t id : ids) {
        Buffer &b = bufs_[id];
        free_buf((int)(id % XK_MAX_GPUS), b.p, b.bytes);
        bufs_.erase(id);
    }
}

int Runtime::wait_stream(cudaStream_t s) {
    if (!rank_mode_) {
        XK_CK(cudaStreamSynchronize(s));
        return XK_OK;
    }
    // a stream may wait on a peer's completion flag: never block without watching the
    // session's abort flag
    for (int spins = 0;; ++spins) {
        cudaError_t e = cudaStreamQuery(s);
        if (e == cudaSuccess) return XK_OK;
        if (e != cudaErrorNotReady) return cuda_fail(e, "cudaStreamQuery");
        if (sess_->aborted()) {
            set_error("rank mode: a peer process failed");
            return XK_ERR_CUDA;
        }
        if (spins > 200) std::this_thread::sleep_for(std::chrono::microseconds(20));
    }
}

int Runtime::wait_event(cudaEvent_t ev) {
    if (!rank_mode_) {
        XK_CK(cudaEventSynchronize(ev));
        return XK_OK;
    }
    for (int spins = 0;; ++spins) {
        cudaError_t e = cudaEventQuery(ev);
        if (e == cudaSuccess) return XK_OK;
        if (e != cudaErrorNotReady) return cuda_fail(e, "cudaEventQuery");
        if (sess_->aborted()) {
            set_error("rank mode: a peer process failed");
            return XK_ERR_CUDA;
        }
        if (spins > 200) std::this_thread::sleep_for(std::chrono::microseconds(20));
    }
}

int Runtime::sync_all() {
    int rc;
    for (size_t g = 0; g < devs_.size(); ++g) {
        Device &d = devs_[g];
        if (!d.local) continue;
        XK_CK(cudaSetDevice(d.phys));
        if ((rc = wait_stream(d.h2d)) || (rc = wait_stream(d.p2p))) return rc;
        for (int k = 0; k < nks_; ++k)
            if ((rc = wait_stream(d.ks[k]))) return rc;
        if ((rc = wait_stream(d.kdiag)) || (rc = wait_stream(d.d2h))) return rc;
    }
    cur_dev_ = -1;
    if (rank_mode_) {
        // every process's streams are idle: every record planned so far has completed
        if (!sess_->barrier()) {
            set_error("rank mode: a peer process failed or timed out at a synchronisation point");
            return XK_ERR_CUDA;
        }
        if (planner_) epoch_seq_ = planner_->next_seq();
    }
    if (tracing_) trace_collect();
    for (size_t q = 0; q < ktimers_.size(); ++q) {
        float ms = 0;
        if (cudaEventElapsedTime(&ms, ktimers_[q].first, ktimers_[q].second) == cudaSuccess) {
            stats.kernel_ms_total += ms;
            stats.kernel_timed_flops += ktimer_flops_[q];
            stats.kernel_timed_launches++;
        }
        cudaEventDestroy(ktimers_[q].first);
        cudaEventDestroy(ktimers_[q].second);
    }
    ktimers_.clear();
    ktimer_flops_.clear();
    // every event of this epoch completed: recycle them
    seq_ev_.clear();
    pending_d2h_.clear();
    for (auto &kv : bufs_) {
        kv.second.writer = Ev();
        kv.second.readers.clear();
    }
    for (size_t g = 0; g < devs_.size(); ++g) {
        if (!devs_[g].local) continue;
        for (cudaEvent_t e : ev_used_[g]) ev_pool_[g].push_back(e);
        ev_used_[g].clear();
    }
    for (auto &sc : scratch_) free_buf(sc.first, sc.second.first, sc.second.second);
    scratch_.clear();
    release_internal_pins();
    return XK_OK;
}

int Runtime::run(const xk_call_t &call, bool wait) {
    std::lock_guard<std::recursive_mutex> lk(mu);
    if (failed_) {
        set_error("an earlier CUDA failure left the tile cache inconsistent: xk_finalize() and xk_init() again");
        return failed_;
    }
    cur_dev_ = -1;
    int rc = XK_OK;
    // rank mode: keep the records in flight well inside the completion-flag ring (every
    // process takes this branch at the same call: the plans are identical)
    if (rank_mode_ && call.routine != XK_ROUTINE_SYNC && planner_->next_seq() - epoch_seq_ > (int64_t)(kFlagCap / 4))
        rc = sync_all();
    if (!rc) rc = run_impl(call, wait);
    if (rc && rank_mode_ && sess_) sess_->abort();
    // after a runtime failure mid-call the directory may describe copies that were never
    // made: refuse further work until re-initialisation (never compute on a stale cache)
    if (rc == XK_ERR_CUDA || rc == XK_ERR_OOM || rc == XK_ERR_INTERNAL) failed_ = rc;
    return rc;
}

int Runtime::run_impl(const xk_call_t &call, bool wait) {
    int rc;
    // page-lock the operands the call touches (excluded from timings when the caller
    // registered them first with xk_register)
    {
        const bool ta = call.transA == 'T' || call.transA == 'C', tb = call.transB == 'T' || call.transB == 'C';
        const bool left = call.side == 'L';
        const int64_t m = call.m, n = call.n, k = call.k;
        auto pin = [&](uint64_t p, int64_t r, int64_t c, uint64_t ld) { return ensure_pinned(p, r, c, (int64_t)ld); };
        switch (call.routine) {
        case XK_ROUTINE_DGEMM:
            if (call.alpha != 0.0 && k > 0) {
                if ((rc = pin(call.A, ta ? k : m, ta ? m : k, call.lda))) return rc;
                if ((rc = pin(call.B, tb ? n : k, tb ? k : n, call.ldb))) return rc;
            }
            break;
        case XK_ROUTINE_DSYRK:
        case XK_ROUTINE_DSYR2K:
            if (call.alpha != 0.0 && k > 0) {
                if ((rc = pin(call.A, ta ? k : n, ta ? n : k, call.lda))) return rc;
                if (call.routine == XK_ROUTINE_DSYR2K && (rc = pin(call.B, ta ? k : n, ta ? n : k, call.ldb))) return rc;
            }
            break;
        case XK_ROUTINE_DSYMM:
            if (call.alpha != 0.0) {
                if ((rc = pin(call.A, left ? m : n, left ? m : n, call.lda))) return rc;
                if ((rc = pin(call.B, m, n, call.ldb))) return rc;
            }
            break;
        case XK_ROUTINE_DTRMM:
        case XK_ROUTINE_DTRSM:
            if (call.alpha != 0.0 && (rc = pin(call.A, left ? m : n, left ? m : n, call.lda))) return rc;
            break;
        default:
            break;
        }
    }
    {
        const bool sy = call.routine == XK_ROUTINE_DSYRK || call.routine == XK_ROUTINE_DSYR2K;
        if ((rc = ensure_pinned(call.C, sy ? call.n : call.m, call.n, (int64_t)call.ldc))) return rc;
    }
    std::vector<Rec> recs;
    std::string err;
    size_t d2h0 = pending_d2h_.size();
    std::fill(batches_in_call_.begin(), batches_in_call_.end(), 0);
    // records are issued as the planner produces them: the GPUs start on the first copies
    // and tasks while the rest of the call is still being planned
    Planner::Sink sink = [this](const Rec &r) {
        stats.plan_records++;
        if (here(r.r)) stats.plan_records_local++;
        return issue(r);
    };
    const auto t_issue = std::chrono::steady_clock::now();
    rc = planner_->plan(call, recs, err, &sink);
    if (rc) {
        if (rc != XK_ERR_CUDA && rc != XK_ERR_OOM) set_error(err);
        return rc;
    }
    for (size_t g = 0; g < batch_.size(); ++g)
        if ((rc = flush_batch((int)g))) return rc;
    stats.host_issue_ms += std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t_issue).count();
    if (call.routine == XK_ROUTINE_SYNC) {
        // xk_sync: everything issued has completed (the API synchronised first), so tiles the
        // planner dropped -- e.g. a call's shadow copies of C -- can go back to the pool
        release_invalid();
        return XK_OK;
    }
    if (call.routine <= XK_ROUTINE_DTRSM && call.sync) {
        // the planner already passed its full sync point and invalidated the operands
        if ((rc = sync_all())) return rc;
        release_invalid();
        return XK_OK;
    }
    if (wait) {
        for (size_t q = d2h0; q < pending_d2h_.size(); ++q)
            if ((rc = wait_event(pending_d2h_[q].e))) return rc;
        // rank mode: the host view is coherent once every process's write-backs landed
        if (rank_mode_ && !sess_->barrier()) {
            set_error("rank mode: a peer process failed or timed out at a synchronisation point");
            return XK_ERR_CUDA;
        }
    }
    return XK_OK;
}

int Runtime::invalidate(uint64_t base, int64_t m, int64_t n, int64_t ld) {
    std::lock_guard<std::recursive_mutex> lk(mu);
    int rc = sync_all();
    if (rc) return rc;
    xk_call_t c{};
    c.routine = XK_ROUTINE_SYNC;
    std::vector<Rec> recs;
    std::string err;
    planner_->plan(c, recs, err);
    planner_->invalidate(base, m, n, ld);
    release_invalid();
    return XK_OK;
}

int Runtime::finalize() {
    std::lock_guard<std::recursive_mutex> lk(mu);
    if (tracing_) trace_stop();
    const bool peer_failed = rank_mode_ && sess_ && sess_->aborted();
    if (peer_failed && sess_->flags()) {
        // a peer died mid-call: release every stream still waiting on one of its flags
        // (values far ahead of any pending seq pass the cyclic GEQ) so the local work drains
        // and the arena can be freed; the session is unusable from here on
        const uint32_t v = (uint32_t)(planner_ ? planner_->next_seq() : 0) + (1u << 30);
        uint32_t *f = sess_->flags();
        for (uint32_t i = 0; i < kFlagCap; ++i) __atomic_store_n(f + i, v, __ATOMIC_RELAXED);
        std::atomic_thread_fence(std::memory_order_seq_cst);
    }
    int rc = peer_failed ? XK_ERR_CUDA : sync_all();
    if (rank_mode_) {
        // close the mappings of the peers' arenas before anyone frees its own
        for (Device &d : devs_)
            if (!d.local && d.arena) cudaIpcCloseMemHandle(d.arena);
        if (sess_ && !peer_failed) sess_->barrier(120.0);
    }
    for (size_t g = 0; g < devs_.size(); ++g) {
        Device &d = devs_[g];
        if (!d.local) continue;
        cudaSetDevice(d.phys);
        if (rank_mode_ && d.arena) cudaFree(d.arena);
        d.arena = nullptr;
        for (auto &pb : d.all_bufs) cudaFree(pb.first);
        d.all_bufs.clear();
        d.free_bufs.clear();
        cudaStreamDestroy(d.h2d);
        cudaStreamDestroy(d.d2h);
        cudaStreamDestroy(d.p2p);
        for (int k = 0; k < nks_; ++k) cudaStreamDestroy(d.ks[k]);
        if (d.kdiag) cudaStreamDestroy(d.kdiag);
        for (cudaEvent_t e : ev_pool_[g]) cudaEventDestroy(e);
    }
    bufs_.clear();
    release_internal_pins();
    for (auto &kv : registered_) cudaHostUnregister((void *)kv.first);
    registered_.clear();
    if (sess_) {
        if (sess_->flags()) cudaHostUnregister(sess_->flags());
        cudaGetLastError();
        sess_->close(rank_ == 0);
        sess_.reset();
    }
    planner_.reset();
    devs_.clear();
    return rc;
}

}  // namespace xk
