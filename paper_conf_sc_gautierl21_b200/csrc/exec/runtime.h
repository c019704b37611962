// runtime.h -- the executor behind the C ABI: logical GPUs, per-GPU streams (one H2D, one
// D2H, one P2P-in, k kernel streams -- "one stream per operation type", PAPER.md
// P:316-321), the device tile cache (compact column-major tiles), events for
// the plan's point-to-point dependencies, and the issue loop that turns plan
// records into cudaMemcpy2DAsync / peer copies / tile-kernel launches.
#pragma once
#include <cuda_runtime.h>

#include <cstdint>
#include <map>
#include <memory>
#include <mutex>
#include <string>
#include <unordered_map>
#include <vector>

#include "kernels/kernels.h"
#include "exec/session.h"
#include "plan/plan.h"
#include "xk.h"

namespace xk {

constexpr int kMaxKStreams = 8;

struct Ev {
    cudaEvent_t e = nullptr;
    cudaStream_t s = nullptr;  // stream it was recorded on
    uint64_t c = 0;            // ordinal of the record on that stream (1, 2, ...)
    int64_t rseq = -1;         // rank mode: plan record executed by another process (flag wait)
    static Ev remote(int64_t seq) { Ev v; v.rseq = seq; return v; }
};

// A device tile: compact column-major, ld = rows rounded up to 16 (128-byte columns).
struct Buffer {
    double *p = nullptr;
    int64_t ld = 0;
    size_t bytes = 0;
    Ev writer;                  // last write (copy in or task)
    std::vector<Ev> readers;    // reads since the last write (tasks, P2P out, D2H)
};

// Tile tasks of one GPU waiting to be launched together (grouped GEMM launch).
struct PendingBatch {
    std::vector<Rec> recs;  // copies (records are issued while they are planned)
    std::vector<int64_t> out_ids, in_ids;  // buffer ids written / read
    // D2H write-backs of tiles this batch produces: issued right after the batch launches,
    // so a write-back does not cut the batch short (their source ids are in in_ids)
    std::vector<Rec> deferred;
    char ta = 'N', tb = 'N';
    int op = XK_OP_GEMM;  // GEMM / GEMM_TRI grouped launch, or TRSM_DIAG / TRMM_DIAG sharing keyA
    bool contains_seq(int64_t seq) const {
        for (const Rec &r : recs)
            if (r.r.seq == seq) return true;
        return false;
    }
    bool touches(int64_t id, bool write) const {
        for (int64_t o : out_ids)
            if (o == id) return true;
        if (write)
            for (int64_t i : in_ids)
                if (i == id) return true;
        return false;
    }
};

struct Device {
    int phys = 0;
    bool local = true;    // rank mode: only the process's own GPU has streams
    int pci = 0;          // PCI id of the physical device (rank mode: from the session)
    char *arena = nullptr;       // rank mode: device tile arena (own: cudaMalloc; peer: IPC mapping)
    int64_t arena_bytes = 0, arena_top = 0;
    cudaStream_t h2d = nullptr, d2h = nullptr, p2p = nullptr;
    cudaStream_t ks[kMaxKStreams] = {};
    cudaStream_t kdiag = nullptr;  // highest priority: diagonal-tile ops (critical path of TRSM)
    std::map<size_t, std::vector<double *>> free_bufs;  // caching allocator
    std::vector<std::pair<double *, size_t>> all_bufs;
    size_t bytes_in_use = 0;
};

class Runtime {
public:
    Runtime() = default;
    ~Runtime();
    int init(const xk_config_t &cfg);
    int finalize();

    // One planned call: plan, issue in plan order; `wait` = block until the D2H records
    // of this call completed.  Sync routines pass call.sync = 1 and then release the
    // device copies the planner invalidated.
    int run(const xk_call_t &call, bool wait);
    int sync_all();
    int invalidate(uint64_t base, int64_t m, int64_t n, int64_t ld);

    int probe_host_links(int64_t bytes_per_gpu);  // SURVEY §8(d) concurrent BW_h2d/d2h/duplex
    int64_t host_all_MBps[3] = {0, 0, 0};
    int64_t host_probe_bytes = 0;
    int register_host(void *p, size_t bytes);
    int unregister_host(void *p);
    int ensure_pinned(uint64_t base, int64_t rows, int64_t cols, int64_t ld);

    xk_stats_t stats{};
    bool kernel_timing = false;
    // ---- timeline tracing
    int trace_start(const std::string &path);
    int trace_stop();
    Topology topo;
    std::vector<int> perf_rank;
    std::recursive_mutex mu;

private:
    int run_impl(const xk_call_t &call, bool wait);
    int failed_ = 0;  // sticky runtime failure (XK_ERR_*), cleared by re-initialisation
    int issue(const Rec &r);
    int flush_batch(int g);
    int issue_deferred(int g);
    int flush_for(const Rec &r);
    Buffer *buf(int key, int g, bool create, int *rc);
    void release_invalid();
    cudaEvent_t new_event(int g);
    int wait_on(cudaStream_t s, const Ev &ev);
    int record(cudaStream_t s, int g, Ev *out);
    int wait_dep(cudaStream_t s, int64_t seq);
    int cuda_fail(cudaError_t e, const char *what);
    double *alloc(int g, size_t bytes, int *rc);
    void free_buf(int g, double *p, size_t bytes);
    int probe_topology();
    void release_internal_pins();
    std::vector<uintptr_t> reg_cuts(uintptr_t lo, uintptr_t hi) const;
    int copy_host(bool h2d, double *dev, int64_t dld, char *host, int64_t hld, int64_t rows,
                  int64_t cols, cudaStream_t s);
    int set_dev(int g);
    // ---- rank mode (one process per GPU)
    bool here(const xk_plan_rec_t &r) const {
        return !rank_mode_ || (r.kind == XK_REC_D2H ? r.src : r.dst) == rank_;
    }
    int init_rank_mode(const xk_config_t &cfg);
    int probe_topology_rank();
    int signal(cudaStream_t s, int64_t seq);   // completion flag of a locally executed record
    int wait_stream(cudaStream_t s);           // abort-aware stream synchronisation
    int wait_event(cudaEvent_t e);
    int issue_remote(const Rec &R);
    bool rank_mode_ = false;
    int rank_ = 0;
    std::unique_ptr<Session> sess_;
    uint32_t *dflags_ = nullptr;  // device address of the session's flag array
    int64_t epoch_seq_ = 0;       // records below this completed at the last full sync

    xk_config_t cfg_{};
    Flags flags_;
    std::unique_ptr<Planner> planner_;
    std::vector<Device> devs_;
    std::unordered_map<int64_t, Buffer> bufs_;  // key * XK_MAX_GPUS + g
    std::unordered_map<int64_t, Ev> seq_ev_;    // plan seq -> completion event (this epoch)
    // event-wait deduplication: events recorded per stream, and per (waiting stream, recorded
    // stream) the latest ordinal already waited for -- a stream's events complete in order, so
    // waiting for a later one covers every earlier one
    std::unordered_map<cudaStream_t, uint64_t> rec_count_;
    struct StreamPairHash {
        size_t operator()(const std::pair<cudaStream_t, cudaStream_t> &p) const {
            return std::hash<const void *>()(p.first) * 31u ^ std::hash<const void *>()(p.second);
        }
    };
    std::unordered_map<std::pair<cudaStream_t, cudaStream_t>, uint64_t, StreamPairHash> waited_;
    int64_t waits_skipped_ = 0;
    std::vector<std::vector<cudaEvent_t>> ev_pool_, ev_used_;  // per logical GPU
    std::vector<Ev> pending_d2h_;
    std::vector<std::pair<cudaEvent_t, cudaEvent_t>> ktimers_;
    std::vector<int64_t> ktimer_flops_;
    std::vector<std::pair<int, std::pair<double *, size_t>>> scratch_;
    struct TraceOp {
        int g, kind;  // kind 0 H2D, 1 P2P, 2 kernel, 3 D2H
        cudaEvent_t a, b;
        std::string name;
        int64_t work;
    };
    bool tracing_ = false;
    std::string trace_path_;
    std::vector<cudaEvent_t> trace_base_;  // per logical GPU
    std::vector<TraceOp> trace_ops_;
    std::vector<std::string> trace_json_;
    int trace_begin(int g, cudaStream_t s, cudaEvent_t *a);
    void trace_end(int g, cudaStream_t s, cudaEvent_t a, int kind, std::string name, int64_t work);
    void trace_collect();  // freed at the next full sync
    std::map<uintptr_t, size_t> registered_;    // user-registered host ranges
    std::map<uintptr_t, size_t> internal_reg_;  // registered by the library on first use
    int cur_dev_ = -1;
    std::vector<PendingBatch> batch_;
    std::unordered_map<int64_t, int> deferred_seq_;  // seq of a deferred copy -> GPU of its batch
    bool defer_d2h_ = true;  // XK_DEFER_D2H=0: a write-back launches its batch at once
    int ramp_div_ = 8;       // batch size doubles every ramp_div_ launches at a call's start (XK_RAMP)
    std::vector<int64_t> batch_count_;
    std::vector<int64_t> batches_in_call_;  // grouped launches issued in the current call, per GPU
    int max_batch_ = kMaxBatch;
    int nks_ = 4;  // kernel streams created per GPU
};

Runtime *runtime();  // global instance (nullptr before xk_init)

}  // namespace xk
