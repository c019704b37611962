// plan.h -- the XKBlas planner: tiling, owner-computes map, coherence directory,
// source selection (topology-aware + optimistic forwarding) and the deterministic
// integer virtual-time model that orders copies and tasks.  Pure C++ (no CUDA): the
// same object drives the executor inside libxk.so and xk_plan_dump() for CPU tests.
//
// Paper: directory of tile copies P:408-412; "initiates data transfers of the tile from
// one of the resources handling a valid copy once the scheduler has decided to map a
// task" P:440-442; topology-aware order P:446-451; optimistic in-flight source
// P:491-498; owner-computes P:384-389 on a 2D block-cyclic grid P:743-747.
// Readings are listed in DESIGN.md.
#pragma once
#include <algorithm>
#include <cstdint>
#include <functional>
#include <string>
#include <unordered_map>
#include <vector>

#include "xk.h"

namespace xk {

struct Topology {
    int G = 1;
    std::vector<int64_t> bw;  // (G+1)^2 MB/s, row = src, col = dst, index G = host
    int64_t rate_mflops = 35000000;
    int64_t bw_at(int s, int d) const { return bw[(size_t)s * (G + 1) + d]; }
};

struct Flags {
    int topo = XK_TOPO_RANKED;
    int optimistic = 1;
    int window = 4;
    int P = 1, Q = 1;
    int64_t T = 2048;
    int64_t mem_bytes = 0;  // tile-cache capacity per GPU the plan must fit (0 = unlimited)
};

// A host matrix as the planner sees it: identity (base, ld) and stored extent.
struct Matrix {
    uint64_t base = 0;
    int64_t ld = 0;
    int64_t rows = 0, cols = 0;  // stored extent covered by the tiles known so far
    bool shadow = false;         // per-call read-only view of C's input values (beta deferral)
    bool host_once = false;      // shadow read from the host at most once (R15: TRMM's B)
    // dense (bi, bj) -> directory id cache of keymap_ for this matrix (-1 = not yet looked
    // up); rebuilt when the tile grid grows, cleared when the matrix's entries are forgotten
    std::vector<int> grid;
    int64_t gr = 0, gc = 0;
};

struct NodeCopy {
    bool present = false;
    int64_t ver = 0;
    int64_t t_done = 0;    // virtual time the copy is complete
    int64_t producer = -1; // seq of the record that produced it (-1 = complete/original)
    int depth = 0;
};

struct Entry {
    int mat = -1;
    int64_t bi = 0, bj = 0;
    int64_t rows = 0, cols = 0;  // tile extent (ragged at the edges)
    int64_t ver = 0;             // current (latest planned) version
    NodeCopy host;               // host copy (present & ver == cur -> host valid)
    std::vector<NodeCopy> gpu;   // per GPU
};

// A plan record plus what the executor needs to act on it.
struct Rec {
    xk_plan_rec_t r;
    int key = -1;                 // directory entry id
    int64_t sub_r0 = 0, sub_c0 = 0, sub_rows = 0, sub_cols = 0;  // D2H intersection (tile-relative)
    // task description (TASK records)
    int op = XK_OP_GEMM;
    char ta = 'N', tb = 'N';
    char side = 'L', uplo = 'L', diag = 'N';  // diagonal-tile ops
    int tri = 0;                  // GEMM_TRI / SCALE on a diagonal tile: 1 lower, 2 upper
    double alpha = 1.0, beta = 0.0;
    int keyA = -1, keyB = -1;     // tiles in the kernel's A and B roles on dst (-1: none)
    int keyC2 = -1;               // deferred-beta input tile: D += beta2 * C2 (-1: none)
    double beta2 = 0.0;
    int64_t m = 0, n = 0, k = 0;  // task shape (output rows, cols, inner / triangle order)
    int64_t remaining = 0;        // TASK: tasks after this one on its GPU in this call
};

class Planner {
public:
    Planner(const Topology &t, const Flags &f);

    // Plan one call.  Records go to `sink` as they are produced (the executor issues them
    // while planning continues -- the GPUs start on the first records) or, without a sink,
    // are appended to out.  Returns 0 or XK_ERR_* (a sink error aborts the plan).
    using Sink = std::function<int(const Rec &)>;
    int plan(const xk_call_t &c, std::vector<Rec> &out, std::string &err, const Sink *sink = nullptr);

    // Full synchronisation point (return of a sync routine, xk_sync): every copy is
    // complete, clocks restart at 0.
    void full_sync();
    // Drop GPU copies of the tiles intersecting a view.
    void invalidate(uint64_t base, int64_t m, int64_t n, int64_t ld);
    // Drop the GPU copies of a view's tiles whose host copy is current (end of a sync call).
    void release(uint64_t base, int64_t m, int64_t n, int64_t ld);

    const Entry &entry(int id) const { return entries_[id]; }
    const Matrix &matrix(int id) const { return mats_[id]; }
    int G() const { return topo_.G; }
    // Grouped-launch cap the current call's task structure suits (0 = the executor's
    // default): set before the call's first record is emitted (R19).
    int batch_hint() const { return batch_hint_; }
    int owner(int64_t i, int64_t j) const {
        return (int)((i % flags_.P) * flags_.Q + (j % flags_.Q));
    }
    // Owner of tile (i, j) of a triangular output (SYRK/SYR2K, reading R11): the stored
    // triangle's tiles in column-major order dealt round-robin over the G GPUs
    int owner_tri(int64_t i, int64_t j, bool lower, int64_t t) const {
        const int64_t idx = lower ? j * t - j * (j - 1) / 2 + (i - j) : j * (j + 1) / 2 + i;
        return (int)(idx % topo_.G);
    }
    // Owner of tile (i, j) of TRSM/TRMM's B.  Reading R13: the grid's larger extent goes
    // along the untouched dimension (columns of B for a left-side op, rows for right-side),
    // so the tiles of the row (column) a step solves are spread over more GPUs and the
    // chain of diagonal steps shortens.  Reading R12 (TRMM only): the grid index along the
    // triangular dimension is snaked (0..P-1, P-1..0, ...) -- the work of B's row r grows
    // with r -- which balances the GPUs; TRSM keeps it plain (its diagonal chain binds).
    static int64_t snake(int64_t x, int64_t n) {
        const int64_t blk = x / n, r = x % n;
        return (blk % 2 == 0) ? r : n - 1 - r;
    }
    int owner_trxm(int64_t i, int64_t j, bool left, bool solve) const {
        const int64_t lo = std::min(flags_.P, flags_.Q), hi = std::max(flags_.P, flags_.Q);
        const int64_t Pg = left ? lo : hi, Qg = left ? hi : lo;
        const int64_t pi = (!solve && left) ? snake(i, Pg) : i % Pg;
        const int64_t qj = (!solve && !left) ? snake(j, Qg) : j % Qg;
        return (int)(pi * Qg + qj);
    }
    const Flags &flags() const { return flags_; }
    int64_t next_seq() const { return seq_; }  // seq of the next record to be emitted
    int link_class(int s, int d) const { return cls_[(size_t)s * (topo_.G + 1) + d]; }

private:
    int batch_hint_ = 0;
    struct Input { int key; int64_t ver; int operand; int cnt = -1; };  // cnt: readers slot
    struct Inputs {  // at most 4 inputs per task, no heap allocation
        Input v[4];
        int n = 0;
        void push_back(const Input &x) { v[n++] = x; }
        size_t size() const { return (size_t)n; }
        Input &operator[](size_t i) { return v[i]; }
        const Input &operator[](size_t i) const { return v[i]; }
        Input *begin() { return v; }
        Input *end() { return v + n; }
        const Input *begin() const { return v; }
        const Input *end() const { return v + n; }
    };
    struct Task {
        int gpu = 0;
        int op = XK_OP_GEMM;
        int out_key = -1;
        int64_t out_ver = 0;        // version produced
        Inputs in;                  // inputs in position order (deps follow this order)
        int war = -1;               // readers slot of (out_key, out_ver - 1)
        int keyA = -1, keyB = -1;   // kernel roles
        int keyC2 = -1;             // deferred beta: D += beta2 * (C's input tile)
        double beta2 = 0.0;
        char ta = 'N', tb = 'N', side = 'L', uplo = 'L', diag = 'N';
        int tri = 0;
        double alpha = 1.0, beta = 0.0;
        int64_t tk = 0;             // step index (-1 scale-only)
        int64_t i = 0, j = 0;       // output tile coords
        int64_t m = 0, n = 0, k = 0;
        int64_t flops = 0;
        bool last_writer = false;   // last write of out_key in this call
        int64_t skey[5] = {0, 0, 0, 0, 0};  // per-GPU list order
    };
    // symbolic versions while a call's task list is generated (program order)
    struct Versions {  // flat by directory id: -1 = not written yet in this call
        std::vector<int64_t> cur;
        const std::vector<Entry> *e = nullptr;
        int64_t get(int key) const {
            return ((size_t)key < cur.size() && cur[key] >= 0) ? cur[key] : (*e)[key].ver;
        }
        int64_t bump(int key) {
            const int64_t v = get(key) + 1;
            if ((size_t)key >= cur.size()) cur.resize(std::max(e->size(), (size_t)key + 1), -1);
            cur[key] = v;
            return v;
        }
    };

    int plan_impl(const xk_call_t &c, std::vector<Rec> &out, std::string &err);
    void emit(const Rec &R, std::vector<Rec> &out);
    const Sink *sink_ = nullptr;
    int sink_rc_ = 0;
    int find_or_add_matrix(uint64_t base, int64_t ld, int64_t rows, int64_t cols, std::string &err);
    int key_of(int mat, int64_t bi, int64_t bj);
    static uint64_t tile_key(int mat, int64_t bi, int64_t bj) {
        return ((uint64_t)mat << 48) | ((uint64_t)bi << 24) | (uint64_t)bj;  // < 2^24 tiles per dim
    }
    int64_t dur(int64_t amount, int64_t rate) const;  // ceil(amount*1000/rate) ns
    int select_source(const Entry &e, int64_t ver, int d, int64_t treq, int *state) const;
    bool emit_copy(int key, int64_t ver, int d, int64_t treq, int operand, std::vector<Rec> &out);
    void emit_d2h(int key, int src, int64_t r0, int64_t c0, int64_t rows, int64_t cols,
                  int64_t ready, int64_t dep, int operand, std::vector<Rec> &out);
    // beta deferral (reading Q12''): per-call shadow view of C, its use, and its removal
    int add_shadow(int mc);
    bool defer_beta(int keyC) const;
    void drop_shadow(int ms);
    // capacity check for a shadow plan: every GPU's tiles (resident now + read or written by
    // this call's tasks on it) fit in flags_.mem_bytes
    bool fits(const std::vector<Task> &tasks) const;
    int plan_gemm(const xk_call_t &c, std::vector<Rec> &out, std::string &err);
    int plan_syrk(const xk_call_t &c, bool two, std::vector<Rec> &out, std::string &err);
    int plan_symm(const xk_call_t &c, std::vector<Rec> &out, std::string &err);
    int plan_trxm(const xk_call_t &c, bool solve, std::vector<Rec> &out, std::string &err);
    void finish_call(const xk_call_t &c);
    int plan_coherent(const xk_call_t &c, std::vector<Rec> &out, std::string &err, bool prefetch);
    int run_tasks(std::vector<Task> &tasks, bool sync, std::vector<Rec> &out, std::string &err);
    bool view_tiles(uint64_t base, int64_t m, int64_t n, int64_t ld, int *mat,
                    int64_t *r0, int64_t *c0) const;

    Topology topo_;
    Flags flags_;
    std::vector<int> cls_;
    std::vector<Matrix> mats_;
    std::vector<Entry> entries_;
    std::unordered_map<uint64_t, int> keymap_;  // (mat, bi, bj) packed, see tile_key()
    std::vector<int64_t> link_free_;     // (G+1)^2
    std::vector<int64_t> gpu_free_;      // G
    std::vector<std::vector<int64_t>> ends_;  // per GPU task end-time history (since last sync)
    int64_t seq_ = 0;
};

// Link classes: distinct off-diagonal bandwidths sorted
// ascending, new class when consecutive values differ by a ratio > 1.25.
std::vector<int> link_classes(int G, const std::vector<int64_t> &bw);

}  // namespace xk
