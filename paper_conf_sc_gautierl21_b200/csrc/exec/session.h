// session.h -- the shared control file of rank mode (one process per GPU).
//
// Layout (one file mapping, MAP_SHARED, created by rank 0, opened by the others):
//   header  : magic, world, a sense-reversing barrier, an abort flag, and one slot per rank
//             (IPC handle + size of its device tile arena, its physical device's PCI id,
//             its measured row of the link-bandwidth matrix, its FP64 tile rate);
//   flags   : kFlagCap 32-bit completion flags.  Record `seq` of the (identical) plan sets
//             flags[seq % kFlagCap] = seq + 1 from the stream that executed it
//             (cuStreamWriteValue32 after the copy / kernel); a stream of another process
//             that depends on it waits with cuStreamWaitValue32(GEQ, cyclic compare).  The
//             page is host memory registered (mapped) in every process, so a wait may be
//             enqueued before the producing record is even issued -- the ordering hazard a
//             cudaStreamWaitEvent on an IPC event cannot express.
#pragma once
#include <cuda_runtime.h>

#include <atomic>
#include <cstdint>
#include <string>

#include "xk.h"

namespace xk {

constexpr uint32_t kFlagCap = 1u << 22;  // records in flight between two full syncs (< cap/2)

struct SessionRank {
    std::atomic<uint32_t> stage;   // init protocol stage reached by this rank
    int32_t pci;                   // PCI domain/bus/device of its physical GPU
    int64_t arena_proposed;        // bytes this rank could give its arena
    int64_t arena_bytes;           // agreed arena size (rank 0 writes it for all)
    cudaIpcMemHandle_t arena;      // IPC handle of its arena
    int64_t bw_in[XK_MAX_GPUS + 1];  // bw[s][rank] MB/s for s = 0..G-1 peers, G = host
    int64_t bw_to_host;            // bw[rank][host]
    int64_t bw_local;              // bw[rank][rank]
    int64_t rate_mflops;           // FP64 tile-task rate (rank 0's is used)
    uint64_t plan_cfg;             // hash of the plan-shaping configuration (must agree)
    double host_probe_ms;          // xk_probe_host_links: this rank's time for one pattern
    int64_t host_probe_bytes;      // ... and the bytes it moved
};

struct SessionHeader {
    uint64_t magic;
    int32_t world;
    std::atomic<uint32_t> bar_count;
    std::atomic<uint32_t> bar_gen;
    std::atomic<int32_t> aborted;  // a rank failed: barriers return an error instead of hanging
    SessionRank rank[XK_MAX_GPUS];
};

class Session {
public:
    ~Session();
    // rank 0 creates `path` (must not exist), the others wait for it (timeout_s).
    int open(const std::string &path, int rank, int world, double timeout_s, std::string &err);
    void close(bool unlink_file);
    // All ranks arrive; returns false on abort or timeout.
    bool barrier(double timeout_s = 900.0);
    void abort() { if (h_) h_->aborted.store(1); }
    bool aborted() const { return h_ && h_->aborted.load() != 0; }
    SessionHeader *hdr() { return h_; }
    uint32_t *flags() { return flags_; }      // host address of the flag array
    size_t flags_bytes() const { return (size_t)kFlagCap * 4; }
    int rank() const { return rank_; }
    int world() const { return world_; }

private:
    SessionHeader *h_ = nullptr;
    uint32_t *flags_ = nullptr;
    void *map_ = nullptr;
    size_t map_bytes_ = 0;
    std::string path_;
    int rank_ = 0, world_ = 1;
};

// Stream memory operations through the driver entry points (no libcuda link).
bool stream_memops_available();
cudaError_t stream_write_flag(cudaStream_t s, uint32_t *dev_addr, uint32_t value);
cudaError_t stream_wait_flag(cudaStream_t s, uint32_t *dev_addr, uint32_t value);

}  // namespace xk
