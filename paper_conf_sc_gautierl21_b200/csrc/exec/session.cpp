// session.cpp -- shared control file of rank mode (see session.h).
#include "exec/session.h"

#include <cuda.h>
#include <fcntl.h>
#include <sys/mman.h>
#include <sys/stat.h>
#include <unistd.h>

#include <cerrno>
#include <chrono>
#include <cstring>
#include <thread>

namespace xk {

namespace {
constexpr uint64_t kMagic = 0x786b2d72616e6b31ull;  // "xk-rank1"
constexpr size_t kHeaderBytes = (size_t)1 << 20;   // header page(s); flags start here

static_assert(sizeof(SessionHeader) <= kHeaderBytes, "session header too large");

double now_s() {
    using namespace std::chrono;
    return duration<double>(steady_clock::now().time_since_epoch()).count();
}

void pause_briefly(int &spins) {
    if (++spins < 2000) return;  // hot spin first: barriers sit between GPU waits
    std::this_thread::sleep_for(std::chrono::microseconds(50));
}

typedef CUresult (*WaitFn)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);
typedef CUresult (*WriteFn)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);
WaitFn g_wait = nullptr;
WriteFn g_write = nullptr;

void load_memops() {
    static bool tried = false;
    if (tried) return;
    tried = true;
    void *p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuStreamWaitValue32", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
        g_wait = reinterpret_cast<WaitFn>(p);
    p = nullptr;
    if (cudaGetDriverEntryPoint("cuStreamWriteValue32", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
        g_write = reinterpret_cast<WriteFn>(p);
    cudaGetLastError();
}
}  // namespace

bool stream_memops_available() {
    load_memops();
    return g_wait && g_write;
}

cudaError_t stream_write_flag(cudaStream_t s, uint32_t *dev_addr, uint32_t value) {
    load_memops();
    if (!g_write) return cudaErrorNotSupported;
    return g_write((CUstream)s, (CUdeviceptr)dev_addr, value, 0) == CUDA_SUCCESS ? cudaSuccess
                                                                                   : cudaErrorLaunchFailure;
}

cudaError_t stream_wait_flag(cudaStream_t s, uint32_t *dev_addr, uint32_t value) {
    load_memops();
    if (!g_wait) return cudaErrorNotSupported;
    return g_wait((CUstream)s, (CUdeviceptr)dev_addr, value, CU_STREAM_WAIT_VALUE_GEQ) == CUDA_SUCCESS
               ? cudaSuccess
               : cudaErrorLaunchFailure;
}

Session::~Session() { close(false); }

int Session::open(const std::string &path, int rank, int world, double timeout_s, std::string &err) {
    rank_ = rank;
    world_ = world;
    path_ = path;
    map_bytes_ = kHeaderBytes + (size_t)kFlagCap * 4;
    int fd = -1;
    const double t0 = now_s();
    if (rank == 0) {
        fd = ::open(path.c_str(), O_CREAT | O_EXCL | O_RDWR, 0600);
        if (fd < 0) {
            err = "rank mode: cannot create session file " + path + " (" + std::strerror(errno) +
                  "; the path must be unique per session)";
            return XK_ERR_CONFIG;
        }
        if (ftruncate(fd, (off_t)map_bytes_) != 0) {
            err = "rank mode: ftruncate(session) failed: " + std::string(std::strerror(errno));
            ::close(fd);
            return XK_ERR_CONFIG;
        }
    } else {
        for (int spins = 0;;) {
            fd = ::open(path.c_str(), O_RDWR);
            if (fd >= 0) {
                struct stat st;
                if (fstat(fd, &st) == 0 && (size_t)st.st_size == map_bytes_) break;
                ::close(fd);
                fd = -1;
            }
            if (now_s() - t0 > timeout_s) {
                err = "rank mode: timed out waiting for rank 0 to create " + path;
                return XK_ERR_CONFIG;
            }
            pause_briefly(spins);
        }
    }
    map_ = mmap(nullptr, map_bytes_, PROT_READ | PROT_WRITE, MAP_SHARED, fd, 0);
    ::close(fd);
    if (map_ == MAP_FAILED) {
        map_ = nullptr;
        err = "rank mode: mmap(session) failed";
        return XK_ERR_CONFIG;
    }
    h_ = reinterpret_cast<SessionHeader *>(map_);
    flags_ = reinterpret_cast<uint32_t *>(static_cast<char *>(map_) + kHeaderBytes);
    if (rank == 0) {
        h_->world = world;
        std::atomic_thread_fence(std::memory_order_release);
        __atomic_store_n(&h_->magic, kMagic, __ATOMIC_RELEASE);
    } else {
        for (int spins = 0; __atomic_load_n(&h_->magic, __ATOMIC_ACQUIRE) != kMagic;) {
            if (now_s() - t0 > timeout_s) {
                err = "rank mode: session file never initialised by rank 0";
                return XK_ERR_CONFIG;
            }
            pause_briefly(spins);
        }
        if (h_->world != world) {
            err = "rank mode: world size differs from rank 0's";
            return XK_ERR_CONFIG;
        }
    }
    return XK_OK;
}

bool Session::barrier(double timeout_s) {
    if (!h_) return false;
    if (world_ <= 1) return true;
    const uint32_t gen = h_->bar_gen.load(std::memory_order_acquire);
    if (h_->bar_count.fetch_add(1, std::memory_order_acq_rel) + 1 == (uint32_t)world_) {
        h_->bar_count.store(0, std::memory_order_relaxed);
        h_->bar_gen.fetch_add(1, std::memory_order_release);
        return true;  // complete: a peer that aborts afterwards is seen at the next wait
    }
    const double t0 = now_s();
    for (int spins = 0; h_->bar_gen.load(std::memory_order_acquire) == gen;) {
        if (aborted()) return false;
        if (now_s() - t0 > timeout_s) {
            abort();
            return false;
        }
        pause_briefly(spins);
    }
    return true;
}

void Session::close(bool unlink_file) {
    if (map_) munmap(map_, map_bytes_);
    map_ = nullptr;
    h_ = nullptr;
    flags_ = nullptr;
    if (unlink_file && !path_.empty()) ::unlink(path_.c_str());
}

}  // namespace xk

// Round r: every rank adds 1 to a per-round counter in the flag area (host memory only),
// then waits at the barrier; after it, all `world` increments must be visible.
extern "C" int xk_session_selftest(const char *path, int rank, int world, int rounds, int abort_at,
                                   double timeout_s, int *flags_out) {
    if (!path || world < 1 || world > XK_MAX_GPUS || rank < 0 || rank >= world || rounds < 0) return XK_ERR_CONFIG;
    xk::Session s;
    std::string err;
    int rc = s.open(path, rank, world, timeout_s, err);
    if (rc) return rc;
    uint32_t *cnt = s.flags();
    for (int r = 0; r < rounds; ++r) {
        if (r == abort_at) {
            s.abort();
            s.close(false);
            return XK_OK;
        }
        __atomic_fetch_add(cnt + r, 1u, __ATOMIC_ACQ_REL);
        if (!s.barrier(timeout_s)) {
            s.close(rank == 0);
            return XK_ERR_CUDA;
        }
        if (flags_out) flags_out[r] = (int)__atomic_load_n(cnt + r, __ATOMIC_ACQUIRE);
    }
    // nobody unmaps before the last reader is done, then rank 0 removes the file
    const bool ok = s.barrier(timeout_s);
    s.close(rank == 0);
    return ok ? XK_OK : XK_ERR_CUDA;
}
