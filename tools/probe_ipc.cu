// probe_ipc.cu -- feasibility probe for the one-process-per-GPU executor (rank mode):
// two processes on the SAME device (the GPU box has one), a CUDA IPC handle to a device
// buffer, and cross-process ordering through stream memory operations on a shared,
// host-registered flag page (cuStreamWaitValue32 / cuStreamWriteValue32).  The waiter
// enqueues its wait BEFORE the producer writes the flag, which is exactly the case a
// cudaStreamWaitEvent cannot express.
//   nvcc -gencode arch=compute_100a,code=sm_100a -o tools/probe_ipc tools/probe_ipc.cu -lcuda
#include <cuda.h>
#include <cuda_runtime.h>
#include <fcntl.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <sys/mman.h>
#include <sys/wait.h>
#include <unistd.h>

#include <atomic>
#include <chrono>
#include <thread>

struct Shm {
    cudaIpcMemHandle_t h;
    std::atomic<int> published;
    std::atomic<int> stage;
    alignas(4096) uint32_t flags[1024];
};

#define CK(x)                                                                      \
    do {                                                                           \
        cudaError_t e = (x);                                                       \
        if (e != cudaSuccess) {                                                    \
            printf("[%d] %s: %s\n", rank, #x, cudaGetErrorString(e));              \
            exit(1);                                                               \
        }                                                                          \
    } while (0)
#define CKD(x)                                                                     \
    do {                                                                           \
        CUresult e = (x);                                                          \
        if (e != CUDA_SUCCESS) {                                                   \
            const char *s = nullptr;                                               \
            cuGetErrorString(e, &s);                                               \
            printf("[%d] %s: %s\n", rank, #x, s ? s : "?");                        \
            exit(1);                                                               \
        }                                                                          \
    } while (0)

__global__ void fill(double *p, size_t n, double v) {
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
        p[i] = v + (double)(i % 1000);
}

static int run(int rank, Shm *shm) {
    const size_t n = (size_t)16 << 20, bytes = n * 8;  // 128 MiB
    CK(cudaSetDevice(0));
    CK(cudaHostRegister(shm->flags, sizeof(shm->flags), cudaHostRegisterPortable | cudaHostRegisterMapped));
    uint32_t *dflags = nullptr;
    CK(cudaHostGetDevicePointer((void **)&dflags, shm->flags, 0));
    int dev = 0, v1 = 0, v2 = 0;
    cuDeviceGet(&dev, 0);
    cuDeviceGetAttribute(&v1, CU_DEVICE_ATTRIBUTE_CAN_USE_STREAM_WAIT_VALUE_NOR, dev);
    cuDeviceGetAttribute(&v2, CU_DEVICE_ATTRIBUTE_CAN_USE_64_BIT_STREAM_MEM_OPS, dev);
    cudaStream_t s;
    CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
    if (rank == 0) {
        printf("[0] attrs: wait_value_nor=%d 64bit_memops=%d\n", v1, v2);
        double *buf;
        CK(cudaMalloc(&buf, bytes));
        CK(cudaIpcGetMemHandle(&shm->h, buf));
        shm->published.store(1);
        while (shm->stage.load() < 1) std::this_thread::sleep_for(std::chrono::milliseconds(1));
        // the peer has enqueued its wait already; produce after a delay
        std::this_thread::sleep_for(std::chrono::milliseconds(200));
        fill<<<592, 256, 0, s>>>(buf, n, 7.0);
        CKD(cuStreamWriteValue32((CUstream)s, (CUdeviceptr)&dflags[0], 1, 0));
        // WAR: overwrite only after the peer's copy signalled flag 1
        CKD(cuStreamWaitValue32((CUstream)s, (CUdeviceptr)&dflags[1], 1, CU_STREAM_WAIT_VALUE_GEQ));
        fill<<<592, 256, 0, s>>>(buf, n, -1.0);
        CK(cudaStreamSynchronize(s));
        printf("[0] done\n");
        CK(cudaFree(buf));
    } else {
        while (shm->published.load() < 1) std::this_thread::sleep_for(std::chrono::milliseconds(1));
        double *rbuf = nullptr, *loc = nullptr;
        auto t0 = std::chrono::steady_clock::now();
        CK(cudaIpcOpenMemHandle((void **)&rbuf, shm->h, cudaIpcMemLazyEnablePeerAccess));
        auto t1 = std::chrono::steady_clock::now();
        printf("[1] ipc open %.3f ms\n", std::chrono::duration<double, std::milli>(t1 - t0).count());
        CK(cudaMalloc(&loc, bytes));
        CKD(cuStreamWaitValue32((CUstream)s, (CUdeviceptr)&dflags[0], 1, CU_STREAM_WAIT_VALUE_GEQ));
        CK(cudaMemcpyAsync(loc, rbuf, bytes, cudaMemcpyDeviceToDevice, s));
        CKD(cuStreamWriteValue32((CUstream)s, (CUdeviceptr)&dflags[1], 1, 0));
        shm->stage.store(1);
        CK(cudaStreamSynchronize(s));
        double *h = (double *)malloc(bytes);
        CK(cudaMemcpy(h, loc, bytes, cudaMemcpyDeviceToHost));
        size_t bad = 0;
        for (size_t i = 0; i < n; ++i)
            if (h[i] != 7.0 + (double)(i % 1000)) ++bad;
        printf("[1] copy check: %zu bad of %zu\n", bad, n);
        // bandwidth of IPC D2D copies (same device here)
        cudaEvent_t a, b;
        cudaEventCreate(&a);
        cudaEventCreate(&b);
        cudaEventRecord(a, s);
        for (int r = 0; r < 10; ++r) cudaMemcpyAsync(loc, rbuf, bytes, cudaMemcpyDeviceToDevice, s);
        cudaEventRecord(b, s);
        cudaEventSynchronize(b);
        float ms = 0;
        cudaEventElapsedTime(&ms, a, b);
        printf("[1] ipc D2D %.1f GB/s\n", 10.0 * bytes / (ms * 1e-3) / 1e9);
        // flag round trip latency: write then wait on the same page, 100 times
        cudaEventRecord(a, s);
        for (int r = 0; r < 100; ++r) {
            cuStreamWriteValue32((CUstream)s, (CUdeviceptr)&dflags[2], r + 1, 0);
            cuStreamWaitValue32((CUstream)s, (CUdeviceptr)&dflags[2], r + 1, CU_STREAM_WAIT_VALUE_GEQ);
        }
        cudaEventRecord(b, s);
        cudaEventSynchronize(b);
        cudaEventElapsedTime(&ms, a, b);
        printf("[1] write+wait on host flag: %.2f us each\n", ms * 1e3 / 100);
        free(h);
        bad = bad ? 1 : 0;
        CK(cudaIpcCloseMemHandle(rbuf));
        return (int)bad;
    }
    return 0;
}

int main() {
    Shm *shm = (Shm *)mmap(nullptr, sizeof(Shm), PROT_READ | PROT_WRITE, MAP_SHARED | MAP_ANONYMOUS, -1, 0);
    memset((void *)shm, 0, sizeof(Shm));
    pid_t pid = fork();
    if (pid == 0) { int r = run(1, shm); fflush(stdout); _exit(r); }
    int rc = run(0, shm);
    int st = 0;
    waitpid(pid, &st, 0);
    printf("parent rc=%d child status=%d\n", rc, WEXITSTATUS(st));
    return rc || WEXITSTATUS(st);
}
