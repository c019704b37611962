"""How long does a tile allocation stall the host while the GPU is busy?  cudaMalloc vs
stream-ordered cudaMallocAsync (+ synchronize of its own stream), 32 MiB each, first-time
(pool empty / fresh memory) and with a long kernel queued on another stream."""
import json, time
import torch
from cuda.bindings import runtime as rt
from cuda.bindings import driver as drv

torch.cuda.init()
dev = 0
MB32 = 32 << 20
a = torch.randn(8192, 8192, device="cuda", dtype=torch.float64)


def busy(ms_target=400):
    # queue ~ms_target of FP64 GEMMs on torch's stream
    for _ in range(int(ms_target / 30)):
        torch.mm(a, a)


def timed(fn, n):
    t0 = time.perf_counter()
    for _ in range(n):
        fn()
    return (time.perf_counter() - t0) * 1e3 / n


out = {}
ptrs = []
err, s = rt.cudaStreamCreateWithFlags(rt.cudaStreamNonBlocking)
err, pool = rt.cudaDeviceGetDefaultMemPool(dev)
rt.cudaMemPoolSetAttribute(pool, rt.cudaMemPoolAttr.cudaMemPoolAttrReleaseThreshold, drv.cuuint64_t(2 ** 64 - 1))


def m():
    err, p = rt.cudaMalloc(MB32)
    ptrs.append(p)


def ma():
    err, p = rt.cudaMallocAsync(MB32, s)
    rt.cudaStreamSynchronize(s)
    ptrs.append(p)


for name, fn in (("cudaMalloc", m), ("cudaMallocAsync+sync", ma)):
    torch.cuda.synchronize()
    out[name + "_idle_ms"] = round(timed(fn, 50), 3)
    busy()
    t0 = time.perf_counter()
    per = timed(fn, 50)
    out[name + "_gpu_busy_ms"] = round(per, 3)
    torch.cuda.synchronize()
    out[name + "_busy_region_ms"] = round((time.perf_counter() - t0) * 1e3, 1)
print(json.dumps(out))
