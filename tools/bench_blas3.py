"""Throughput of the other BLAS-3 routines at the BASELINE configs[2]/[3] shape (N=32768,
T=2048) on the visible GPUs -- context numbers for profiles/ (the driver's bench.py line is
DGEMM).  Each routine: one warm-up, then 2 timed synchronous calls from pinned host memory
(end to end, H2D/D2H included) and 2 data-on-device async calls (A/B/C prefetched)."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import inputs
import paper_conf_sc_gautierl21_b200 as xk

N = int(os.environ.get("N", 32768))
T = int(os.environ.get("T", 2048))
G = int(os.environ.get("G", 1))
A = inputs.uniform(1, N, N)
B = inputs.uniform(2, N, N)
C = inputs.uniform(3, N, N)
L = inputs.tri_dd(4, N, lower=True, fill=0.0)
xk.init(ngpus=G, tile=T, probe=True)
for X in (A, B, C, L):
    xk.register(X)
flops = {"dsyrk": N * N * (N + 1), "dsyr2k": 2 * N * N * N + N, "dtrsm": N * N * N, "dtrmm": N * N * N,
         "dsymm": 2 * N * N * N, "dgemm": 2 * N * N * N}


def call(name, asynchronous):
    if name == "dsyrk":
        return xk.dsyrk("L", "N", N, N, 1.5, A, N, -0.75, C, N, asynchronous=asynchronous)
    if name == "dsyr2k":
        return xk.dsyr2k("L", "N", N, N, 1.5, A, N, B, N, -0.75, C, N, asynchronous=asynchronous)
    if name == "dsymm":
        return xk.dsymm("L", "L", N, N, 1.5, A, N, B, N, -0.75, C, N, asynchronous=asynchronous)
    if name == "dgemm":
        f = xk.dgemm_async if asynchronous else xk.dgemm
        return f("N", "N", N, N, N, 1.5, A, N, B, N, -0.75, C, N)
    f = xk.dtrsm if name == "dtrsm" else xk.dtrmm
    return f("L", "L", "N", "N", N, N, 1.0, L, N, B, N, asynchronous=asynchronous)


out = {}
for name in (os.environ.get("ROUTINES") or "dgemm dsyrk dsyr2k dsymm dtrmm dtrsm").split():
    call(name, False)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(2):
        call(name, False)
    torch.cuda.synchronize()
    e2e = 2 * flops[name] / (time.perf_counter() - t0) / 1e12
    for X in (A, B, C, L):
        xk.memory_prefetch_async(N, N, X, N)
    xk.sync()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(2):
        call(name, True)
        xk.sync()
    torch.cuda.synchronize()
    dod = 2 * flops[name] / (time.perf_counter() - t0) / 1e12
    for X in (A, B, C, L):
        xk.memory_coherent_sync(N, N, X, N)
        xk.memory_invalidate(N, N, X, N)
    out[name] = {"e2e_tflops": round(e2e, 2), "device_resident_tflops": round(dod, 2)}
    print(name, out[name], flush=True)
xk.finalize()
print(json.dumps({"N": N, "tile": T, "gpus": G, "routines": out}))
