"""BASELINE configs[4] on the one B200 we have: DGEMM N=65536 host-resident with a tile sweep
(P:612-621), and the composed GEMM->GEMM sequence without intermediate coherence:
D = A*B async, E = D*C2 async, coherence of E only -- compared with two synchronous calls
(D written back and re-read).  Context numbers for profiles/ (8-GPU runs need a bigger box).
"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import inputs
import paper_conf_sc_gautierl21_b200 as xk

out = {"gpus": 1}
N = int(os.environ.get("N5", 65536))
tiles = [int(t) for t in os.environ.get("TILES", "1024,2048,4096").split(",")]
REPS = int(os.environ.get("REPS", 2))  # timed calls per tile, after one warm-up (paper: 8)
A = inputs.uniform(1, N, N)
B = inputs.uniform(2, N, N)
C = inputs.uniform(3, N, N)
sweep = {}
for T in tiles:
    xk.init(ngpus=1, tile=T, probe=True)
    for X in (A, B, C):
        xk.register(X)
    xk.dgemm("N", "N", N, N, N, 1.5, A, N, B, N, -0.75, C, N)  # warm-up (tile buffers allocated)
    xk.reset_stats()
    ts = []
    for _ in range(REPS):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        xk.dgemm("N", "N", N, N, N, 1.5, A, N, B, N, -0.75, C, N)
        torch.cuda.synchronize()
        ts.append(time.perf_counter() - t0)
    st = xk.get_stats()
    dt = sum(ts) / len(ts)
    sweep[T] = {"tflops": 2.0 * N ** 3 / dt / 1e12, "s_mean": dt, "s_each": ts,
                "h2d_GB_per_call": sum(st["h2d_bytes"]) / 1e9 / REPS, "timed_calls": REPS,
                "tasks_per_call": sum(st["tasks"]) // REPS, "kernel_launches_per_call": st["kernel_launches"] // REPS}
    print("N=%d T=%d" % (N, T), sweep[T], flush=True)
    xk.finalize()
out["dgemm_n%d_tile_sweep" % N] = sweep
del A, B, C

# composition at N=32768 (host memory: A, B, C2, D, E)
M = int(os.environ.get("NC", 32768))
T = 4096
A = inputs.uniform(1, M, M)
B = inputs.uniform(2, M, M)
C2 = inputs.uniform(6, M, M)
D = np.zeros((M, M), order="F")
E = np.zeros((M, M), order="F")
xk.init(ngpus=1, tile=T, probe=True)
for X in (A, B, C2, D, E):
    xk.register(X)
xk.dgemm("N", "N", M, M, M, 1.0, A, M, B, M, 0.0, D, M)  # warm-up
torch.cuda.synchronize()
t0 = time.perf_counter()
xk.dgemm("N", "N", M, M, M, 1.0, A, M, B, M, 0.0, D, M)
xk.dgemm("N", "N", M, M, M, 1.0, D, M, C2, M, 0.0, E, M)
torch.cuda.synchronize()
t_sync = time.perf_counter() - t0
E_sync = E.copy(order="F")
xk.reset_stats()
torch.cuda.synchronize()
t0 = time.perf_counter()
xk.dgemm_async("N", "N", M, M, M, 1.0, A, M, B, M, 0.0, D, M)
xk.dgemm_async("N", "N", M, M, M, 1.0, D, M, C2, M, 0.0, E, M)
xk.memory_coherent_sync(M, M, E, M)
torch.cuda.synchronize()
t_async = time.perf_counter() - t0
st = xk.get_stats()
xk.finalize()
same = bool(np.array_equal(E, E_sync))
out["composition_n%d" % M] = {
    "two_sync_calls_tflops": 4.0 * M ** 3 / t_sync / 1e12, "two_sync_calls_s": t_sync,
    "async_composed_tflops": 4.0 * M ** 3 / t_async / 1e12, "async_composed_s": t_async,
    "composed_h2d_GB": sum(st["h2d_bytes"]) / 1e9, "composed_d2h_GB": sum(st["d2h_bytes"]) / 1e9,
    "bitwise_equal_to_sync_path": same}
print(json.dumps(out), flush=True)
