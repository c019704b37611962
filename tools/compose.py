"""Composition of async calls (paper §IV-F) where PCIe matters: G
logical GPUs on the one B200 share one PCIe link.  D = A*B then E = D*C2, either as two
synchronous calls (D goes back to the host and is re-read) or as two async calls with only E
made coherent (D stays in the GPU caches and moves by peer forwarding).

ROUTINE=trsm: the paper's TRSM+GEMM composition (Figs. 8/9): X = alpha L^-1 B
(left, lower, N, non-unit), then E = X * C2 -- two synchronous calls vs two async calls with
only E made coherent (X never returns to the host before the GEMM reads it)."""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import inputs
import paper_conf_sc_gautierl21_b200 as xk

N = int(os.environ.get("N", 16384)); T = int(os.environ.get("T", 2048)); G = int(os.environ.get("G", 8))
R = os.environ.get("ROUTINE", "gemm")
A, B, C2 = inputs.uniform(1, N, N), inputs.uniform(2, N, N), inputs.uniform(6, N, N)
if R == "trsm":
    A = inputs.tri_dd(4, N, lower=True, fill=0.0)
    B0 = B.copy(order="F")
D, E = np.zeros((N, N), order="F"), np.zeros((N, N), order="F")
xk.init(ngpus=G, phys=[0] * G, tile=T, probe=True)
for X in (A, B, C2, D, E):
    xk.register(X)
xk.dgemm("N", "N", N, N, N, 1.0, A, N, B, N, 0.0, D, N)
res = {}
for mode in ("sync", "async", "sync", "async"):
    xk.reset_stats()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    if R == "trsm":
        np.copyto(D, B0)  # the solve is in place: D holds B, becomes X (untimed reset)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
    if mode == "sync":
        if R == "trsm":
            xk.dtrsm("L", "L", "N", "N", N, N, 1.5, A, N, D, N)
        else:
            xk.dgemm("N", "N", N, N, N, 1.0, A, N, B, N, 0.0, D, N)
        xk.dgemm("N", "N", N, N, N, 1.0, D, N, C2, N, 0.0, E, N)
    else:
        if R == "trsm":
            xk.dtrsm("L", "L", "N", "N", N, N, 1.5, A, N, D, N, asynchronous=True)
        else:
            xk.dgemm_async("N", "N", N, N, N, 1.0, A, N, B, N, 0.0, D, N)
        xk.dgemm_async("N", "N", N, N, N, 1.0, D, N, C2, N, 0.0, E, N)
        xk.memory_coherent_sync(N, N, E, N)
        xk.sync()
        xk.memory_invalidate(N, N, D, N)
        xk.memory_invalidate(N, N, A, N); xk.memory_invalidate(N, N, B, N)
        xk.memory_invalidate(N, N, C2, N); xk.memory_invalidate(N, N, E, N)
    torch.cuda.synchronize()
    dt = time.perf_counter() - t0
    st = xk.get_stats()
    fl = (1.0 if R == "trsm" else 2.0) * N ** 3 + 2.0 * N ** 3
    res[mode] = {"tflops": fl / dt / 1e12, "ms": dt * 1e3, "h2d_GB": sum(st["h2d_bytes"]) / 1e9,
                 "d2h_GB": sum(st["d2h_bytes"]) / 1e9, "p2p_GB": sum(st["p2p_in_bytes"]) / 1e9}
xk.finalize()
out = {"routine": R, "N": N, "tile": T, "logical_gpus": G, "two_sync_calls": res["sync"], "async_composed": res["async"]}
print(json.dumps(out))
