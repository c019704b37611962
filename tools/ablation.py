"""Heuristic ablation (paper Fig. 3 / Table II) on the B200 we have.

G logical GPUs share the one physical B200 (logical-device mode): every logical GPU has its
own tile cache and streams, peer forwarding is a device-to-device copy-engine copy, and all
host pulls share the one PCIe Gen5 link -- the resource the heuristics save.  Modes:
  full        RANKED + optimistic  (XKBlas)
  no_opt      RANKED, optimistic off  (paper "no heuristic")
  no_opt_topo UNRANKED, optimistic off (paper "no heuristic, no topo")
  home        HOME: host first (link-oblivious)
  dod         data-on-device (Table II's first column): operands prefetched onto their
              owners (untimed), async call + xk_sync timed, result left on the GPUs
ROUTINE = dgemm | dsyr2k | dtrsm (Table II's three rows; lower / NoTrans, left-lower-N-nonunit).
Each line: TFLOP/s of the synchronous host-resident call (H2D + D2H timed) and the bytes
per link kind measured by the executor.  Context, not the driver's bench line.
"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import inputs
import paper_conf_sc_gautierl21_b200 as xk

N = int(os.environ.get("N", 16384))
T = int(os.environ.get("T", 2048))
G = int(os.environ.get("G", 8))
REPS = int(os.environ.get("REPS", 3))
R = os.environ.get("ROUTINE", "dgemm")
MODES = [("full", "ranked", True), ("no_opt", "ranked", False), ("no_opt_topo", "unranked", False),
         ("home", "home", True), ("dod", "ranked", True)]
FLOPS = {"dgemm": 2.0 * N ** 3, "dsyr2k": 2.0 * N ** 3 + N, "dtrsm": 1.0 * N ** 3, "dtrmm": 1.0 * N ** 3}[R]

A = inputs.uniform(1, N, N)
B = inputs.uniform(2, N, N)
C = inputs.uniform(3, N, N)
L = inputs.tri_dd(4, N, lower=True, fill=0.0)


def call(asynchronous=False):
    if R == "dgemm":
        return (xk.dgemm_async if asynchronous else xk.dgemm)("N", "N", N, N, N, 1.5, A, N, B, N, -0.75, C, N)
    if R == "dsyr2k":
        return xk.dsyr2k("L", "N", N, N, 1.5, A, N, B, N, -0.75, C, N, asynchronous=asynchronous)
    if R == "dtrmm":
        return xk.dtrmm("L", "L", "N", "N", N, N, 1.0, L, N, B, N, asynchronous=asynchronous)
    return xk.dtrsm("L", "L", "N", "N", N, N, 1.0, L, N, B, N, asynchronous=asynchronous)


out = {"routine": R, "N": N, "tile": T, "logical_gpus": G, "physical_gpus": 1, "modes": {}}
ONLY = os.environ.get("ONLY", "").split()
for name, topo, opt in [m for m in MODES if not ONLY or m[0] in ONLY]:
    xk.init(ngpus=G, phys=[0] * G, tile=T, topo=topo, optimistic=opt, probe=True)
    for X in (A, B, C, L):
        xk.register(X)
    call()  # warm-up
    if name == "dod":
        for X in (A, B, C, L):
            xk.memory_prefetch_async(N, N, X, N)
        xk.sync()
        # a discarded data-on-device warm-up call too: the first one allocates the
        # forwarded tiles' device buffers (316 cudaMalloc for DTRSM N=32768 on 8 logical GPUs,
        # up to ~1 s of host time), which the host-resident warm-up above does not cover
        call(True)
        xk.sync()
    xk.reset_stats()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(REPS):
        if name == "dod":
            call(True)
            xk.sync()
        else:
            call()
    torch.cuda.synchronize()
    dt = (time.perf_counter() - t0) / REPS
    st = xk.get_stats()
    xk.finalize()
    res = {"tflops": FLOPS / dt / 1e12, "ms": dt * 1e3,
           "h2d_GB": sum(st["h2d_bytes"]) / REPS / 1e9, "p2p_GB": sum(st["p2p_in_bytes"]) / REPS / 1e9,
           "d2h_GB": sum(st["d2h_bytes"]) / REPS / 1e9,
           "forwards_inflight": st["forwards_inflight"] // REPS, "forwards_valid": st["forwards_valid"] // REPS,
           "h2d_per_gpu_GB": [round(b / REPS / 1e9, 2) for b in st["h2d_bytes"]]}
    out["modes"][name] = res
    print(name, json.dumps(res), flush=True)
full = out["modes"]["full"]["tflops"] if "full" in out["modes"] else 1.0
out["vs_full_percent"] = {k: round(100.0 * (v["tflops"] / full - 1.0), 1) for k, v in out["modes"].items()}
print(json.dumps(out))
