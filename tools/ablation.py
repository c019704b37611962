"""Heuristic ablation (paper Fig. 3 / Table II) on the B200 we have.

G logical GPUs share the one physical B200 (logical-device mode): every logical GPU has its
own tile cache and streams, peer forwarding is a device-to-device copy-engine copy, and all
host pulls share the one PCIe Gen5 link -- the resource the heuristics save.  Modes:
  full        RANKED + optimistic  (XKBlas)
  no_opt      RANKED, optimistic off  (paper "no heuristic")
  no_opt_topo UNRANKED, optimistic off (paper "no heuristic, no topo")
  home        HOME: host first (link-oblivious)
Each line: TFLOP/s of the synchronous host-resident DGEMM (H2D + D2H timed) and the bytes
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
MODES = [("full", "ranked", True), ("no_opt", "ranked", False), ("no_opt_topo", "unranked", False),
         ("home", "home", True)]

A = inputs.uniform(1, N, N)
B = inputs.uniform(2, N, N)
C = inputs.uniform(3, N, N)
out = {"N": N, "tile": T, "logical_gpus": G, "physical_gpus": 1, "modes": {}}
for name, topo, opt in MODES:
    xk.init(ngpus=G, phys=[0] * G, tile=T, topo=topo, optimistic=opt, probe=True)
    for X in (A, B, C):
        xk.register(X)
    xk.dgemm("N", "N", N, N, N, 1.5, A, N, B, N, -0.75, C, N)  # warm-up
    xk.reset_stats()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(REPS):
        xk.dgemm("N", "N", N, N, N, 1.5, A, N, B, N, -0.75, C, N)
    torch.cuda.synchronize()
    dt = (time.perf_counter() - t0) / REPS
    st = xk.get_stats()
    xk.finalize()
    res = {"tflops": 2.0 * N ** 3 / dt / 1e12, "ms": dt * 1e3,
           "h2d_GB": sum(st["h2d_bytes"]) / REPS / 1e9, "p2p_GB": sum(st["p2p_in_bytes"]) / REPS / 1e9,
           "d2h_GB": sum(st["d2h_bytes"]) / REPS / 1e9,
           "forwards_inflight": st["forwards_inflight"] // REPS, "forwards_valid": st["forwards_valid"] // REPS,
           "h2d_per_gpu_GB": [round(b / REPS / 1e9, 2) for b in st["h2d_bytes"]]}
    out["modes"][name] = res
    print(name, json.dumps(res), flush=True)
print(json.dumps(out))
