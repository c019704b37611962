"""Timing fidelity of the planner's virtual-time model (DESIGN.md §3 "parity unpinned" item).

The planner (plan.cpp) places every record at an integer-ns virtual time from the link matrix
and the task rate the runtime measured at xk_init (get_topology()).  Its byte counts are
pinned exactly; this tool measures how close its *makespan* is to the wall time of the same
synchronous host-resident call on the B200:

  G = 1 (one physical GPU, the only configuration where the model's resources -- one compute
  engine, one H2D and one D2H link -- are the real ones): every routine at BASELINE shapes.
  G = 8 logical GPUs on the one B200 (shared SMs, one shared PCIe link): the model is given the
  measured topology with every per-GPU resource divided by 8 (compute rate, host links, peer
  copy rate) -- an approximation of sharing, reported for the heuristic modes.

Output: one JSON object, predicted vs measured TFLOP/s and their ratio per case.
"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import inputs
import paper_conf_sc_gautierl21_b200 as xk
from paper_conf_sc_gautierl21_b200 import _abi

RT = {"dgemm": _abi.ROUTINE_DGEMM, "dsyrk": _abi.ROUTINE_DSYRK, "dsyr2k": _abi.ROUTINE_DSYR2K,
      "dsymm": _abi.ROUTINE_DSYMM, "dtrmm": _abi.ROUTINE_DTRMM, "dtrsm": _abi.ROUTINE_DTRSM}


def flops(name, N):
    return {"dsyrk": N * N * (N + 1), "dsyr2k": 2 * N * N * N + N, "dtrsm": N * N * N,
            "dtrmm": N * N * N, "dsymm": 2 * N * N * N, "dgemm": 2 * N * N * N}[name]


def user_call(name, N, M, asynchronous=False):
    A, B, C, L = M
    if name == "dsyrk":
        return xk.dsyrk("L", "N", N, N, 1.5, A, N, -0.75, C, N, asynchronous=asynchronous)
    if name == "dsyr2k":
        return xk.dsyr2k("L", "N", N, N, 1.5, A, N, B, N, -0.75, C, N, asynchronous=asynchronous)
    if name == "dsymm":
        return xk.dsymm("L", "L", N, N, 1.5, A, N, B, N, -0.75, C, N, asynchronous=asynchronous)
    if name == "dgemm":
        return xk.dgemm("N", "N", N, N, N, 1.5, A, N, B, N, -0.75, C, N)
    f = xk.dtrsm if name == "dtrsm" else xk.dtrmm
    return f("L", "L", "N", "N", N, N, 1.0, L, N, B, N, asynchronous=asynchronous)


def model_call(name, N, M):
    A, B, C, L = (x.ctypes.data for x in M)
    if name in ("dtrsm", "dtrmm"):
        return xk.make_call(routine=RT[name], uplo="L", side="L", transA="N", diag="N", m=N, n=N, k=N,
                            alpha=1.0, A=L, lda=N, C=B, ldc=N, sync=True)
    if name == "dsymm":
        return xk.make_call(routine=RT[name], uplo="L", side="L", m=N, n=N, k=N, alpha=1.5, beta=-0.75,
                            A=A, lda=N, B=B, ldb=N, C=C, ldc=N, sync=True)
    if name in ("dsyrk", "dsyr2k"):
        return xk.make_call(routine=RT[name], uplo="L", transA="N", m=N, n=N, k=N, alpha=1.5, beta=-0.75,
                            A=A, lda=N, B=B, ldb=N, C=C, ldc=N, sync=True)
    return xk.make_call(m=N, n=N, k=N, alpha=1.5, beta=-0.75, A=A, lda=N, B=B, ldb=N, C=C, ldc=N, sync=True)


def measure(name, N, M, reps=2):
    user_call(name, N, M)  # warm-up
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(reps):
        user_call(name, N, M)
    torch.cuda.synchronize()
    return (time.perf_counter() - t0) / reps


def predict(name, N, T, M, bw, rate, topo="ranked", optimistic=True):
    recs = xk.plan_dump(model_call(name, N, M), bw, rate_mflops=rate, topo=topo, optimistic=optimistic,
                        tile=T, cap=1 << 20)
    return max(r[12] for r in recs) * 1e-9


def main():
    cases = [(n, int(N), int(T)) for n, N, T in
             (c.split(":") for c in os.environ.get(
                 "CASES", "dgemm:16384:2048 dgemm:32768:2048 dgemm:32768:4096 dsyrk:32768:2048 "
                          "dsyr2k:32768:2048 dsymm:32768:2048 dtrmm:32768:2048 dtrsm:32768:2048").split())]
    out = {"g1": [], "g8_logical": []}
    Nmax = max(N for _, N, _ in cases)
    Mx = [inputs.uniform(1, Nmax, Nmax), inputs.uniform(2, Nmax, Nmax), inputs.uniform(3, Nmax, Nmax),
          inputs.tri_dd(4, Nmax, lower=True, fill=0.0)]
    for name, N, T in cases:
        M = [x[:N, :N].copy(order="F") if N < Nmax else x for x in Mx]
        xk.init(ngpus=1, tile=T, probe=True)
        for X in M:
            xk.register(X)
        topo = xk.get_topology()
        meas = measure(name, N, M)
        pred = predict(name, N, T, M, topo["bw_MBps"], topo["task_rate_mflops"])
        xk.finalize()
        f = flops(name, N)
        row = {"routine": name, "N": N, "T": T, "meas_tflops": round(f / meas / 1e12, 2),
               "pred_tflops": round(f / pred / 1e12, 2), "pred_over_meas_time": round(pred / meas, 3),
               "h2d_MBps": topo["bw_MBps"][1][0], "d2h_MBps": topo["bw_MBps"][0][1],
               "rate_mflops": topo["task_rate_mflops"]}
        out["g1"].append(row)
        print(json.dumps(row), flush=True)
    # 8 logical GPUs on the one B200: measured per-mode time vs the model with shared resources
    G = 8
    N, T = int(os.environ.get("N8", 16384)), 2048
    M = [x[:N, :N].copy(order="F") if N < Nmax else x for x in Mx]
    for mode, topo_name, opt in (("full", "ranked", True), ("no_opt", "ranked", False), ("home", "home", True)):
        xk.init(ngpus=G, phys=[0] * G, tile=T, topo=topo_name, optimistic=opt, probe=True)
        for X in M:
            xk.register(X)
        topo = xk.get_topology()
        meas = measure("dgemm", N, M)
        xk.finalize()
        bw = [[v // G if s != d else v for d, v in enumerate(r)] for s, r in enumerate(topo["bw_MBps"])]
        pred = predict("dgemm", N, T, M, bw, topo["task_rate_mflops"] // G, topo=topo_name, optimistic=opt)
        f = flops("dgemm", N)
        row = {"routine": "dgemm", "N": N, "T": T, "mode": mode, "meas_tflops": round(f / meas / 1e12, 2),
               "pred_tflops": round(f / pred / 1e12, 2), "pred_over_meas_time": round(pred / meas, 3)}
        out["g8_logical"].append(row)
        print(json.dumps(row), flush=True)
    print(json.dumps(out))


if __name__ == "__main__":
    main()
