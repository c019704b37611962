"""Timeline of one host-resident BLAS-3 call (any routine) from the library's own trace
(xk_trace): where the kernel streams sit idle and what the copy streams do meanwhile.

  ROUTINE=dtrsm N=32768 T=2048 python tools/trace_routine.py

Prints a JSON summary: wall time of the call, union of kernel-busy time, the largest idle
gaps of the kernel streams (with the copy traffic inside each gap), and when the H2D / D2H
streams start and finish.  Writes the Chrome trace to gpurun_out/trace_<routine>_n<N>.json."""
import json
import os
import re
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import inputs
import paper_conf_sc_gautierl21_b200 as xk

R = os.environ.get("ROUTINE", "dtrsm")
N = int(os.environ.get("N", 32768))
T = int(os.environ.get("T", 2048))
G = int(os.environ.get("G", 1))
out_dir = os.environ.get("OUT", "gpurun_out")
os.makedirs(out_dir, exist_ok=True)
A = inputs.uniform(1, N, N)
B = inputs.uniform(2, N, N)
C = inputs.uniform(3, N, N)
L = inputs.tri_dd(4, N, lower=True, fill=0.0)
xk.init(ngpus=G, phys=[0] * G, tile=T, probe=True)
for X in (A, B, C, L):
    xk.register(X)
flops = {"dsyrk": N * N * (N + 1), "dsyr2k": 2 * N * N * N + N, "dtrsm": N * N * N, "dtrmm": N * N * N,
         "dsymm": 2 * N * N * N, "dgemm": 2 * N * N * N}[R]


def call():
    if R == "dgemm":
        return xk.dgemm("N", "N", N, N, N, 1.5, A, N, B, N, -0.75, C, N)
    if R == "dsyrk":
        return xk.dsyrk("L", "N", N, N, 1.5, A, N, -0.75, C, N)
    if R == "dsyr2k":
        return xk.dsyr2k("L", "N", N, N, 1.5, A, N, B, N, -0.75, C, N)
    if R == "dsymm":
        return xk.dsymm("L", "L", N, N, 1.5, A, N, B, N, -0.75, C, N)
    f = xk.dtrsm if R == "dtrsm" else xk.dtrmm
    return f("L", "L", "N", "N", N, N, 1.0, L, N, B, N)


DOD = os.environ.get("DOD", "0") == "1"  # data-on-device: operands prefetched, async call + xk_sync


def call_async():
    if R == "dgemm":
        xk.dgemm_async("N", "N", N, N, N, 1.5, A, N, B, N, -0.75, C, N)
    elif R in ("dtrsm", "dtrmm"):
        (xk.dtrsm if R == "dtrsm" else xk.dtrmm)("L", "L", "N", "N", N, N, 1.0, L, N, B, N, asynchronous=True)
    elif R == "dsyrk":
        xk.dsyrk("L", "N", N, N, 1.5, A, N, -0.75, C, N, asynchronous=True)
    elif R == "dsyr2k":
        xk.dsyr2k("L", "N", N, N, 1.5, A, N, B, N, -0.75, C, N, asynchronous=True)
    else:
        xk.dsymm("L", "L", N, N, 1.5, A, N, B, N, -0.75, C, N, asynchronous=True)
    xk.sync()


if DOD and os.environ.get("SYNC_WARMUP") == "1":  # the ablation's sequence: a sync call first
    call()
    torch.cuda.synchronize()
if DOD:
    for X in (A, B, C, L):
        xk.memory_prefetch_async(N, N, X, N)
    xk.sync()
    call = call_async
call()
torch.cuda.synchronize()
xk.reset_stats()
path = os.path.join(out_dir, "trace_%s_n%d_g%d%s.json" % (R, N, G, "_dod" if DOD else ""))
xk.trace(path)
torch.cuda.synchronize()
t0 = time.perf_counter()
call()
torch.cuda.synchronize()
wall = (time.perf_counter() - t0) * 1e3
xk.trace(None)
st = xk.get_stats()
xk.finalize()

ev = json.load(open(path))["traceEvents"]


def union(iv):
    iv = sorted(iv)
    out = []
    for a, b in iv:
        if out and a <= out[-1][1]:
            out[-1][1] = max(out[-1][1], b)
        else:
            out.append([a, b])
    return out


kern = union([(e["ts"], e["ts"] + e["dur"]) for e in ev if e["tid"] == "kernels"])
busy = sum(b - a for a, b in kern)
t_end = max(e["ts"] + e["dur"] for e in ev)
gaps = [(kern[0][0], 0.0, kern[0][0])] if kern else []
gaps += [(b - a, a, b) for (_, a), (b, _) in zip(kern, kern[1:])]
if kern:
    gaps.append((t_end - kern[-1][1], kern[-1][1], t_end))
gaps.sort(reverse=True)


def inside(tid, a, b):
    return sum(max(0.0, min(b, e["ts"] + e["dur"]) - max(a, e["ts"])) for e in ev if e["tid"] == tid)


top = [{"gap_ms": round(g / 1e3, 3), "at_ms": round(a / 1e3, 3),
        "h2d_busy_ms": round(inside("H2D", a, b) / 1e3, 3), "d2h_busy_ms": round(inside("D2H", a, b) / 1e3, 3),
        "p2p_busy_ms": round(inside("P2P-in", a, b) / 1e3, 3)} for g, a, b in gaps[:12]]
span = {}
for tid in ("H2D", "D2H", "P2P-in", "kernels"):
    xs = [e for e in ev if e["tid"] == tid]
    if xs:
        span[tid] = {"first_ms": round(min(e["ts"] for e in xs) / 1e3, 3),
                     "last_end_ms": round(max(e["ts"] + e["dur"] for e in xs) / 1e3, 3),
                     "busy_ms": round(sum(b - a for a, b in union([(e["ts"], e["ts"] + e["dur"]) for e in xs])) / 1e3, 3),
                     "ops": len(xs)}
byname = {}
for e in ev:
    if e["tid"] != "kernels":
        continue
    nm = re.sub(r" x\d+$", "", e["name"])
    nb = int(e["name"].rsplit("x", 1)[1]) if re.search(r" x\d+$", e["name"]) else 1
    d = byname.setdefault(nm, {"launches": 0, "tasks": 0, "ms": 0.0, "gflop": 0.0})
    d["launches"] += 1
    d["tasks"] += nb
    d["ms"] += e["dur"] / 1e3
    d["gflop"] += e["args"].get("flops", 0) / 1e9
for d in byname.values():
    d["tflops_per_launch_time"] = round(d["gflop"] / max(1e-9, d["ms"]), 2)
    d["ms"] = round(d["ms"], 3)
# delivered FP64 rate over time: each kernel op's flops spread uniformly over its duration,
# summed per 50 ms window (where a host-resident call loses against data-on-device)
WIN = 50e3
nwin = int(t_end // WIN) + 1
win = [0.0] * nwin
for e in ev:
    if e["tid"] != "kernels" or e["dur"] <= 0:
        continue
    f = e["args"].get("flops", 0)
    a, b = e["ts"], e["ts"] + e["dur"]
    for w in range(int(a // WIN), min(nwin, int(b // WIN) + 1)):
        ov = max(0.0, min(b, (w + 1) * WIN) - max(a, w * WIN))
        win[w] += f * ov / e["dur"]
summary = {"tflops_by_50ms_window": [round(x / (WIN * 1e-6) / 1e12, 2) for x in win],
           "routine": R, "mode": "data-on-device" if DOD else "host-resident", "kernel_ops": byname, "N": N, "tile": T, "gpus": G, "wall_ms": round(wall, 3),
           "tflops": round(flops / wall / 1e9, 2), "trace_span_ms": round(t_end / 1e3, 3),
           "kernel_busy_union_ms": round(busy / 1e3, 3), "streams": span, "largest_kernel_idle_gaps": top,
           "h2d_gb": sum(st["h2d_bytes"]) / 1e9, "d2h_gb": sum(st["d2h_bytes"]) / 1e9}
print(json.dumps(summary))
json.dump(summary, open(os.path.join(out_dir, "trace_%s_n%d_g%d%s_summary.json" % (R, N, G, "_dod" if DOD else "")), "w"), indent=1)
