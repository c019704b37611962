"""Per-call times of repeated data-on-device DTRSM calls on G logical GPUs (the ablation's
sequence: sync warm-up, prefetch, then async call + xk_sync per repetition)."""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import inputs
import paper_conf_sc_gautierl21_b200 as xk

N = int(os.environ.get("N", 16384)); G = int(os.environ.get("G", 8)); T = int(os.environ.get("T", 2048))
REPS = int(os.environ.get("REPS", 10))
B = inputs.uniform(2, N, N)
L = inputs.tri_dd(4, N, lower=True, fill=0.0)
xk.init(ngpus=G, phys=[0] * G, tile=T, probe=True)
for X in (B, L):
    xk.register(X)
xk.dtrsm("L", "L", "N", "N", N, N, 1.0, L, N, B, N)
for X in (B, L):
    xk.memory_prefetch_async(N, N, X, N)
xk.sync()
torch.cuda.synchronize()
ts = []
for r in range(REPS):
    xk.reset_stats()
    t0 = time.perf_counter()
    xk.dtrsm("L", "L", "N", "N", N, N, 1.0, L, N, B, N, asynchronous=True)
    t1 = time.perf_counter()
    xk.sync()
    torch.cuda.synchronize()
    t2 = time.perf_counter()
    ts.append((round((t1 - t0) * 1e3, 1), round((t2 - t0) * 1e3, 1), round(N ** 3 / (t2 - t0) / 1e12, 2)))
    st = xk.get_stats()
    print(json.dumps({"rep": r, "issue_ms": ts[-1][0], "call_ms": ts[-1][1], "tflops": ts[-1][2],
                      "plan_issue_ms": round(st["host_issue_ms"], 1), "records": st["plan_records"],
                      "allocs": st["device_allocs"], "alloc_ms": round(st["device_alloc_ms"], 1)}), flush=True)
xk.finalize()
