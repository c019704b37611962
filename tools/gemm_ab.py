"""A/B driver for the DGEMM tile kernel: data-on-device DGEMM (A, B, C prefetched) at each
tile size, 1 warm-up + REPS timed xk_dgemm_async + xk_sync calls (CUDA events, device
synchronized), then one pass with every grouped launch timed (average launch TF/s).  Knobs
come from the environment (XK_PERSIST, XK_GROUP_M, ...).  Prints one JSON line."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import inputs  # noqa: E402
import paper_conf_sc_gautierl21_b200 as xk  # noqa: E402

N = int(os.environ.get("N", 32768))
REPS = int(os.environ.get("REPS", 3))
tiles = [int(t) for t in os.environ.get("TILES", "1024,2048,4096").split(",")]
TA, TB = os.environ.get("TRANS", "NN")
A, B, C = inputs.uniform(1, N, N), inputs.uniform(2, N, N), inputs.uniform(3, N, N)
out = {"N": N, "trans": TA + TB, "env": {k: v for k, v in os.environ.items() if k.startswith("XK_")}}
for T in tiles:
    xk.init(ngpus=1, tile=T, probe=False)
    for X in (A, B, C):
        xk.register(X)
        xk.memory_prefetch_async(N, N, X, N)
    xk.sync()
    xk.dgemm_async(TA, TB, N, N, N, 1.5, A, N, B, N, -0.75, C, N)
    xk.sync()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    e0.record()
    for _ in range(REPS):
        xk.dgemm_async(TA, TB, N, N, N, 1.5, A, N, B, N, -0.75, C, N)
        xk.sync()
    torch.cuda.synchronize()
    e1.record()
    e1.synchronize()
    ms = e0.elapsed_time(e1) / REPS
    xk.reset_stats()
    xk.set_kernel_timing(True)
    xk.dgemm_async(TA, TB, N, N, N, 1.5, A, N, B, N, -0.75, C, N)
    xk.sync()
    st = xk.get_stats()
    xk.set_kernel_timing(False)
    kt = st["kernel_timed_flops"] / (st["kernel_ms_total"] * 1e-3) / 1e12 if st["kernel_ms_total"] else None
    out["T%d" % T] = {"dod_tflops": round(2.0 * N ** 3 / (ms * 1e-3) / 1e12, 3),
                      "kernel_tflops": round(kt, 3) if kt else None, "launches": st["kernel_timed_launches"]}
    xk.finalize()
print(json.dumps(out), flush=True)
