"""Paper Fig. 6 style breakdown: time in HtoD / PtoP / kernels / DtoH
for one host-resident DGEMM, from the library's own timeline (xk_trace).  Writes the Chrome
trace next to the JSON summary."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import inputs
import paper_conf_sc_gautierl21_b200 as xk

N = int(os.environ.get("N", 32768))
T = int(os.environ.get("T", 2048))
G = int(os.environ.get("G", 1))
out_dir = os.environ.get("OUT", "gpurun_out")
A, B, C = inputs.uniform(1, N, N), inputs.uniform(2, N, N), inputs.uniform(3, N, N)
xk.init(ngpus=G, phys=[0] * G, tile=T, probe=True)
for X in (A, B, C):
    xk.register(X)
xk.dgemm("N", "N", N, N, N, 1.5, A, N, B, N, -0.75, C, N)
xk.reset_stats()
path = os.path.join(out_dir, "trace_n%d_g%d.json" % (N, G))
xk.trace(path)
torch.cuda.synchronize()
t0 = time.perf_counter()
xk.dgemm("N", "N", N, N, N, 1.5, A, N, B, N, -0.75, C, N)
torch.cuda.synchronize()
wall = (time.perf_counter() - t0) * 1e3
xk.trace(None)
st = xk.get_stats()
xk.finalize()
tm = st["trace_ms"]
xfer = tm["h2d"] + tm["p2p"] + tm["d2h"]
summary = {"N": N, "tile": T, "gpus": G, "wall_ms": wall, "busy_ms_by_kind": tm,
           "transfer_share_of_busy": xfer / max(1e-9, xfer + tm["kernel"]),
           "note": "sums of per-op durations over all streams (they overlap); the paper's Fig. 6 reports "
                   "cumulative time by kind the same way"}
print(json.dumps(summary))
json.dump(summary, open(os.path.join(out_dir, "trace_breakdown_n%d_g%d.json" % (N, G)), "w"), indent=1)
