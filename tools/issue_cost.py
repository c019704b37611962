"""Host cost of planning + issuing plan records ("overhead of
creation and scheduling of dynamic tasks"): for each (G logical GPUs, N, T) one warm-up and
one timed synchronous xk_dgemm from pinned host memory; prints JSON with the records planned
(all GPUs), records issued here, host plan+issue time, us per record, and the call's wall time.
G > 1 runs in logical-device mode on one B200 (every GPU's records issued by this thread)."""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import inputs  # noqa: E402
import paper_conf_sc_gautierl21_b200 as xk  # noqa: E402
from tests.gpu_util import device_map  # noqa: E402


def one(G, N, T):
    A, B, C = (inputs.uniform(s, N, N) for s in (1, 2, 3))
    xk.init(ngpus=G, phys=device_map(G), tile=T, probe=True)
    try:
        for X in (A, B, C):
            xk.register(X)
        xk.dgemm("N", "N", N, N, N, 1.5, A, N, B, N, -0.75, C, N)
        xk.reset_stats()
        t0 = time.perf_counter()
        xk.dgemm("N", "N", N, N, N, 1.5, A, N, B, N, -0.75, C, N)
        wall = time.perf_counter() - t0
        st = xk.get_stats()
    finally:
        xk.finalize()
    return {"G": G, "N": N, "T": T, "records": st["plan_records"], "records_local": st["plan_records_local"],
            "host_issue_ms": st["host_issue_ms"], "us_per_record": 1e3 * st["host_issue_ms"] / max(1, st["plan_records"]),
            "call_ms": 1e3 * wall, "tflops": 2.0 * N ** 3 / wall / 1e12, "launches": st["kernel_launches"]}


if __name__ == "__main__":
    cfgs = [(int(g), int(n), int(t)) for g, n, t in (c.split(",") for c in sys.argv[1:])] or \
        [(8, 16384, 1024), (8, 32768, 1024), (1, 32768, 1024), (8, 32768, 2048), (1, 65536, 1024)]
    for G, N, T in cfgs:
        print(json.dumps(one(G, N, T)), flush=True)
