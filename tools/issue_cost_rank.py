"""Host plan + issue cost in rank mode (one process per GPU): run under
torchrun; every rank plans the whole call and issues its own GPU's records.  Prints, from
rank 0, each rank's records planned / executed locally and host plan+issue time.  On a box
with fewer GPUs than ranks the ranks share a device (the GPU time then stretches, the host
issue time is what this measures)."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402

N = int(os.environ.get("N", 32768))
T = int(os.environ.get("T", 1024))
rank, ws = bench.dist_setup(os.environ.get("XK_DIST_BACKEND", "gloo"))
import paper_conf_sc_gautierl21_b200 as xk  # noqa: E402

A, B, C, paths, base = bench.share_inputs(N, rank, ws)
xk.init(rank=rank, world=ws, session=base + ".session1", tile=T, probe=False, arena_bytes=int(os.environ.get("ARENA", 12 << 30)))
for X in (A, B, C):
    xk.register(X)
xk.dgemm_async("N", "N", N, N, N, 1.5, A, N, B, N, -0.75, C, N)
xk.sync()
xk.reset_stats()
xk.dgemm_async("N", "N", N, N, N, 1.5, A, N, B, N, -0.75, C, N)
st = xk.get_stats()
xk.sync()
mine = [st["plan_records"], st["plan_records_local"], st["host_issue_ms"]]
allr = bench.sum_over_ranks([v if r == rank else 0.0 for r in range(ws) for v in mine], ws)
xk.finalize()
bench.barrier(ws)
if rank == 0:
    for p in paths:
        if os.path.exists(p):
            os.unlink(p)
    rows = [allr[3 * r:3 * r + 3] for r in range(ws)]
    print(json.dumps({"N": N, "T": T, "ranks": ws, "per_rank": [{"records": int(a), "local": int(b), "host_issue_ms": round(c, 2),
                                                                 "us_per_record": round(1e3 * c / max(1, a), 3)} for a, b, c in rows]}))
