"""Plan-predicted heuristic ablation on 8 GPUs (virtual-time model of the planner; no GPU):
makespan = max t_end of the plan, for the paper's DGX-1 (Fig. 2 matrix, PCIe Gen3 host links,
V100 FP64 rate) and an 8x B200 NVSwitch box (measured single-GPU PCIe/NVLink/FP64 rates).
Informative only: the model's timing fidelity is not pinned."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_gautierl21_b200 as xk
from tests.test_planner import fig2, with_host, uniform

MODES = [("full", "ranked", True), ("no_opt", "ranked", False), ("no_opt_topo", "unranked", False), ("home", "home", True)]
boxes = {
    # DGX-1: Fig. 2 GPU matrix; host links PCIe Gen3 x16 shared by 2 GPUs -> ~6 GB/s each
    "dgx1_v100": (with_host(fig2(), host=6000), 7000000),
    # 8x B200: 55 GB/s PCIe Gen5 per GPU (measured), ~700 GB/s CE peer copies, 35.8 TF tile rate
    # (round-2 grouped launch, measured)
    "hgx_b200": (uniform(8, peer=700000, host=55000), 35800000),
}
out = {"params": {"window": 4, "note": "planner defaults (window W = 4, DESIGN.md Q17); the model's makespan is pinned to one-GPU measurements within 4% (profiles/r02_model_fidelity.jsonl), multi-GPU timing unpinned"}}
for box, (bw, rate) in boxes.items():
    for N in (16384, 32768):
        T = 2048
        call = xk.make_call(m=N, n=N, k=N, alpha=1.0, beta=1.0, A=1 << 40, lda=N, B=2 << 40, ldb=N, C=3 << 40, ldc=N, sync=True)
        row = {}
        for name, topo, opt in MODES:
            recs = xk.plan_dump(call, bw, rate_mflops=rate, topo=topo, optimistic=opt, tile=T, cap=1 << 18)
            t = max(r[12] for r in recs) * 1e-9
            h2d = sum(r[13] for r in recs if r[1] == 0) / 1e9
            per = [0] * 8
            for r in recs:
                if r[1] == 0:
                    per[r[7]] += r[13]
            row[name] = {"pred_tflops": round(2.0 * N ** 3 / t / 1e12, 2), "h2d_GB": round(h2d, 2),
                         "h2d_max_over_mean": round(max(per) / (sum(per) / 8), 3)}
        out["%s_N%d" % (box, N)] = row
        print(box, N, json.dumps(row))
# the north-star configuration (BASELINE configs[4]): N=65536 on 8x B200, tile sweep, full
# heuristics vs host-first; fraction of 8 x 37.2 TFLOP/s
bw, rate = boxes["hgx_b200"]
N = 65536
for T in (1024, 2048, 4096):
    call = xk.make_call(m=N, n=N, k=N, alpha=1.5, beta=-0.75, A=1 << 40, lda=N, B=2 << 40, ldb=N, C=3 << 40, ldc=N, sync=True)
    row = {}
    for name, topo, opt in (MODES[0], MODES[3]):
        recs = xk.plan_dump(call, bw, rate_mflops=rate, topo=topo, optimistic=opt, tile=T, cap=1 << 20)
        t = max(r[12] for r in recs) * 1e-9
        h2d = sum(r[13] for r in recs if r[1] == 0) / 1e9
        tf = 2.0 * N ** 3 / t / 1e12
        row[name] = {"pred_tflops": round(tf, 1), "frac_of_8x_fp64_peak": round(tf / (8 * 37.22), 3),
                     "h2d_GB": round(h2d, 1)}
    out["hgx_b200_N65536_T%d" % T] = row
    print("hgx_b200 N=65536 T=%d" % T, json.dumps(row))
# BASELINE configs[2]/[3] on 8x B200 (N=32768, T=2048): DSYRK / DSYR2K (lower, N) and
# DTRSM / DTRMM (left, lower, N, non-unit), host-resident, full heuristics vs host-first;
# per-GPU task-time balance of the owner map (max / mean busy time)
N, T = 32768, 2048
fl = {"dsyrk": N * N * (N + 1), "dsyr2k": 2 * N * N * N + N, "dtrsm": N * N * N, "dtrmm": N * N * N}
rt = {"dsyrk": xk._abi.ROUTINE_DSYRK, "dsyr2k": xk._abi.ROUTINE_DSYR2K, "dtrsm": xk._abi.ROUTINE_DTRSM, "dtrmm": xk._abi.ROUTINE_DTRMM}
for name in ("dsyrk", "dsyr2k", "dtrsm", "dtrmm"):
    row = {}
    for mode, topo, opt in (MODES[0], MODES[3]):
        call = xk.make_call(routine=rt[name], uplo="L", transA="N", side="L", diag="N", m=N, n=N, k=N,
                            alpha=1.5, beta=-0.75, A=1 << 40, lda=N, B=2 << 40, ldb=N, C=3 << 40, ldc=N, sync=True)
        recs = xk.plan_dump(call, bw, rate_mflops=rate, topo=topo, optimistic=opt, tile=T, cap=1 << 20)
        t = max(r[12] for r in recs) * 1e-9
        busy = [0] * 8
        for r in recs:
            if r[1] == 2:
                busy[r[7]] += r[12] - r[11]
        tf = fl[name] / t / 1e12
        row[mode] = {"pred_tflops": round(tf, 1), "frac_of_8x_fp64_peak": round(tf / (8 * 37.22), 3),
                     "busy_max_over_mean": round(max(busy) / (sum(busy) / 8), 3),
                     "h2d_GB": round(sum(r[13] for r in recs if r[1] == 0) / 1e9, 1)}
    out["hgx_b200_%s_N32768_T2048" % name] = row
    print("hgx_b200", name, json.dumps(row))
print(json.dumps(out))
