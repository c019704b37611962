"""Rank mode -- one process per GPU -- through the C ABI.

`world` processes (tests/rank_worker.py) share a session file and host matrices in shared
file mappings.  Each runs the same deterministic planner and executes only its own GPU's
records: peer tiles are pulled through CUDA IPC mappings of the other processes' arenas,
cross-process dependencies are per-record completion flags (stream memory operations).
On a one-GPU box every rank maps to the same device (the IPC pulls are then device-local
copies); on a multi-GPU box rank r runs on GPU r.

Checks: exact-integer results bitwise equal to the CPU oracle (TRSM: Q13 residual bound +
relative Frobenius); every rank's measured H2D / P2P-in / D2H bytes equal the bytes the
plan assigns to its GPU (the planner replayed on the CPU with the same topology); closed
forms for the composed call (D never crosses PCIe).
"""
import json
import os
import subprocess
import sys
import tempfile

import pytest

import paper_conf_sc_gautierl21_b200 as xk

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def run_ranks(world, case, n=1000, tile=256, probe=0, timeout=600, topo="ranked", optimistic=1, arena=1 << 30):
    with tempfile.TemporaryDirectory(dir="/dev/shm" if os.path.isdir("/dev/shm") else None) as d:
        session = os.path.join(d, "session")
        procs = [subprocess.Popen([sys.executable, os.path.join(ROOT, "tests", "rank_worker.py"),
                                   "--rank", str(r), "--world", str(world), "--session", session,
                                   "--dir", d, "--case", case, "--n", str(n), "--tile", str(tile),
                                   "--probe", str(probe), "--arena", str(arena), "--topo", topo,
                                   "--optimistic", str(optimistic)],
                                  stdout=subprocess.PIPE, stderr=subprocess.PIPE, text=True, cwd=ROOT)
                 for r in range(world)]
        outs = []
        try:
            for p in procs:
                o, e = p.communicate(timeout=timeout)
                assert p.returncode == 0, e[-3000:]
                outs.append(json.loads(o.strip().splitlines()[-1]))
        finally:
            for p in procs:
                if p.poll() is None:
                    p.kill()
        assert not os.path.exists(session), "rank 0 removes the session file at finalize"
    outs.sort(key=lambda o: o["rank"])
    assert outs[0]["ok"], outs[0].get("failed")
    return outs


def plan_bytes(links, calls, tile, world, **flags):
    """Per-GPU H2D / P2P-in / D2H bytes of the plan, replayed on the CPU planner."""
    s = xk.PlanSession(links["bw_MBps"], links["task_rate_mflops"], tile=tile, **flags)
    h2d, p2p, d2h = [0] * world, [0] * world, [0] * world
    try:
        for c in calls:
            for rec in s.call(c, cap=1 << 18):
                r = dict(zip(xk.REC_FIELDS, rec))
                if r["kind"] == xk.REC_H2D:
                    h2d[r["dst"]] += r["work"]
                elif r["kind"] == xk.REC_P2P:
                    p2p[r["dst"]] += r["work"]
                elif r["kind"] == xk.REC_D2H:
                    d2h[r["src"]] += r["work"]
    finally:
        s.close()
    return h2d, p2p, d2h


def assert_bytes_follow_plan(outs, calls, tile, **flags):
    world = len(outs)
    links = outs[0]["topology"]
    for o in outs[1:]:
        assert o["topology"] == links, "every rank must build the identical link matrix"
    h2d, p2p, d2h = plan_bytes(links, calls, tile, world, **flags)
    for o in outs:
        r, st = o["rank"], o["stats"]
        assert (st["h2d_bytes"], st["p2p_in_bytes"], st["d2h_bytes"]) == (h2d[r], p2p[r], d2h[r]), (r, st)
    assert sum(o["stats"]["p2p_in_bytes"] for o in outs) == sum(o["stats"]["p2p_out_bytes"] for o in outs)


BASE = 1 << 40  # fake, non-overlapping host addresses for the CPU replay of the calls


def addr(i, n):
    return BASE + i * (8 * n * n + (1 << 20))


@pytest.mark.parametrize("world,topo,opt", [(2, "ranked", 1), (4, "ranked", 1), (8, "ranked", 1),
                                             (8, "ranked", 0), (8, "unranked", 0), (8, "home", 1)])
def test_rank_mode_gemm_bitwise_and_bytes(world, topo, opt):
    """Every heuristic mode (paper Table II ablations) at 2/4/8 processes: same bits, bytes
    per GPU as planned."""
    N, T = 1000, 256
    outs = run_ranks(world, "gemm", N, T, topo=topo, optimistic=opt)
    A, B, C, E = (addr(i, N) for i in range(4))
    calls = [xk.make_call(m=N, n=N, k=N, alpha=-2.0, beta=0.5, A=A, lda=N, B=B, ldb=N, C=C, ldc=N, sync=True),
             xk.make_call(transA="T", m=N, n=N, k=N, alpha=1.0, beta=0.0, A=A, lda=N, B=C, ldb=N, C=E, ldc=N,
                          sync=True)]
    assert_bytes_follow_plan(outs, calls, T, topo=topo, optimistic=bool(opt))
    p2p = sum(o["stats"]["p2p_in_bytes"] for o in outs)
    assert (p2p == 0) if topo == "home" else (p2p > 0), "tiles are forwarded between processes unless host-first"


def test_rank_mode_composition_no_h2d_of_intermediate():
    world, N, T = 4, 1000, 256
    outs = run_ranks(world, "compose", N, T)
    A, B, C, E, D = (addr(i, N) for i in range(5))
    calls = [xk.make_call(m=N, n=N, k=N, alpha=1.0, beta=0.0, A=A, lda=N, B=B, ldb=N, C=D, ldc=N),
             xk.make_call(m=N, n=N, k=N, alpha=1.0, beta=0.0, A=D, lda=N, B=C, ldb=N, C=E, ldc=N),
             xk.make_call(routine=xk.ROUTINE_COHERENT, m=N, n=N, C=E, ldc=N),
             xk.make_call(routine=xk.ROUTINE_COHERENT, m=N, n=N, C=D, ldc=N)]
    assert_bytes_follow_plan(outs, calls, T)
    h2d = sum(o["stats"]["h2d_bytes"] for o in outs)
    d2h = sum(o["stats"]["d2h_bytes"] for o in outs)
    assert h2d == 3 * 8 * N * N, "A, B, C each cross PCIe once; D never does"
    assert d2h == 2 * 8 * N * N


def test_rank_mode_data_on_device_and_probe():
    """Prefetched operands (data-on-device): the GEMM moves no host bytes; the link matrix
    is probed collectively (every rank must end with the same matrix)."""
    outs = run_ranks(2, "dod", 768, 256, probe=1)
    for o in outs:
        assert o["stats"]["h2d_bytes"] == 0
        bw = o["topology"]["bw_MBps"]
        assert all(bw[s][d] > 0 for s in range(3) for d in range(3))


def test_rank_mode_distribute_2dbc():
    """xk_distribute_2dbc_async in rank mode: each process loads the tiles of its grid column
    (block-cyclic on a 1 x world grid, (1,1) blocks); the DGEMM then moves no host byte, its
    operands pulled from the peers' arenas; bitwise vs the oracle."""
    world, N, T = 4, 1024, 256
    outs = run_ranks(world, "distribute", N, T)
    t = N // T
    for o in outs:
        cols = sum(1 for bj in range(t) if bj % world == o["rank"])
        assert o["dist_h2d"] == 3 * t * cols * 8 * T * T
        assert o["stats"]["h2d_bytes"] == 0
    assert sum(o["stats"]["p2p_in_bytes"] for o in outs) > 0


def test_rank_mode_blas3():
    run_ranks(4, "blas3", 700, 128)


def test_rank_mode_bench_configuration_freivalds():
    """bench.py's multi-GPU launch configuration at full size: rank mode, N=32768, T=4096,
    alpha=1.5, beta=-0.75, 2 processes -- exact-integer inputs, Freivalds check exact in FP64;
    bytes per rank as planned."""
    N, T = 32768, 4096
    outs = run_ranks(2, "big", N, T, timeout=1200, arena=24 << 30)
    A, B, C = (addr(i, N) for i in range(3))
    calls = [xk.make_call(m=N, n=N, k=N, alpha=1.5, beta=-0.75, A=A, lda=N, B=B, ldb=N, C=C, ldc=N, sync=True)]
    assert_bytes_follow_plan(outs, calls, T)
    assert "freivalds" in outs[0]["checks"]


def test_rank_mode_refuses_diverging_configuration():
    """Ranks whose plan-shaping configuration differs (here the tile size) would execute
    different plans: xk_init fails with XK_ERR_CONFIG on every rank, nobody hangs."""
    outs = run_ranks(2, "mismatch", 512, 128, timeout=300)
    assert [o["init_error"] for o in outs] == [4, 4]


def test_bench_under_torchrun_emits_round2_keys():
    """bench.py under torchrun (2 ranks on the box's GPU(s), rank mode): one JSON line with the
    host-resident value, e2e (with the concurrent-probe roofline), data_on_device, the
    heuristic ablation (every mode, per-GPU H2D bytes) and the north-star block (forced at
    G = 2, small N to stay quick)."""
    env = dict(os.environ, XK_DIST_BACKEND="gloo")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", "29631", os.path.join(ROOT, "bench.py"),
           "--gpus", "2", "--size", "16384", "--tile", "2048", "--steps", "1", "--warmup", "1",
           "--no-cpu-baseline", "--north-star", "--ns-n", "8192", "--host-probe-mib", "256"]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=900, cwd=ROOT, env=env)
    assert r.returncode == 0, r.stderr[-3000:]
    line = json.loads([ln for ln in r.stdout.splitlines() if ln.startswith("{")][-1])
    assert line["n_gpus"] == 2 and line["value"] > 0 and line["gpu_launches"] > 0
    assert line["e2e"]["h2d_bytes_per_step"] == 3 * 8 * 16384 ** 2
    assert line["host_links_all_MBps"]["h2d"] > 0 and line["host_links_all_MBps"]["duplex"] > 0
    assert line["data_on_device"]["value"] > 0
    abl = line["ablation"]
    for mode in ("full", "no_optimistic", "no_optimistic_no_topo", "home"):
        assert abl[mode]["tflops"] > 0 and len(abl[mode]["h2d_bytes_per_gpu"]) == 2
    # closed forms at N=16384, T=2048 on the 2x1 grid: FULL reads A, B, C once
    # (6.44 GB), HOME reads every A row tile once per requesting GPU (r_A = min(Q, t) = 1) and
    # every B column tile once per grid row (r_B = min(P, t) = 2)
    tile = 8 * 2048 * 2048
    assert abl["full"]["h2d_bytes"] == 3 * 64 * tile
    assert abl["home"]["h2d_bytes"] == (8 * 8 * 1 + 8 * 8 * 2 + 64) * tile
    assert line["north_star"]["tflops"] > 0


def test_probe_host_links_single_process():
    """xk_probe_host_links: all GPUs copying at once; one GPU and 2 logical GPUs (which share
    one physical link, so the aggregate stays near one link's bandwidth)."""
    from tests.gpu_util import device_map
    for G in (1, 2):
        xk.init(ngpus=G, phys=device_map(G), probe=True, tile=512)
        try:
            assert xk.probe_host_links(256 << 20) == 0
            t = xk.get_topology()
        finally:
            xk.finalize()
        ha = t["host_all_MBps"]
        single = t["bw_MBps"][G][0]
        assert t["host_probe_bytes"] == 256 << 20
        assert ha["h2d"] > 0.5 * single and ha["d2h"] > 0 and ha["duplex"] > 0
        assert ha["h2d"] < 1.5 * G * single
