#!/usr/bin/env python
"""bench.py -- end-to-end DGEMM TFLOP/s of the B200-native XKBlas-style library.

Metric (BASELINE.json): "end-to-end DGEMM TFlop/s at N=32768/65536 on 1/2/4/8 B200,
% FP64 roofline".  Workload at N GPUs: DGEMM N=32768 (m=n=k), tile T=4096 (the best of the
paper's tile sweep {1024, 2048, 4096}, measured in profiles/), NN,
alpha=1.5, beta=-0.75 (reading Q10), column-major host matrices from the seeded
splitmix64 generator (uniform [-1,1)), owner grid near-square P x Q.

A step is one whole DGEMM (every §8(a) row: tiling, owner map, directory, source
selection, transfers, tile kernels, coherence):
  value : data-on-device -- A, B, C already resident in HBM (prefetched into the tile
          cache, untimed); one xk_dgemm_async + xk_sync per step, C updated on the GPUs.
  e2e   : the paper's host-resident measurement -- xk_dgemm (synchronous) from pinned
          host buffers; every step copies A, B, C tiles H2D and C D2H inside the timed
          region and ends with C coherent on the host.
Timing: CUDA events on a side stream with a full device synchronize on both sides of the
K timed steps (the library's work spans its own H2D/D2H/P2P/kernel streams), barrier and
max over ranks under torchrun.  Inputs (8.6 GB per matrix) are far larger than L2 (126 MB).

Multi-GPU: under torchrun the library runs in rank mode -- one process per GPU.  The host
matrices live in /dev/shm file mappings shared by the processes; every xk call is
collective; each process executes its own GPU's records of the identical plan (peer tiles
pulled through CUDA IPC, cross-process order by per-record completion flags).  Each rank
times its own GPU with CUDA events; the max over ranks is reported.  Total work is fixed
as the GPU count grows: "scaling": "strong".  (--gpus G without torchrun: one process
drives G GPUs, the paper's single-process library.)

--impl reference: the CPU oracle (oracle/oracle.c, plain triple loop) timed on the host
cores on bounded row slabs of the same workload (the reference arm of this tier).
"""
import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

N_DEFAULT, T_DEFAULT = 32768, 4096  # tile: best of the paper's sweep {1024, 2048, 4096}
ALPHA, BETA = 1.5, -0.75
FP64_PEAK_TFLOPS = 148 * 64 * 2 * 1.965e9 / 1e12  # 37.2: SMs x FP64 FMA/clk x 2 x max clock
METRIC = "end-to-end DGEMM TFlop/s at N=32768/65536 on 1/2/4/8 B200, % FP64 roofline"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="xk", choices=["xk", "reference"])
    ap.add_argument("--n", "--size", dest="n", type=int, default=N_DEFAULT)
    ap.add_argument("--tile", type=int, default=T_DEFAULT)
    ap.add_argument("--topo", default="ranked")
    ap.add_argument("--optimistic", type=int, default=1)
    ap.add_argument("--kstreams", type=int, default=2)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    return ap.parse_args()


# --------------------------------------------------------------------------- distributed
_HOST_GROUP = None  # gloo group for barriers / timing reductions: host-side waits only


def dist_setup(backend=None):
    """One process per GPU under torchrun (RANK/LOCAL_RANK/WORLD_SIZE/MASTER_* from the env).
    backend: "nccl" on GPU boxes (default), "gloo" for the CPU tests of this path.
    The barriers and the max-over-ranks reduction go through a gloo group: a rank waiting in
    a barrier must not park an NCCL kernel on its GPU while rank 0's library computes on it."""
    global _HOST_GROUP
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    if ws > 1:
        import torch
        import torch.distributed as dist
        backend = backend or os.environ.get("XK_DIST_BACKEND", "nccl")
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        lr = int(os.environ.get("LOCAL_RANK", rank))
        if torch.cuda.is_available():  # this process's GPU (ranks share it on a one-GPU box)
            lr = lr % torch.cuda.device_count()
            torch.cuda.set_device(lr)
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", lr))
            _HOST_GROUP = dist.new_group(backend="gloo")
        else:
            dist.init_process_group(backend)
            _HOST_GROUP = dist.group.WORLD
    return rank, ws


def barrier(ws):
    if ws > 1:
        import torch.distributed as dist
        dist.barrier(group=_HOST_GROUP)


def max_over_ranks(x, ws):
    """Timing is taken as the max over ranks (every rank measured the same barrier-bracketed
    interval; rank 0 drove all GPUs)."""
    if ws == 1:
        return x
    import torch
    import torch.distributed as dist
    t = torch.tensor([x], dtype=torch.float64)
    dist.all_reduce(t, op=dist.ReduceOp.MAX, group=_HOST_GROUP)
    return float(t.item())


# --------------------------------------------------------------------------- clocks
class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region (B200_PROFILING.md)."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self):
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "--query-gpu=" + self.Q, "--format=csv,noheader",
                                          "-lms", "200"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL,
                                         text=True)
            self.th = threading.Thread(target=self._read, daemon=True)
            self.th.start()
        except OSError:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self, gpus):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except subprocess.TimeoutExpired:
            self.proc.kill()
        self.th.join(timeout=2)
        sm, smax, reasons, power = [], [], set(), []
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 9 or not f[0].isdigit() or int(f[0]) >= gpus:
                continue
            try:
                sm.append(float(f[1].split()[0]))
                smax.append(float(f[2].split()[0]))
                power.append(float(f[3].split()[0]))
            except ValueError:
                continue
            for nm, v in zip(names, f[5:9]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        loaded = [s for s, p in zip(sm, power) if p > 300] or sm
        return {"sm_mhz": statistics.median(loaded) if loaded else None,
                "sm_max_mhz": max(smax) if smax else None, "reasons": sorted(reasons),
                "samples": len(sm), "power_w_max": max(power) if power else None}


# --------------------------------------------------------------------------- device timing
class DevTimer:
    """CUDA events on a side stream, full device synchronize on both sides."""

    def __init__(self):
        import torch
        self.torch = torch
        self.s = torch.cuda.Stream()
        self.e0 = torch.cuda.Event(enable_timing=True)
        self.e1 = torch.cuda.Event(enable_timing=True)

    def start(self):
        self.torch.cuda.synchronize()
        self.e0.record(self.s)

    def stop_ms(self):
        self.torch.cuda.synchronize()
        self.e1.record(self.s)
        self.e1.synchronize()
        return self.e0.elapsed_time(self.e1)


# --------------------------------------------------------------------------- CPU baseline
def oracle_block(N, rows, cols, A, B, C):
    """The oracle on the rows x cols top-left block of C (full k = N): 2*rows*cols*N flops."""
    import oracle
    t0 = time.perf_counter()
    oracle.dgemm("N", "N", rows, cols, N, ALPHA, A, B, BETA, C, lda=N, ldb=N, ldc=N)
    return time.perf_counter() - t0


def sized_block(N, A, B, C, budget_s):
    """Calibrate on a 16 x 256 block, then pick the column count that fills budget_s."""
    rows, cols = 16, min(N, 256)
    t = oracle_block(N, rows, cols, A, B, C)
    cols = max(16, min(N, int(cols * budget_s / max(t, 1e-4))))
    return rows, cols


def cpu_baseline(N, A, B, C, budget_s=15.0):
    """The oracle as it stands on all host cores, on a bounded block of C."""
    import oracle
    rows, cols = sized_block(N, A, B, C, budget_s)
    t = oracle_block(N, rows, cols, A, B, C)
    tf = 2.0 * rows * cols * N / t / 1e12
    return {"value": tf, "unit": "TFLOP/s", "cores": oracle.num_threads(), "kind": "oracle",
            "sample": "the %dx%d top-left block of C (full k=%d) of the N=%d DGEMM, %.1f s; rate extrapolated "
                      "to the full problem" % (rows, cols, N, N, t)}


# --------------------------------------------------------------------------- inputs
def make_inputs(N):
    import inputs
    A = inputs.uniform(inputs.SEED_A, N, N)
    B = inputs.uniform(inputs.SEED_B, N, N)
    C = inputs.uniform(inputs.SEED_C, N, N)
    return A, B, C


def traffic_from_profiles(T):
    p = os.path.join(ROOT, "profiles", "dgemm_tile_ncu.json")
    try:
        with open(p) as f:
            d = json.load(f)
        if int(d.get("tile", 0)) == T:
            return d.get("dram_bytes_per_launch")
    except (OSError, ValueError):
        pass
    return None


# --------------------------------------------------------------------------- arms
def run_reference(args, rank, ws):
    if rank != 0:
        return
    cores = len(os.sched_getaffinity(0))
    os.environ["OMP_NUM_THREADS"] = str(cores)
    N = args.n
    A, B, C = make_inputs(N)
    import oracle
    per_step_budget = max(2.0, 100.0 / max(1, args.steps + args.warmup))
    rows, cols = sized_block(N, A, B, C, per_step_budget)
    for _ in range(args.warmup):
        oracle_block(N, rows, cols, A, B, C)
    times = [oracle_block(N, rows, cols, A, B, C) for _ in range(args.steps)]
    tot = sum(times)
    tf = args.steps * 2.0 * rows * cols * N / tot / 1e12
    sample = "each step: the %dx%d top-left block of C (full k=%d) of the N=%d DGEMM; rate extrapolated" % (
        rows, cols, N, N)
    line = {"metric": METRIC, "value": tf, "unit": "TFLOP/s", "n_gpus": args.gpus, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": 1000.0 * tot / args.steps, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "impl": "reference",
            "config": {"workload": "DGEMM N=%d (m=n=k) NN alpha=1.5 beta=-0.75, column-major host, CPU oracle "
                                   "triple loop on row slabs" % N, "N": N},
            "cpu_baseline": {"value": tf, "unit": "TFLOP/s", "cores": oracle.num_threads(), "kind": "oracle",
                             "sample": sample},
            "e2e": {"value": tf, "unit": "TFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def share_inputs(N, rank, ws):
    """Host matrices for the run.  One process: plain numpy arrays.  Rank mode (one process
    per GPU): file mappings every process maps (the library's "host memory" is shared by its
    processes) -- files in /dev/shm when it has room, else anonymous memfds that the other
    ranks open through /proc/<rank 0>/fd (a small /dev/shm mount must not cap the run);
    rank 0 fills them, the others map them after a barrier.  Returns (A, B, C, paths) with
    the session-file path last; only real files in the list are unlinked at the end."""
    import inputs
    if ws == 1:
        A, B, C = make_inputs(N)
        return A, B, C, []
    import torch.distributed as dist
    import paper_conf_sc_gautierl21_b200 as xk
    obj = [None]
    if rank == 0:
        base = xk.new_session_path("xkbench")
        need = 3 * N * N * 8
        try:
            st = os.statvfs("/dev/shm")
            room = st.f_bavail * st.f_frsize > 1.1 * need
        except OSError:
            room = False
        if room and os.environ.get("XK_SHARE") != "memfd":
            paths = [base + s for s in (".A", ".B", ".C")]
            for p in paths:
                xk.shared_matrix(p, N, N, create=True)
        else:
            global _MEMFDS
            _MEMFDS = [os.memfd_create("xkbench" + s) for s in "ABC"]
            for fd in _MEMFDS:
                os.ftruncate(fd, N * N * 8)
            paths = ["/proc/%d/fd/%d" % (os.getpid(), fd) for fd in _MEMFDS]
        obj = [paths + [base + ".session"]]
    dist.broadcast_object_list(obj, src=0, group=_HOST_GROUP)
    paths = obj[0]
    mats = [xk.shared_matrix(p, N, N, create=False) for p in paths[:3]]
    if rank == 0:
        for M, seed in zip(mats, (inputs.SEED_A, inputs.SEED_B, inputs.SEED_C)):
            inputs.uniform(seed, N, N, out=M)
    barrier(ws)
    return mats[0], mats[1], mats[2], [p for p in paths if not p.startswith("/proc/")]


_MEMFDS = []


def sum_over_ranks(vals, ws):
    if ws == 1:
        return vals
    import torch
    import torch.distributed as dist
    t = torch.tensor(vals, dtype=torch.float64)
    dist.all_reduce(t, op=dist.ReduceOp.SUM, group=_HOST_GROUP)
    return t.tolist()


def run_xk(args, rank, ws):
    """ws == 1: one process drives the GPU(s) (--gpus G > 1 = the single-process multi-GPU
    runtime).  Under torchrun (ws > 1): rank mode -- one process per GPU, every xk call
    collective, each process executing its own GPU's part of the identical plan."""
    import torch
    import paper_conf_sc_gautierl21_b200 as xk
    G = ws if ws > 1 else args.gpus
    N, T = args.n, args.tile
    flops = 2.0 * N * N * N
    A, B, C, paths = share_inputs(N, rank, ws)
    kw = dict(tile=T, topo=args.topo, optimistic=bool(args.optimistic), kstreams=args.kstreams, probe=True)
    if ws > 1:
        xk.init(rank=rank, world=ws, session=paths[-1], **kw)
    else:
        xk.init(ngpus=G, **kw)
    for X in (A, B, C):
        xk.register(X)
    topo = xk.get_topology()
    timer = DevTimer()
    clocks = ClockSampler()

    # ---------------- value: data-on-device (A, B, C resident in HBM)
    for X in (A, B, C):
        xk.memory_prefetch_async(N, N, X, N)
    xk.sync()
    for _ in range(args.warmup):
        xk.dgemm_async("N", "N", N, N, N, ALPHA, A, N, B, N, BETA, C, N)
        xk.sync()
    xk.reset_stats()
    barrier(ws)
    if rank == 0:
        clocks.start()
    timer.start()
    for _ in range(args.steps):
        xk.dgemm_async("N", "N", N, N, N, ALPHA, A, N, B, N, BETA, C, N)
        xk.sync()
    ms = max_over_ranks(timer.stop_ms(), ws)
    barrier(ws)
    clk = clocks.stop(G) if rank == 0 else None
    launches = int(sum_over_ranks([xk.get_stats()["kernel_launches"]], ws)[0])
    # roofline pass: the same K steps with every grouped launch timed by CUDA events on its
    # kernel stream (timing serialises launches, so each duration is the kernel's own)
    xk.reset_stats()
    xk.set_kernel_timing(True)
    for _ in range(args.steps):
        xk.dgemm_async("N", "N", N, N, N, ALPHA, A, N, B, N, BETA, C, N)
        xk.sync()
    st = xk.get_stats()
    xk.set_kernel_timing(False)
    k_ms, k_n, k_fl = sum_over_ranks([st["kernel_ms_total"], st["kernel_timed_launches"],
                                      st["kernel_timed_flops"]], ws)
    xk.memory_coherent_sync(N, N, C, N)
    for X in (C, A, B):
        xk.memory_invalidate(N, N, X, N)
    value = args.steps * flops / (ms * 1e-3) / 1e12

    # ---------------- e2e: host-resident, H2D + D2H inside the timed region
    e2e = None
    if not args.no_e2e:
        for _ in range(max(1, args.warmup - 1)):
            xk.dgemm("N", "N", N, N, N, ALPHA, A, N, B, N, BETA, C, N)
        xk.reset_stats()
        barrier(ws)
        timer.start()
        for _ in range(args.steps):
            xk.dgemm("N", "N", N, N, N, ALPHA, A, N, B, N, BETA, C, N)
        ms_e2e = max_over_ranks(timer.stop_ms(), ws)
        se = xk.get_stats()
        mine = [sum(se["h2d_bytes"]), sum(se["d2h_bytes"]), sum(se["p2p_in_bytes"])]
        h2d, d2h, p2p = (int(v) // args.steps for v in sum_over_ranks(mine, ws))
        tf_e2e = args.steps * flops / (ms_e2e * 1e-3) / 1e12
        bw_h2d = min(topo["bw_MBps"][G][g] for g in range(G)) * 1e6 * G
        bw_d2h = min(topo["bw_MBps"][g][G] for g in range(G)) * 1e6 * G
        t_roof = max(flops / (G * FP64_PEAK_TFLOPS * 1e12), h2d / bw_h2d, d2h / bw_d2h)
        e2e = {"value": tf_e2e, "unit": "TFLOP/s", "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
               "ms_per_step": ms_e2e / args.steps, "p2p_bytes_per_step": p2p,
               "roofline_frac": t_roof / (ms_e2e * 1e-3 / args.steps),
               "roofline": "max(F/(G*P64), B_h2d/BW_h2d, B_d2h/BW_d2h) with P64=%.1f TFLOP/s/GPU and the "
                           "probed PCIe bandwidths" % FP64_PEAK_TFLOPS}

    timed = max(1, int(k_n))
    avg_ms = k_ms / timed
    flops_per_launch = k_fl / timed
    achieved = flops_per_launch / (avg_ms * 1e-3) / 1e12 if avg_ms > 0 else None
    mode = "rank mode: one process per GPU" if ws > 1 else "one process"
    roof = {"bound": "tensor", "achieved": achieved, "peak": FP64_PEAK_TFLOPS, "unit": "TFLOP/s",
            "frac": (achieved / FP64_PEAK_TFLOPS) if achieved else None, "traffic": traffic_from_profiles(T),
            "kernel": "dgemm_tma_kernel (grouped launch; TMA + mbarrier pipeline; FP64 DMMA.8x8x4 via mma.sync.m8n8k4.f64)",
            "peak_source": "derived: 148 SMs x 64 FP64 FMA/clk x 2 x 1965 MHz (no FP64 entry in "
                           "MEASURED_PEAKS.json); DMMA microbenchmark on this pool measured 37.07",
            "per_launch": "one grouped launch = a batch of tile tasks, 2*T^3 flops each (T=%d); %.3g flops "
                          "per launch on average; %d launches (all GPUs) timed with CUDA events on their kernel "
                          "stream in a second pass of the same K steps (launches serialised while timed), avg "
                          "%.3f ms; share of the step: %.3f" % (T, flops_per_launch, timed, avg_ms,
                                                                k_ms / G / (ms * 1.0))}
    line = {"metric": METRIC, "value": value, "unit": "TFLOP/s", "n_gpus": G, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms / args.steps, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": "DGEMM N=%d (m=n=k), tile %d, NN, alpha=1.5, beta=-0.75, %d GPU(s), grid %s, "
                                   "heuristics %s%s" % (N, T, G, "x".join(map(str, _grid(G))), args.topo,
                                                        "+optimistic" if args.optimistic else ""),
                       "N": N, "tile": T,
                       "parallelism": "%s; owner-computes 2D block-cyclic %s" % (mode, "x".join(map(str, _grid(G)))),
                       "value_mode": "data-on-device: A,B,C resident (prefetched), xk_dgemm_async + xk_sync per step",
                       "e2e_mode": "xk_dgemm from pinned host memory, all H2D/D2H in the timed region",
                       "l2": "no flush: each matrix is 8.6 GB >> 126 MB L2",
                       "inputs": "splitmix64 uniform [-1,1), seeds A=1 B=2 C=3"},
            "gpu_launches": launches, "clocks": clk, "roofline": roof, "e2e": e2e,
            "topology_MBps": topo["bw_MBps"], "task_rate_mflops": topo["task_rate_mflops"]}
    if rank == 0 and not args.no_cpu_baseline and ws == 1:
        line["cpu_baseline"] = cpu_baseline(N, A, B, C)
    xk.finalize()
    barrier(ws)
    if rank == 0:
        for p in paths:
            if os.path.exists(p):
                os.unlink(p)
        print(json.dumps(line), flush=True)


def _grid(G):
    q = max(c for c in range(1, G + 1) if G % c == 0 and c * c <= G)
    return (G // q, q)


def main():
    args = parse()
    rank, ws = dist_setup()
    if args.impl == "reference":
        run_reference(args, rank, ws)
    else:
        run_xk(args, rank, ws)
    if ws > 1:
        import torch.distributed as dist
        barrier(ws)
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
