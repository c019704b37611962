#!/usr/bin/env python
"""bench.py -- end-to-end DGEMM TFLOP/s of the B200-native XKBlas-style library.

Metric (BASELINE.json): "end-to-end DGEMM TFlop/s at N=32768/65536 on 1/2/4/8 B200,
% FP64 roofline".  Workload at N GPUs: DGEMM N=32768 (m=n=k), tile T=4096 (the best of the
paper's tile sweep {1024, 2048, 4096}, measured in profiles/), NN,
alpha=1.5, beta=-0.75 (reading Q10), column-major host matrices from the seeded
splitmix64 generator (uniform [-1,1)), owner grid near-square P x Q.

A step is one whole DGEMM (every §8(a) row: tiling, owner map, directory, source
selection, transfers, tile kernels, coherence):
  value : the metric, end to end -- xk_dgemm (synchronous) from pinned host buffers; every
          step copies A, B, C tiles H2D and C D2H inside the timed region and ends with C
          coherent on the host.  CUDA events + a full device
          synchronize on both sides of the K steps, barrier and max over ranks.
  e2e   : the same K calls timed by the host wall clock (API entry to return), with the
          H2D/D2H bytes per step and the fraction of the e2e roofline, the
          host-link terms taken from a concurrent probe of all GPUs' links.
  data_on_device : A, B, C already resident in HBM (prefetched, untimed); xk_dgemm_async +
          xk_sync per step (paper §IV-C, Table II "data on device").
  roofline : the tile kernel (grouped launch) timed by CUDA events in a second pass of the
          data-on-device steps, against the FP64 peak.
  ablation (G > 1) : BASELINE configs[1], N=16384 T=2048, every heuristic mode (paper Table II).
  north_star (G = 8, or --north-star) : N=65536 T=4096 host-resident vs 70% of G x FP64 peak.
Inputs (8.6 GB per matrix) are far larger than L2 (126 MB): no flush needed.

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
    ap.add_argument("--no-ablation", action="store_true", help="skip the N>1 heuristic ablation")
    ap.add_argument("--north-star", action="store_true", help="run the N=65536 north-star point at any G")
    ap.add_argument("--no-north-star", action="store_true")
    ap.add_argument("--ns-n", type=int, default=65536, help="north-star N (default 65536)")
    ap.add_argument("--host-probe-mib", type=int, default=4096,
                    help="bytes per GPU per direction of the concurrent host-link probe")
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


def traffic_from_profiles(T, tasks_per_launch):
    """DRAM bytes per launch for the roofline: the committed ncu capture's bytes per tile task
    (one full capture of a grouped launch at this tile size) times the average tasks per
    launch of the timed pass -- per launch, like `achieved`."""
    p = os.path.join(ROOT, "profiles", "dgemm_tile_ncu.json")
    try:
        with open(p) as f:
            d = json.load(f)
        if int(d.get("tile", 0)) == T and d.get("tasks_per_launch"):
            return d["dram_bytes_per_launch"] / d["tasks_per_launch"] * tasks_per_launch
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
    rank 0 fills them, the others map them after a barrier.  Returns (A, B, C, paths, base):
    only real files in `paths` are unlinked at the end; `base` names the session files."""
    import inputs
    import paper_conf_sc_gautierl21_b200 as xk
    if ws == 1:
        A, B, C = make_inputs(N)
        return A, B, C, [], None
    import torch.distributed as dist
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
            fds = [os.memfd_create("xkbench%d%s" % (N, s)) for s in "ABC"]
            _MEMFDS.extend(fds)
            for fd in fds:
                os.ftruncate(fd, N * N * 8)
            paths = ["/proc/%d/fd/%d" % (os.getpid(), fd) for fd in fds]
        obj = [(paths, base)]
    dist.broadcast_object_list(obj, src=0, group=_HOST_GROUP)
    paths, base = obj[0]
    mats = [xk.shared_matrix(p, N, N, create=False) for p in paths]
    if rank == 0:
        inputs.set_threads(len(os.sched_getaffinity(0)))  # torchrun sets OMP_NUM_THREADS=1
        for M, seed in zip(mats, (inputs.SEED_A, inputs.SEED_B, inputs.SEED_C)):
            inputs.uniform(seed, N, N, out=M)
    barrier(ws)
    return mats[0], mats[1], mats[2], [p for p in paths if not p.startswith("/proc/")], base


_MEMFDS = []


def sum_over_ranks(vals, ws):
    if ws == 1:
        return vals
    import torch
    import torch.distributed as dist
    t = torch.tensor(vals, dtype=torch.float64)
    dist.all_reduce(t, op=dist.ReduceOp.SUM, group=_HOST_GROUP)
    return t.tolist()


def gather_per_gpu(v, ws):
    """Rank mode: every rank's own value, in rank order (rank r drives GPU r)."""
    if ws == 1:
        return [v]
    vec = [0.0] * ws
    vec[int(os.environ.get("RANK", "0"))] = float(v)
    return sum_over_ranks(vec, ws)


class Lib:
    """One library session (xk_init .. xk_finalize) of the run; rank mode gets a fresh
    session file per (re-)initialisation (the heuristic ablation re-initialises per mode)."""

    def __init__(self, args, rank, ws, base):
        self.args, self.rank, self.ws, self.base, self.n = args, rank, ws, base, 0

    def init(self, mats, tile, topo="ranked", optimistic=True, probe=True):
        import paper_conf_sc_gautierl21_b200 as xk
        kw = dict(tile=tile, topo=topo, optimistic=bool(optimistic), kstreams=self.args.kstreams, probe=probe)
        if self.ws > 1:
            self.n += 1
            xk.init(rank=self.rank, world=self.ws, session="%s.session%d" % (self.base, self.n), **kw)
        else:
            xk.init(ngpus=self.args.gpus, **kw)
        for X in mats:
            xk.register(X)
        return xk


def host_step_bytes(xk, steps, ws):
    se = xk.get_stats()
    mine = [sum(se["h2d_bytes"]), sum(se["d2h_bytes"]), sum(se["p2p_in_bytes"])]
    per_gpu_h2d = se["h2d_bytes"][:se["ngpus"]] if ws == 1 else gather_per_gpu(se["h2d_bytes"][int(os.environ.get("RANK", "0"))], ws)
    tot = [int(v) // steps for v in sum_over_ranks(mine, ws)]
    return tot[0], tot[1], tot[2], [int(v) // steps for v in per_gpu_h2d]


def timed_host_resident(xk, A, B, C, N, T, steps, warmup, ws, timer, clocks=None, rank=0, gpus=1):
    """xk_dgemm from pinned host memory: every H2D/D2H inside the timed region, C coherent on
    the host at the end of each call.  Device time (CUDA events, full device synchronize on
    both sides, max over ranks) and host wall time of the API calls."""
    flops = 2.0 * N * N * N
    for _ in range(warmup):
        xk.dgemm("N", "N", N, N, N, ALPHA, A, A.strides[1] // 8, B, B.strides[1] // 8, BETA, C, C.strides[1] // 8)
    xk.reset_stats()
    barrier(ws)
    if clocks is not None and rank == 0:
        clocks.start()
    wall = 0.0
    timer.start()
    for _ in range(steps):
        t0 = time.perf_counter()
        xk.dgemm("N", "N", N, N, N, ALPHA, A, A.strides[1] // 8, B, B.strides[1] // 8, BETA, C, C.strides[1] // 8)
        wall += time.perf_counter() - t0
    ms = max_over_ranks(timer.stop_ms(), ws)
    wall_ms = max_over_ranks(1000.0 * wall, ws)
    barrier(ws)
    clk = clocks.stop(gpus) if (clocks is not None and rank == 0) else None
    launches = int(sum_over_ranks([xk.get_stats()["kernel_launches"]], ws)[0])
    h2d, d2h, p2p, per_gpu = host_step_bytes(xk, steps, ws)
    return {"tflops": steps * flops / (ms * 1e-3) / 1e12, "ms": ms / steps,
            "wall_tflops": steps * flops / (wall_ms * 1e-3) / 1e12, "wall_ms": wall_ms / steps,
            "h2d": h2d, "d2h": d2h, "p2p": p2p, "h2d_per_gpu": per_gpu, "launches": launches, "clocks": clk}


def e2e_roofline(topo, G, N, h2d, d2h, p2p):
    """T_roof = max(F/(G*P64), B_h2d/BW_h2d(G), B_d2h/BW_d2h(G), (B_h2d+B_d2h)/BW_duplex(G),
    B_p2p/BW_p2p(G)); BW_*(G) = all GPUs copying at once (probed by
    xk_probe_host_links), BW_p2p(G) = G x the slowest probed peer link."""
    flops = 2.0 * N * N * N
    ha = topo.get("host_all_MBps") or {}
    if ha.get("h2d"):
        bw_h2d, bw_d2h, bw_dup = ha["h2d"] * 1e6, ha["d2h"] * 1e6, ha["duplex"] * 1e6
        src = "concurrent probe (all %d GPU(s) at once, %d MiB per GPU per direction)" % (
            G, topo.get("host_probe_bytes", 0) >> 20)
    else:
        bw_h2d = min(topo["bw_MBps"][G][g] for g in range(G)) * 1e6 * G
        bw_d2h = min(topo["bw_MBps"][g][G] for g in range(G)) * 1e6 * G
        bw_dup = bw_h2d + bw_d2h
        src = "G x the per-GPU probe (no concurrent probe)"
    terms = {"fp64": flops / (G * FP64_PEAK_TFLOPS * 1e12), "h2d": h2d / bw_h2d, "d2h": d2h / bw_d2h,
             "duplex": (h2d + d2h) / bw_dup}
    if G > 1 and p2p:
        peer = min(topo["bw_MBps"][s][d] for s in range(G) for d in range(G) if s != d) * 1e6
        terms["p2p"] = p2p / (peer * G)
    return max(terms.values()), {k: round(v * 1e3, 3) for k, v in terms.items()}, src


ABLATION_MODES = (("full", "ranked", True), ("no_optimistic", "ranked", False),
                  ("no_optimistic_no_topo", "unranked", False), ("home", "home", True))


def run_ablation(lib, A, B, C, ws, timer, N=16384, T=2048, steps=2):
    """Paper Table II / BASELINE configs[1]: DGEMM N=16384, T=2048 host-resident, every
    heuristic mode (one library session each), 1 warm-up + `steps` timed calls; TF/s and
    H2D bytes per GPU.  The N x N operands are views of the bench matrices (ld = their N)."""
    out = {"config": "DGEMM N=%d tile %d NN alpha=1.5 beta=-0.75 host-resident, %d GPU(s)" % (N, T, lib.args.gpus if ws == 1 else ws)}
    Av, Bv, Cv = A[:N, :N], B[:N, :N], C[:N, :N]
    for name, topo, opt in ABLATION_MODES:
        xk = lib.init((A, B, C), T, topo=topo, optimistic=opt)
        r = timed_host_resident(xk, Av, Bv, Cv, N, T, steps, 1, ws, timer)
        xk.finalize()
        out[name] = {"tflops": r["tflops"], "ms_per_step": r["ms"], "h2d_bytes": r["h2d"],
                     "p2p_bytes": r["p2p"], "h2d_bytes_per_gpu": r["h2d_per_gpu"]}
    full = out["full"]["tflops"]
    for name, _, _ in ABLATION_MODES[1:]:
        out[name]["vs_full"] = out[name]["tflops"] / full - 1.0
    return out


def host_mem_available():
    try:
        with open("/proc/meminfo") as f:
            for ln in f:
                if ln.startswith("MemAvailable:"):
                    return int(ln.split()[1]) * 1024
    except OSError:
        pass
    return 0


def run_north_star(args, rank, ws, timer, N=65536, T=4096, steps=2):
    """north_star: host-resident DGEMM N=65536, T=4096 on all GPUs, 1 warm-up + 2 steps;
    fraction of G x the FP64 peak (target >= 0.70)."""
    G = ws if ws > 1 else args.gpus
    need = 3 * N * N * 8
    ok = host_mem_available() > 1.15 * need
    ok = sum_over_ranks([1.0 if ok else 0.0], ws)[0] == ws
    if not ok:
        return {"skipped": "host memory: %d GB needed for A, B, C" % (need >> 30)}
    A, B, C, paths, base = share_inputs(N, rank, ws)
    try:
        lib = Lib(args, rank, ws, base or "")
        xk = lib.init((A, B, C), T)
        try:
            xk.probe_host_links(1 << 30)
        except xk.XKError:
            pass
        topo = xk.get_topology()
        r = timed_host_resident(xk, A, B, C, N, T, steps, 1, ws, timer)
        xk.finalize()
    finally:
        barrier(ws)
        if rank == 0:
            for p in paths:
                if os.path.exists(p):
                    os.unlink(p)
    t_roof, terms, src = e2e_roofline(topo, G, N, r["h2d"], r["d2h"], r["p2p"])
    return {"config": "DGEMM N=%d tile %d NN host-resident on %d GPU(s)" % (N, T, G), "tflops": r["tflops"],
            "ms_per_step": r["ms"], "frac_of_fp64_peak": r["tflops"] / (G * FP64_PEAK_TFLOPS),
            "target_frac": 0.70, "roofline_frac": t_roof / (r["ms"] * 1e-3), "roofline_terms_ms": terms,
            "h2d_bytes_per_step": r["h2d"], "d2h_bytes_per_step": r["d2h"], "p2p_bytes_per_step": r["p2p"]}


def run_xk(args, rank, ws):
    """ws == 1: one process drives the GPU(s) (--gpus G > 1 = the single-process multi-GPU
    runtime).  Under torchrun (ws > 1): rank mode -- one process per GPU, every xk call
    collective, each process executing its own GPU's part of the identical plan."""
    G = ws if ws > 1 else args.gpus
    N, T = args.n, args.tile
    flops = 2.0 * N * N * N
    A, B, C, paths, base = share_inputs(N, rank, ws)
    lib = Lib(args, rank, ws, base)
    xk = lib.init((A, B, C), T)
    # host links with every GPU copying at once (untimed set-up, like a1); a
    # failure (collective in rank mode) leaves the e2e roofline on the per-GPU probe
    try:
        xk.probe_host_links(args.host_probe_mib << 20)
    except xk.XKError as e:
        print("bench: concurrent host-link probe failed: %s" % e, file=sys.stderr)
    topo = xk.get_topology()
    timer = DevTimer()
    clocks = ClockSampler()

    # ---------------- value: the metric, host-resident end to end through xk_dgemm
    host = timed_host_resident(xk, A, B, C, N, T, args.steps, args.warmup, ws, timer, clocks, rank, G)
    t_roof, terms, bw_src = e2e_roofline(topo, G, N, host["h2d"], host["d2h"], host["p2p"])

    # ---------------- data-on-device: A, B, C resident in HBM (prefetched, untimed)
    for X in (A, B, C):
        xk.memory_prefetch_async(N, N, X, N)
    xk.sync()
    for _ in range(args.warmup):
        xk.dgemm_async("N", "N", N, N, N, ALPHA, A, N, B, N, BETA, C, N)
        xk.sync()
    xk.reset_stats()
    barrier(ws)
    timer.start()
    for _ in range(args.steps):
        xk.dgemm_async("N", "N", N, N, N, ALPHA, A, N, B, N, BETA, C, N)
        xk.sync()
    ms_dod = max_over_ranks(timer.stop_ms(), ws)
    barrier(ws)
    dod_launches = int(sum_over_ranks([xk.get_stats()["kernel_launches"]], ws)[0])
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
    xk.finalize()
    dod = {"value": args.steps * flops / (ms_dod * 1e-3) / 1e12, "unit": "TFLOP/s",
           "ms_per_step": ms_dod / args.steps, "gpu_launches": dod_launches,
           "mode": "A, B, C resident in HBM (prefetched, untimed); xk_dgemm_async + xk_sync per step, "
                   "C updated on the GPUs (no host traffic)"}

    ablation = None
    if G > 1 and not args.no_ablation and N >= 16384:
        try:  # an extra: a failure here must not cost the main line
            ablation = run_ablation(lib, A, B, C, ws, timer)
        except Exception as e:  # noqa: BLE001
            ablation = {"error": repr(e)[:300]}
    cpu = cpu_baseline(N, A, B, C) if (rank == 0 and not args.no_cpu_baseline and ws == 1) else None
    barrier(ws)
    if rank == 0:
        for p in paths:
            if os.path.exists(p):
                os.unlink(p)
    north = None
    if (G == 8 or args.north_star) and not args.no_north_star:
        try:
            north = run_north_star(args, rank, ws, timer, N=args.ns_n)
        except Exception as e:  # noqa: BLE001
            north = {"error": repr(e)[:300]}

    timed = max(1, int(k_n))
    avg_ms = k_ms / timed
    line = assemble_line(args, G, ws, N, T, host, t_roof, terms, bw_src, dod, avg_ms, k_fl / timed, timed,
                         k_ms, ms_dod, topo, ablation, north, cpu)
    if rank == 0:
        print(json.dumps(line), flush=True)


def assemble_line(args, G, ws, N, T, host, t_roof, terms, bw_src, dod, avg_ms, flops_per_launch, timed,
                  k_ms, ms_dod, topo, ablation=None, north=None, cpu=None):
    """The one JSON line (pure: tested on CPU by tests/test_bench_line.py)."""
    achieved = flops_per_launch / (avg_ms * 1e-3) / 1e12 if avg_ms > 0 else None
    mode = "rank mode: one process per GPU" if ws > 1 else "one process"
    grid = "x".join(map(str, _grid(G)))
    roof = {"bound": "tensor", "achieved": achieved, "peak": FP64_PEAK_TFLOPS, "unit": "TFLOP/s",
            "frac": (achieved / FP64_PEAK_TFLOPS) if achieved else None,
            "traffic": traffic_from_profiles(T, flops_per_launch / (2.0 * T ** 3)),
            "traffic_note": "ncu dram__bytes_read+write of one grouped launch (profiles/dgemm_tile_ncu.json) per tile "
                            "task x the average tasks per timed launch; algorithmic %.3g bytes per launch (A, B, C "
                            "read + C write per task)" % (4 * 8.0 * T * T * flops_per_launch / (2.0 * T ** 3)),
            "kernel": "dgemm_tma_kernel (grouped launch; TMA + mbarrier pipeline; FP64 DMMA.8x8x4 via mma.sync.m8n8k4.f64)",
            "peak_source": "derived: 148 SMs x 64 FP64 FMA/clk x 2 x 1965 MHz (no FP64 entry in "
                           "MEASURED_PEAKS.json); DMMA microbenchmark on this pool measured 37.07",
            "per_launch": "one grouped launch = a batch of tile tasks, 2*T^3 flops each (T=%d); %.3g flops "
                          "per launch on average; %d launches (all GPUs) timed with CUDA events on their kernel "
                          "stream in a second pass of the data-on-device steps (launches serialised while "
                          "timed), avg %.3f ms; share of the data-on-device step: %.3f"
                          % (T, flops_per_launch, timed, avg_ms, k_ms / G / max(ms_dod, 1e-9))}
    e2e = {"value": host["wall_tflops"], "unit": "TFLOP/s", "h2d_bytes_per_step": host["h2d"],
           "d2h_bytes_per_step": host["d2h"], "p2p_bytes_per_step": host["p2p"],
           "ms_per_step": host["wall_ms"], "roofline_frac": t_roof / (host["wall_ms"] * 1e-3),
           "clock": "host wall clock from xk_dgemm entry to its return (C coherent on the host), summed "
                    "over the K calls, max over ranks",
           "roofline": "max(F/(G*P64), B_h2d/BW_h2d(G), B_d2h/BW_d2h(G), (B_h2d+B_d2h)/BW_duplex(G)[, "
                       "B_p2p/BW_p2p(G)]) with P64=%.1f TFLOP/s/GPU; BW: %s" % (FP64_PEAK_TFLOPS, bw_src),
           "roofline_terms_ms": terms}
    line = {"metric": METRIC, "value": host["tflops"], "unit": "TFLOP/s", "n_gpus": G, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": host["ms"], "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": "DGEMM N=%d (m=n=k), tile %d, NN, alpha=1.5, beta=-0.75, host-resident "
                                   "column-major, %d GPU(s), grid %s, heuristics %s%s"
                                   % (N, T, G, grid, args.topo, "+optimistic" if args.optimistic else ""),
                       "N": N, "tile": T,
                       "parallelism": "%s; owner-computes 2D block-cyclic %s" % (mode, grid),
                       "value_mode": "end to end (the metric): xk_dgemm from pinned host memory, every "
                                     "H2D/D2H inside the timed region, C coherent on the host after each "
                                     "step; CUDA events with a full device synchronize on both sides",
                       "l2": "no flush: each matrix is %.1f GB >> 126 MB L2" % (8.0 * N * N / 1e9),
                       "inputs": "splitmix64 uniform [-1,1), seeds A=1 B=2 C=3"},
            "gpu_launches": host["launches"], "clocks": host["clocks"], "roofline": roof, "e2e": e2e,
            "roofline_frac_e2e": t_roof / (host["ms"] * 1e-3),
            "data_on_device": dod, "h2d_bytes_per_gpu": host["h2d_per_gpu"],
            "topology_MBps": topo["bw_MBps"], "host_links_all_MBps": topo.get("host_all_MBps"),
            "task_rate_mflops": topo["task_rate_mflops"]}
    if ablation is not None:
        line["ablation"] = ablation
    if north is not None:
        line["north_star"] = north
    if cpu is not None:
        line["cpu_baseline"] = cpu
    return line


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
