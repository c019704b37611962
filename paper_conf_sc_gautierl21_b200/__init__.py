"""paper_conf_sc_gautierl21_b200 -- B200-native XKBlas-style multi-GPU level-3 BLAS.

Thin Python binding over the C ABI in include/xk.h (libxk.so, built in-tree).  Argument
marshalling only: planning, transfers and every tile kernel run inside libxk.so.  There
is no CPU fallback; if the library cannot be loaded the import of any entry point raises.

Matrices are numpy float64 arrays in Fortran (column-major) order, or raw addresses (int).
BLAS entry points return the BLAS info code (0, or -i for an invalid argument i) and raise
XKError for runtime failures (positive XK_ERR_* codes).
"""
import ctypes
import os

from . import _abi
from ._abi import (HOST, REC_D2H, REC_FIELDS, REC_H2D, REC_P2P, REC_TASK, ROUTINE_COHERENT,  # noqa: F401
                   ROUTINE_DGEMM, ROUTINE_INVALIDATE, ROUTINE_PREFETCH, ROUTINE_SYNC, SRC_HOST,
                   SRC_INFLIGHT, SRC_NONE, SRC_VALID, TOPO_HOME, TOPO_RANKED, TOPO_UNRANKED)

__all__ = ["init", "finalize", "register", "unregister", "dgemm", "dgemm_async",
           "memory_coherent_sync", "memory_coherent_async", "sync", "memory_invalidate",
           "memory_prefetch_async", "distribute_2dbc_async", "probe_host_links", "get_stats", "reset_stats", "set_kernel_timing",
           "get_topology", "PlanSession", "plan_dump", "dgemm_tile_device", "XKError", "lib"]

TOPO_NAMES = {"ranked": TOPO_RANKED, "unranked": TOPO_UNRANKED, "home": TOPO_HOME}


class XKError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__("xk error %d: %s" % (code, msg))
        self.code = code


def lib():
    return _abi.lib()


def _check(rc):
    if rc > 0:
        raise XKError(rc, (lib().xk_last_error() or b"").decode(errors="replace"))
    return rc


def _p(x):
    if x is None:
        return None
    if isinstance(x, int):
        return x
    if hasattr(x, "ctypes"):
        return x.ctypes.data
    if hasattr(x, "data_ptr"):
        return x.data_ptr()
    raise TypeError("expected numpy array, tensor or address, got %r" % type(x))


def _c(ch):
    return ch.encode() if isinstance(ch, str) else ch


# ---------------------------------------------------------------------------- lifecycle
def init(ngpus=0, tile=0, topo=None, optimistic=None, window=0, kstreams=0, probe=None,
         grid=None, phys=None, task_rate_mflops=0, rank=None, world=None, session=None, arena_bytes=0,
         mem_bytes=0):
    """xk_init.  `phys` maps logical GPUs to physical devices (logical-device mode).

    Rank mode (one process per GPU): every one of `world` processes calls
    init(rank=r, world=world, session=path) with the same unique `path` (see
    new_session_path); from then on every call is collective and host matrices must live
    in memory shared by the processes (shared_matrix)."""
    cfg = _abi.Config()
    lib().xk_config_default(ctypes.byref(cfg))
    if ngpus:
        cfg.ngpus = ngpus
    if tile:
        cfg.tile = tile
    if topo is not None:
        cfg.topo = TOPO_NAMES[topo] if isinstance(topo, str) else int(topo)
    if optimistic is not None:
        cfg.optimistic = int(bool(optimistic))
    if window:
        cfg.window = window
    if kstreams:
        cfg.kstreams = kstreams
    if probe is not None:
        cfg.probe = int(bool(probe))
    if grid is not None:
        cfg.grid_p, cfg.grid_q = grid
    if phys is not None:
        cfg.map_devices = 1
        for i, d in enumerate(phys):
            cfg.phys[i] = d
    if task_rate_mflops:
        cfg.task_rate_mflops = task_rate_mflops
    if world is not None and world > 1:
        cfg.rank, cfg.world = int(rank), int(world)
        cfg.session = os.fsencode(session)
        if phys is not None:  # phys[rank] = this process's device
            cfg.map_devices = 1
    if arena_bytes:
        cfg.arena_bytes = int(arena_bytes)
    if mem_bytes:
        cfg.mem_bytes = int(mem_bytes)
    return _check(lib().xk_init(ctypes.byref(cfg)))


# ---------------------------------------------------------------------------- rank mode
def new_session_path(tag="xk"):
    """A fresh path for the rank-mode session file (rank 0 picks it and shares it)."""
    d = "/dev/shm" if os.path.isdir("/dev/shm") else "/tmp"
    return os.path.join(d, "%s_%d_%s" % (tag, os.getpid(), os.urandom(6).hex()))


def session_selftest(path, rank, world, rounds, abort_at=-1, timeout_s=60.0):
    """Host side of rank mode's synchronisation (no CUDA): returns (rc, arrivals per round)."""
    out = (ctypes.c_int * max(1, rounds))()
    rc = lib().xk_session_selftest(os.fsencode(path), rank, world, rounds, abort_at, timeout_s, out)
    return rc, list(out)[:rounds]


def shared_matrix(path, rows, cols, create):
    """A column-major float64 host matrix backed by a file mapping (MAP_SHARED) that every
    rank-mode process maps: the "host memory" of the library's processes.  Plumbing only --
    the creator sizes the file, the others open it; each process registers its own mapping."""
    import numpy as np
    nbytes = max(8, int(rows) * int(cols) * 8)
    if create:
        with open(path, "wb") as f:
            f.truncate(nbytes)
    mm = np.memmap(path, dtype=np.float64, mode="r+", shape=(int(rows), int(cols)), order="F")
    return mm


def finalize():
    return _check(lib().xk_finalize())


def register(arr, nbytes=None):
    if nbytes is None:
        nbytes = arr.nbytes
    return _check(lib().xk_register(_p(arr), nbytes))


def unregister(arr):
    return _check(lib().xk_unregister(_p(arr)))


# ---------------------------------------------------------------------------- BLAS-3
def dgemm(transA, transB, m, n, k, alpha, A, lda, B, ldb, beta, C, ldc):
    return _check(lib().xk_dgemm(_c(transA), _c(transB), m, n, k, alpha, _p(A), lda, _p(B), ldb,
                                 beta, _p(C), ldc))


def dgemm_async(transA, transB, m, n, k, alpha, A, lda, B, ldb, beta, C, ldc):
    return _check(lib().xk_dgemm_async(_c(transA), _c(transB), m, n, k, alpha, _p(A), lda, _p(B),
                                       ldb, beta, _p(C), ldc))


def dsyrk(uplo, trans, n, k, alpha, A, lda, beta, C, ldc, asynchronous=False):
    f = lib().xk_dsyrk_async if asynchronous else lib().xk_dsyrk
    return _check(f(_c(uplo), _c(trans), n, k, alpha, _p(A), lda, beta, _p(C), ldc))


def dsyr2k(uplo, trans, n, k, alpha, A, lda, B, ldb, beta, C, ldc, asynchronous=False):
    f = lib().xk_dsyr2k_async if asynchronous else lib().xk_dsyr2k
    return _check(f(_c(uplo), _c(trans), n, k, alpha, _p(A), lda, _p(B), ldb, beta, _p(C), ldc))


def dsymm(side, uplo, m, n, alpha, A, lda, B, ldb, beta, C, ldc, asynchronous=False):
    f = lib().xk_dsymm_async if asynchronous else lib().xk_dsymm
    return _check(f(_c(side), _c(uplo), m, n, alpha, _p(A), lda, _p(B), ldb, beta, _p(C), ldc))


def dtrmm(side, uplo, transA, diag, m, n, alpha, A, lda, B, ldb, asynchronous=False):
    f = lib().xk_dtrmm_async if asynchronous else lib().xk_dtrmm
    return _check(f(_c(side), _c(uplo), _c(transA), _c(diag), m, n, alpha, _p(A), lda, _p(B), ldb))


def dtrsm(side, uplo, transA, diag, m, n, alpha, A, lda, B, ldb, asynchronous=False):
    f = lib().xk_dtrsm_async if asynchronous else lib().xk_dtrsm
    return _check(f(_c(side), _c(uplo), _c(transA), _c(diag), m, n, alpha, _p(A), lda, _p(B), ldb))


# ---------------------------------------------------------------------------- coherence
def memory_coherent_sync(m, n, A, lda):
    return _check(lib().xk_memory_coherent_sync(m, n, _p(A), lda))


def memory_coherent_async(m, n, A, lda):
    return _check(lib().xk_memory_coherent_async(m, n, _p(A), lda))


def sync():
    return _check(lib().xk_sync())


def memory_invalidate(m, n, A, lda):
    return _check(lib().xk_memory_invalidate(m, n, _p(A), lda))


def memory_prefetch_async(m, n, A, lda):
    return _check(lib().xk_memory_prefetch_async(m, n, _p(A), lda))


def distribute_2dbc_async(m, n, A, lda, P, Q, mb=1, nb=1):
    """xk_distribute_2dbc_async (the paper's xkblas_distribute_2Dblock_cyclic_async)."""
    return _check(lib().xk_distribute_2dbc_async(m, n, _p(A), lda, P, Q, mb, nb))


# ---------------------------------------------------------------------------- observability
def get_stats():
    st = _abi.Stats()
    _check(lib().xk_get_stats(ctypes.byref(st)))
    G = st.ngpus
    out = {"ngpus": G}
    for f in ("h2d_bytes", "d2h_bytes", "p2p_in_bytes", "p2p_out_bytes", "tasks", "flops"):
        out[f] = list(getattr(st, f))[:G]
    for f in ("forwards_inflight", "forwards_valid", "kernel_launches", "host_registrations",
              "kernel_ms_total", "kernel_timed_launches", "kernel_timed_flops", "plan_records",
              "plan_records_local", "host_issue_ms", "device_allocs", "device_alloc_ms"):
        out[f] = getattr(st, f)
    out["trace_ms"] = dict(zip(("h2d", "p2p", "kernel", "d2h"), list(st.trace_ms)))
    out["link_bytes"] = [[st.link_bytes[s * (G + 1) + d] for d in range(G + 1)] for s in range(G + 1)]
    return out


def trace(path):
    """Start (path) or stop and write (None) the Chrome-trace timeline."""
    return _check(lib().xk_trace(path.encode() if path else None))


def reset_stats():
    return _check(lib().xk_reset_stats())


def set_kernel_timing(on):
    return _check(lib().xk_set_kernel_timing(int(bool(on))))


def get_topology():
    t = _abi.Topo()
    _check(lib().xk_get_topology(ctypes.byref(t)))
    G = t.ngpus
    bw = [[t.bw_MBps[s * (G + 1) + d] for d in range(G + 1)] for s in range(G + 1)]
    rank = [[t.perf_rank[s * G + d] for d in range(G)] for s in range(G)]
    return {"ngpus": G, "bw_MBps": bw, "perf_rank": rank, "task_rate_mflops": t.task_rate_mflops,
            "host_all_MBps": {"h2d": t.host_all_MBps[0], "d2h": t.host_all_MBps[1],
                              "duplex": t.host_all_MBps[2]},
            "host_probe_bytes": t.host_probe_bytes}


def probe_host_links(bytes_per_gpu=4 << 30):
    """xk_probe_host_links: all GPUs copy at once (H2D, D2H, duplex); see get_topology()."""
    return _check(lib().xk_probe_host_links(int(bytes_per_gpu)))


# ---------------------------------------------------------------------------- planner
def _topo(bw, rate_mflops):
    G = len(bw) - 1
    t = _abi.Topo()
    t.ngpus = G
    for s in range(G + 1):
        for d in range(G + 1):
            t.bw_MBps[s * (G + 1) + d] = int(bw[s][d])
    t.task_rate_mflops = int(rate_mflops)
    return t


def _flags(topo="ranked", optimistic=True, window=4, grid=(0, 0), tile=2048, mem_bytes=0):
    f = _abi.Flags()
    f.mem_bytes = int(mem_bytes)
    f.topo = TOPO_NAMES[topo] if isinstance(topo, str) else int(topo)
    f.optimistic = int(bool(optimistic))
    f.window = window
    f.grid_p, f.grid_q = grid
    f.tile = tile
    return f


def make_call(routine=ROUTINE_DGEMM, transA="N", transB="N", m=0, n=0, k=0, alpha=1.0, beta=0.0,
              A=0, lda=1, B=0, ldb=1, C=0, ldc=1, sync=False, uplo="L", side="L", diag="N",
              grid=(0, 0), mb=0, nb=0):
    c = _abi.Call()
    c.grid_p, c.grid_q = grid
    c.mb, c.nb = mb, nb
    c.routine = routine
    c.transA, c.transB = _c(transA), _c(transB)
    c.uplo, c.side, c.diag = _c(uplo), _c(side), _c(diag)
    c.m, c.n, c.k = m, n, k
    c.alpha, c.beta = alpha, beta
    c.A, c.lda, c.B, c.ldb, c.C, c.ldc = A, lda, B, ldb, C, ldc
    c.sync = int(bool(sync))
    return c


class PlanSession:
    """Planner session with G virtual GPUs and an injected (G+1)^2 link matrix (MB/s)."""

    def __init__(self, bw, rate_mflops=35000000, **flags):
        self._h = ctypes.c_void_p()
        t = _topo(bw, rate_mflops)
        f = _flags(**flags)
        _check(lib().xk_plan_session_create(ctypes.byref(t), ctypes.byref(f), ctypes.byref(self._h)))

    def call(self, call, cap=1 << 16):
        while True:
            buf = (_abi.PlanRec * cap)()
            n = ctypes.c_int64(0)
            rc = lib().xk_plan_session_call(self._h, ctypes.byref(call), buf, cap, ctypes.byref(n))
            if rc == _abi.XK_ERR_CAPACITY:
                raise XKError(rc, "capacity (need %d)" % n.value)
            _check(rc)
            return [buf[i].as_tuple() for i in range(n.value)]

    def close(self):
        if self._h:
            lib().xk_plan_session_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def plan_dump(call, bw, rate_mflops=35000000, cap=1 << 16, **flags):
    s = PlanSession(bw, rate_mflops, **flags)
    try:
        return s.call(call, cap)
    finally:
        s.close()


# ---------------------------------------------------------------------------- kernel entry
def dgemm_tile_device(transA, transB, m, n, k, alpha, A, lda, B, ldb, beta, C, ldc, stream=0):
    """One tile task on device pointers (torch tensors or raw addresses)."""
    return _check(lib().xk_dgemm_tile_device(_c(transA), _c(transB), m, n, k, alpha, _p(A), lda,
                                             _p(B), ldb, beta, _p(C), ldc, stream or None))
