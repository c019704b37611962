"""ctypes mirror of include/xk.h (argument marshalling only; every step of the path runs in
libxk.so).  The library is built in-tree by tools/build_native.build_xk() and loaded from
this package directory; there is no fallback of any kind: a missing library raises.
"""
import ctypes
import os

MAX_GPUS = 16
HOST = -1

XK_OK = 0
XK_ERR_NOT_INITIALIZED = 1
XK_ERR_CUDA = 2
XK_ERR_OOM = 3
XK_ERR_CONFIG = 4
XK_ERR_CAPACITY = 5
XK_ERR_UNSUPPORTED = 6
XK_ERR_NO_DEVICE = 7
XK_ERR_INTERNAL = 8

TOPO_RANKED, TOPO_UNRANKED, TOPO_HOME = 0, 1, 2
REC_H2D, REC_P2P, REC_TASK, REC_D2H = 0, 1, 2, 3
SRC_NONE, SRC_VALID, SRC_INFLIGHT, SRC_HOST = 0, 1, 2, 3
ROUTINE_DGEMM, ROUTINE_DSYRK, ROUTINE_DSYR2K, ROUTINE_DSYMM, ROUTINE_DTRMM, ROUTINE_DTRSM = 0, 1, 2, 3, 4, 5
OP_GEMM, OP_SCALE, OP_GEMM_TRI, OP_SYMM_DIAG, OP_TRMM_DIAG, OP_TRSM_DIAG = 0, 1, 2, 3, 4, 5
ROUTINE_COHERENT, ROUTINE_SYNC, ROUTINE_INVALIDATE, ROUTINE_PREFETCH = 100, 101, 102, 103
ROUTINE_DISTRIBUTE = 104

i64 = ctypes.c_int64
u64 = ctypes.c_uint64
c_int = ctypes.c_int
c_double = ctypes.c_double
c_char = ctypes.c_char
vp = ctypes.c_void_p


class Config(ctypes.Structure):
    _fields_ = [("ngpus", c_int), ("phys", c_int * MAX_GPUS), ("map_devices", c_int),
                ("grid_p", c_int), ("grid_q", c_int), ("tile", i64), ("topo", c_int),
                ("optimistic", c_int), ("window", c_int), ("kstreams", c_int), ("probe", c_int),
                ("task_rate_mflops", i64), ("rank", c_int), ("world", c_int), ("arena_bytes", i64),
                ("session", ctypes.c_char * 128), ("mem_bytes", i64)]


class Stats(ctypes.Structure):
    _fields_ = [("ngpus", c_int), ("h2d_bytes", i64 * MAX_GPUS), ("d2h_bytes", i64 * MAX_GPUS),
                ("p2p_in_bytes", i64 * MAX_GPUS), ("p2p_out_bytes", i64 * MAX_GPUS),
                ("tasks", i64 * MAX_GPUS), ("flops", i64 * MAX_GPUS),
                ("forwards_inflight", i64), ("forwards_valid", i64), ("kernel_launches", i64),
                ("host_registrations", i64), ("kernel_ms_total", c_double),
                ("kernel_timed_launches", i64), ("kernel_timed_flops", i64),
                ("link_bytes", i64 * ((MAX_GPUS + 1) * (MAX_GPUS + 1))),
                ("trace_ms", c_double * 4), ("plan_records", i64), ("plan_records_local", i64),
                ("host_issue_ms", c_double), ("device_allocs", i64), ("device_alloc_ms", c_double)]


class Topo(ctypes.Structure):
    _fields_ = [("ngpus", c_int), ("bw_MBps", i64 * ((MAX_GPUS + 1) * (MAX_GPUS + 1))),
                ("perf_rank", c_int * (MAX_GPUS * MAX_GPUS)), ("task_rate_mflops", i64),
                ("host_all_MBps", i64 * 3), ("host_probe_bytes", i64)]


class Flags(ctypes.Structure):
    _fields_ = [("topo", c_int), ("optimistic", c_int), ("window", c_int), ("grid_p", c_int),
                ("grid_q", c_int), ("tile", i64), ("mem_bytes", i64)]


class Call(ctypes.Structure):
    _fields_ = [("routine", c_int), ("transA", c_char), ("transB", c_char), ("uplo", c_char),
                ("side", c_char), ("diag", c_char), ("m", i64), ("n", i64),
                ("k", i64), ("alpha", c_double), ("beta", c_double), ("A", u64), ("lda", u64),
                ("B", u64), ("ldb", u64), ("C", u64), ("ldc", u64), ("sync", c_int),
                ("grid_p", c_int), ("grid_q", c_int), ("mb", i64), ("nb", i64)]


class PlanRec(ctypes.Structure):
    _fields_ = [("seq", i64), ("kind", ctypes.c_int32), ("operand", ctypes.c_int32), ("bi", i64),
                ("bj", i64), ("tk", i64), ("version", i64), ("dst", ctypes.c_int32),
                ("src", ctypes.c_int32), ("src_state", ctypes.c_int32), ("depth", ctypes.c_int32),
                ("op", ctypes.c_int32), ("reserved", ctypes.c_int32),
                ("t_start", i64), ("t_end", i64), ("work", i64), ("dep", i64 * 4)]

    def as_tuple(self):
        return (self.seq, self.kind, self.operand, self.bi, self.bj, self.tk, self.version,
                self.dst, self.src, self.src_state, self.depth, self.t_start, self.t_end,
                self.work, tuple(self.dep), self.op)


REC_FIELDS = ("seq", "kind", "operand", "bi", "bj", "tk", "version", "dst", "src", "src_state",
              "depth", "t_start", "t_end", "work", "dep", "op")

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libxk.so")
_LIB = None

# (name, restype, argtypes) for every symbol include/xk.h declares
_D = c_double
_SIGS = [
    ("xk_config_default", None, [ctypes.POINTER(Config)]),
    ("xk_init", c_int, [ctypes.POINTER(Config)]),
    ("xk_finalize", c_int, []),
    ("xk_register", c_int, [vp, ctypes.c_size_t]),
    ("xk_unregister", c_int, [vp]),
    ("xk_last_error", ctypes.c_char_p, []),
    ("xk_dgemm", c_int, [c_char, c_char, i64, i64, i64, _D, vp, i64, vp, i64, _D, vp, i64]),
    ("xk_dgemm_async", c_int, [c_char, c_char, i64, i64, i64, _D, vp, i64, vp, i64, _D, vp, i64]),
    ("xk_dsyrk", c_int, [c_char, c_char, i64, i64, _D, vp, i64, _D, vp, i64]),
    ("xk_dsyrk_async", c_int, [c_char, c_char, i64, i64, _D, vp, i64, _D, vp, i64]),
    ("xk_dsyr2k", c_int, [c_char, c_char, i64, i64, _D, vp, i64, vp, i64, _D, vp, i64]),
    ("xk_dsyr2k_async", c_int, [c_char, c_char, i64, i64, _D, vp, i64, vp, i64, _D, vp, i64]),
    ("xk_dsymm", c_int, [c_char, c_char, i64, i64, _D, vp, i64, vp, i64, _D, vp, i64]),
    ("xk_dsymm_async", c_int, [c_char, c_char, i64, i64, _D, vp, i64, vp, i64, _D, vp, i64]),
    ("xk_dtrmm", c_int, [c_char, c_char, c_char, c_char, i64, i64, _D, vp, i64, vp, i64]),
    ("xk_dtrmm_async", c_int, [c_char, c_char, c_char, c_char, i64, i64, _D, vp, i64, vp, i64]),
    ("xk_dtrsm", c_int, [c_char, c_char, c_char, c_char, i64, i64, _D, vp, i64, vp, i64]),
    ("xk_dtrsm_async", c_int, [c_char, c_char, c_char, c_char, i64, i64, _D, vp, i64, vp, i64]),
    ("xk_memory_coherent_sync", c_int, [i64, i64, vp, i64]),
    ("xk_memory_coherent_async", c_int, [i64, i64, vp, i64]),
    ("xk_sync", c_int, []),
    ("xk_memory_invalidate", c_int, [i64, i64, vp, i64]),
    ("xk_memory_prefetch_async", c_int, [i64, i64, vp, i64]),
    ("xk_distribute_2dbc_async", c_int, [i64, i64, vp, i64, c_int, c_int, i64, i64]),
    ("xk_get_stats", c_int, [ctypes.POINTER(Stats)]),
    ("xk_reset_stats", c_int, []),
    ("xk_set_kernel_timing", c_int, [c_int]),
    ("xk_get_topology", c_int, [ctypes.POINTER(Topo)]),
    ("xk_probe_host_links", c_int, [i64]),
    ("xk_trace", c_int, [ctypes.c_char_p]),
    ("xk_plan_session_create", c_int, [ctypes.POINTER(Topo), ctypes.POINTER(Flags), ctypes.POINTER(vp)]),
    ("xk_plan_session_call", c_int, [vp, ctypes.POINTER(Call), ctypes.POINTER(PlanRec), i64,
                                     ctypes.POINTER(i64)]),
    ("xk_plan_session_destroy", None, [vp]),
    ("xk_session_selftest", c_int, [ctypes.c_char_p, c_int, c_int, c_int, c_int, c_double,
                                    ctypes.POINTER(c_int)]),
    ("xk_plan_dump", c_int, [ctypes.POINTER(Call), ctypes.POINTER(Topo), ctypes.POINTER(Flags),
                             ctypes.POINTER(PlanRec), i64, ctypes.POINTER(i64)]),
    ("xk_dgemm_tile_device", c_int, [c_char, c_char, i64, i64, i64, _D, vp, i64, vp, i64, _D, vp,
                                     i64, vp]),
]
SYMBOLS = [s[0] for s in _SIGS]


def lib():
    """Load libxk.so (building it in-tree first if the sources are newer)."""
    global _LIB
    if _LIB is None:
        if not os.path.exists(LIB_PATH):
            try:
                from tools.build_native import build_xk
            except ImportError as e:  # pragma: no cover
                raise RuntimeError("libxk.so missing and the build helper is unavailable") from e
            build_xk()
        L = ctypes.CDLL(LIB_PATH)
        for name, res, args in _SIGS:
            f = getattr(L, name, None)
            if f is None:  # reported by tests/test_abi.py (every declared symbol must exist)
                continue
            f.restype = res
            f.argtypes = args
        _LIB = L
    return _LIB
