/*
 * xk.h -- C ABI of the B200-native XKBlas-style multi-GPU level-3 BLAS (libxk.so).
 *
 * The method (Gautier & Lima, PAW-ATM/SC21, /root/reference/PAPER.md):
 *   - LAPACK-layout (column-major) BLAS-3 split into tile tasks on sub-matrix views
 *     (§III, §III-A "memory view" / compact device tile),
 *   - owner-computes mapping of tasks, here a static 2D block-cyclic P x Q
 *     grid,
 *   - a per-tile coherence directory of valid copies on host and GPUs,
 *   - source selection for every input tile by two heuristics:
 *       (i)  topology-aware: among GPUs holding a valid copy, prefer the best link
 *            toward the destination (§III-B),
 *       (ii) optimistic forwarding: when no GPU holds a valid copy, take the best GPU
 *            whose copy is still in flight instead of the host (§III-C),
 *   - lazy host coherence: results stay on the GPUs until the user asks for them
 *     (xkblas_memory_coherent_async),
 *   - asynchronous calls that compose through the cache.
 *
 * Conventions:
 *   - All matrices are column-major host arrays owned by the caller; dimensions and
 *     leading dimensions are int64_t.  Char arguments are case-insensitive; 'C' == 'T'.
 *   - Return value: 0 on success; -i when argument i is invalid (numbered like the
 *     reference BLAS XERBLA, in argument order); a positive XK_ERR_* on runtime failure.
 *     The library never aborts; xk_last_error() returns a message for the last failure.
 *   - BLAS "not referenced" rules hold: beta == 0 -> C is not read (and not copied to a
 *     GPU); alpha == 0 -> A, B not read; quick return when m == 0, n == 0 or
 *     ((alpha == 0 || k == 0) && beta == 1); rows beyond m in ld-padded storage are
 *     never written.
 *   - Synchronous routines = async + coherence of the output + wait + invalidation of
 *     the device copies of their operands (drop-in semantics).
 *     Asynchronous routines return as soon as the work is issued; inputs must stay
 *     unmodified and outputs unread until xk_memory_coherent_sync() on that view (or
 *     xk_sync() followed by coherence).  Device copies stay in the library cache, so a
 *     following async call reads them from the GPUs (composition).
 *   - Calls must come from one host thread at a time (an internal mutex serialises).
 *   - Host memory should be registered with xk_register() before timed calls
 *     (page-locking is excluded from the paper's timings); unregistered
 *     memory is registered internally on first use and counted in the stats.
 */
#ifndef XK_H
#define XK_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* ------------------------------------------------------------------ error codes */
#define XK_OK 0
#define XK_ERR_NOT_INITIALIZED 1 /* xk_init() not called */
#define XK_ERR_CUDA 2            /* a CUDA runtime/driver call failed; see xk_last_error() */
#define XK_ERR_OOM 3             /* device tile cache full (no eviction: SURVEY A13) */
#define XK_ERR_CONFIG 4          /* invalid xk_config_t / topology / flags */
#define XK_ERR_CAPACITY 5        /* caller-provided output array too small */
#define XK_ERR_UNSUPPORTED 6     /* view overlaps a cached matrix with another tiling */
#define XK_ERR_NO_DEVICE 7       /* no CUDA device visible */
#define XK_ERR_INTERNAL 8

#define XK_MAX_GPUS 16
#define XK_HOST (-1) /* node id of host memory in plan records */

/* topology-aware source selection modes (a5) */
#define XK_TOPO_RANKED 0   /* paper's heuristic: best link class first */
#define XK_TOPO_UNRANKED 1 /* paper's "no topo" ablation: lowest-index holder */
#define XK_TOPO_HOME 2     /* link-oblivious ablation: host first, then GPUs */

/* ------------------------------------------------------------------ configuration */
typedef struct xk_config {
    int ngpus;            /* logical GPUs G (0 = every visible device, max XK_MAX_GPUS) */
    int phys[XK_MAX_GPUS];/* logical -> physical device map; used when map_devices != 0,
                             else logical g -> physical g mod device_count.  Several
                             logical GPUs on one physical device = "logical-device mode"
                             (peer copies become device-to-device copies). */
    int map_devices;
    int grid_p, grid_q;   /* owner grid P x Q (0,0 = near-square P >= Q: 1x1,2x1,2x2,4x2) */
    int64_t tile;         /* tile size T (0 = 2048) */
    int topo;             /* XK_TOPO_* (default RANKED) */
    int optimistic;       /* optimistic forwarding on (1, default) / off (0) */
    int window;           /* planner prefetch window W in tasks (0 = 4; Q17) */
    int kstreams;         /* kernel streams per GPU (0 = 2); plus 1 H2D, 1 D2H, 1 P2P-in */
    int probe;            /* 1 = time the (G+1)^2 link matrix at init (a1); 0 = defaults */
    int64_t task_rate_mflops; /* planner's tile-task rate (0 = measured at init on one grouped launch of 8 tile tasks; 35e6 without the probe) */
    /* ---- rank mode: one process per GPU.  `world` processes each call
     * xk_init with their own `rank` and the same `session`; process r drives logical GPU r
     * only.  Every process runs the same deterministic planner on the same calls, so all
     * hold the identical plan; each executes the records of its own GPU (H2D/P2P/task into
     * it, D2H out of it), pulls peer tiles through CUDA IPC mappings of the peers' tile
     * arenas and orders cross-process dependencies with per-record completion flags in the
     * shared session file (stream memory operations, no host round trip).  In rank mode
     * EVERY later API call is collective: all ranks make the same calls with the same
     * arguments, host matrices live in memory shared by the processes (the same file
     * mapping; addresses may differ per process), and xk_last_error() is per process.
     * A failing rank marks the session so the others return XK_ERR_CUDA at their next
     * synchronisation point instead of waiting forever. */
    int rank;             /* this process's logical GPU, 0 <= rank < world */
    int world;            /* number of processes = logical GPUs (0 or 1 = single-process mode) */
    int64_t arena_bytes;  /* rank mode: device tile arena per GPU, the same on every rank
                             (0 = 85% of the smallest free memory / ranks sharing a device) */
    char session[128];    /* rank mode: path of the shared control file, unique per session
                             (e.g. "/dev/shm/xk_<token>"); rank 0 creates it, rank 0 removes
                             it at xk_finalize */
    int64_t mem_bytes;    /* tile-cache capacity per logical GPU the planner plans against
                             (xk_flags_t.mem_bytes); 0 = derived at init: 90% of the device's
                             free memory / logical GPUs sharing it (rank mode: the arena) */
} xk_config_t;

/* Fill *cfg with defaults, then apply the environment (XK_NGPUS, XK_TILE,
 * XK_TOPO=ranked|unranked|home, XK_OPTIMISTIC=0|1, XK_WINDOW, XK_KSTREAMS, XK_PROBE, XK_TASK_RATE). */
void xk_config_default(xk_config_t *cfg);

/* ------------------------------------------------------------------ lifecycle */
/* xk_init: set up the GPUs, streams and the planner; with cfg->probe, time the (G+1)^2 link
 * matrix "during the library initialization" (SecIII-B).  Errors: XK_ERR_CONFIG
 * (bad grid / topo / ngpus), XK_ERR_NO_DEVICE, XK_ERR_CUDA, XK_ERR_OOM (rank-mode arena). */
int xk_init(const xk_config_t *cfg); /* NULL -> xk_config_default(); probes topology */
int xk_finalize(void);               /* waits, frees every device copy, destroys streams */
int xk_register(void *p, size_t bytes);   /* cudaHostRegister(Portable) once, all GPUs */
int xk_unregister(void *p);
const char *xk_last_error(void);

/* ------------------------------------------------------------------ BLAS-3 (FP64) */
/* The six routines of the paper's report (SecI, Fig. 5, SecIV-D
 * P:834-835), each the operation the BLAS standard defines (ref. [1], P:66-67 and
 * P:1187-1188; argument order and XERBLA numbering as in the reference BLAS), computed by
 * PLASMA-style tiled algorithms on LAPACK-layout views (SecIII).  The synchronous
 * form returns with the output coherent on the host; the _async form is the paper's
 * xkblas_*_async (SecIV-F): it returns once the work is issued and composes with
 * later calls through the tile cache.  Only the arguments' referenced parts are read
 * (BLAS "not referenced" rules, header comment above).  Errors: -i for argument i, or a
 * positive XK_ERR_*.
 *
 * DGEMM (Fig. 3, Table II):
 * C <- alpha*op(A)*op(B) + beta*C ; op(X) = X ('N') or X^T ('T'/'C').
 * A is m x k ('N') or k x m ('T') with lda >= max(1, rows); B is k x n or n x k; C m x n.
 * Errors: -1 transA, -2 transB, -3 m, -4 n, -5 k, -8 lda, -10 ldb, -13 ldc. */
int xk_dgemm(char transA, char transB, int64_t m, int64_t n, int64_t k, double alpha,
             const double *A, int64_t lda, const double *B, int64_t ldb,
             double beta, double *C, int64_t ldc);
int xk_dgemm_async(char transA, char transB, int64_t m, int64_t n, int64_t k, double alpha,
                   const double *A, int64_t lda, const double *B, int64_t ldb,
                   double beta, double *C, int64_t ldc);

/* DSYRK (SecIV-D):
 * C <- alpha*op(A)*op(A)^T + beta*C on the uplo triangle only (op(A) n x k).
 * Errors: -1 uplo, -2 trans, -3 n, -4 k, -7 lda, -10 ldc. */
int xk_dsyrk(char uplo, char trans, int64_t n, int64_t k, double alpha,
             const double *A, int64_t lda, double beta, double *C, int64_t ldc);
int xk_dsyrk_async(char uplo, char trans, int64_t n, int64_t k, double alpha,
                   const double *A, int64_t lda, double beta, double *C, int64_t ldc);

/* DSYR2K (Fig. 3):
 * C <- alpha*op(A)*op(B)^T + alpha*op(B)*op(A)^T + beta*C, uplo triangle only.
 * Errors: -1 uplo, -2 trans, -3 n, -4 k, -7 lda, -9 ldb, -12 ldc. */
int xk_dsyr2k(char uplo, char trans, int64_t n, int64_t k, double alpha,
              const double *A, int64_t lda, const double *B, int64_t ldb,
              double beta, double *C, int64_t ldc);
int xk_dsyr2k_async(char uplo, char trans, int64_t n, int64_t k, double alpha,
                    const double *A, int64_t lda, const double *B, int64_t ldb,
                    double beta, double *C, int64_t ldc);

/* DSYMM: C <- alpha*sym(A)*B + beta*C ('L') or alpha*B*sym(A) + beta*C ('R'); only the uplo
 * triangle of A is read.  Errors: -1 side, -2 uplo, -3 m, -4 n, -7 lda, -9 ldb, -12 ldc. */
int xk_dsymm(char side, char uplo, int64_t m, int64_t n, double alpha,
             const double *A, int64_t lda, const double *B, int64_t ldb,
             double beta, double *C, int64_t ldc);
int xk_dsymm_async(char side, char uplo, int64_t m, int64_t n, double alpha,
                   const double *A, int64_t lda, const double *B, int64_t ldb,
                   double beta, double *C, int64_t ldc);

/* DTRMM: B <- alpha*op(A)*B ('L') or alpha*B*op(A) ('R'), A triangular
 * (uplo), diag 'U' = unit.
 * Errors: -1 side, -2 uplo, -3 transA, -4 diag, -5 m, -6 n, -9 lda, -11 ldb. */
int xk_dtrmm(char side, char uplo, char transA, char diag, int64_t m, int64_t n,
             double alpha, const double *A, int64_t lda, double *B, int64_t ldb);
int xk_dtrmm_async(char side, char uplo, char transA, char diag, int64_t m, int64_t n,
                   double alpha, const double *A, int64_t lda, double *B, int64_t ldb);

/* DTRSM (Fig. 3, Table II; composed with DGEMM in SecIV-F):
 * solve op(A)*X = alpha*B ('L') or X*op(A) = alpha*B ('R'); B <- X.  Same errors as TRMM. */
int xk_dtrsm(char side, char uplo, char transA, char diag, int64_t m, int64_t n,
             double alpha, const double *A, int64_t lda, double *B, int64_t ldb);
int xk_dtrsm_async(char side, char uplo, char transA, char diag, int64_t m, int64_t n,
                   double alpha, const double *A, int64_t lda, double *B, int64_t ldb);

/* ------------------------------------------------------------------ coherence / sync */
/* Make the host view (m x n at A, leading dimension lda) coherent: copy back every
 * cached tile intersection whose host copy is stale (only the intersection is written),
 * after its last writer.  _sync blocks until done. */
int xk_memory_coherent_sync(int64_t m, int64_t n, double *A, int64_t lda);
int xk_memory_coherent_async(int64_t m, int64_t n, double *A, int64_t lda);
/* Wait for all issued work.  Does NOT make host copies coherent (lazy). */
int xk_sync(void);
/* Drop the device copies of the tiles of a view (waits for pending work first); from then
 * on the host array is the valid copy of those tiles (whatever the caller holds there is
 * read by the next call).  Stale host tiles are NOT written back: call
 * xk_memory_coherent_sync first to keep results that live only on the GPUs. */
int xk_memory_invalidate(int64_t m, int64_t n, const double *A, int64_t lda);
/* Load the tiles of a host view onto their owner GPUs now (data-on-device runs). */
int xk_memory_prefetch_async(int64_t m, int64_t n, const double *A, int64_t lda);
/* The paper's xkblas_distribute_2Dblock_cyclic_async (SecIV-C, "data on device"):
 * distribute the tiles of a host view over a P x Q grid of GPUs in 2D block-cyclic blocks
 * of mb x nb tiles (ScaLAPACK layout; the paper's runs use the (4,2) grid and (1,1) blocks):
 * tile (bi, bj) goes to GPU ((bi / mb) mod P) * Q + ((bj / nb) mod Q).  Asynchronous; the
 * tiles stay in the cache as valid copies, so later calls read them from the GPUs (a tile
 * whose task runs on another GPU is forwarded over the peer links, never re-read from the
 * host).  Tiles are the library's T x T tiles of the view anchored at A (as every call).
 * Errors: -1 m < 0, -2 n < 0, -4 lda < max(1, m), -5 P < 1, -6 Q < 1 or P*Q > ngpus,
 * -7 mb < 1, -8 nb < 1; XK_ERR_* as the BLAS calls. */
int xk_distribute_2dbc_async(int64_t m, int64_t n, const double *A, int64_t lda, int P, int Q,
                             int64_t mb, int64_t nb);

/* ------------------------------------------------------------------ observability */
typedef struct xk_stats {
    int ngpus;
    int64_t h2d_bytes[XK_MAX_GPUS];  /* host -> GPU g */
    int64_t d2h_bytes[XK_MAX_GPUS];  /* GPU g -> host */
    int64_t p2p_in_bytes[XK_MAX_GPUS];  /* peer -> GPU g */
    int64_t p2p_out_bytes[XK_MAX_GPUS]; /* GPU g -> peer */
    int64_t tasks[XK_MAX_GPUS];
    int64_t flops[XK_MAX_GPUS];
    int64_t forwards_inflight;       /* P2P copies sourced from an in-flight copy (A2) */
    int64_t forwards_valid;          /* P2P copies sourced from a valid copy (A1) */
    int64_t kernel_launches;         /* tile-kernel launches (one grouped launch per batch) */
    int64_t host_registrations;      /* unregistered host ranges registered internally */
    double kernel_ms_total;          /* summed tile-kernel launch time (when timing on) */
    int64_t kernel_timed_launches;   /* launches included in kernel_ms_total */
    int64_t kernel_timed_flops;      /* algorithmic flops of those launches (2*m*n*k per task) */
    int64_t link_bytes[(XK_MAX_GPUS + 1) * (XK_MAX_GPUS + 1)]; /* bytes per link, row = source,
                                        column = destination, stride ngpus+1, index ngpus = host */
    double trace_ms[4];              /* with tracing on: summed op time by kind
                                        [H2D, P2P, kernel, D2H] (paper Fig. 6 breakdown) */
    int64_t plan_records;            /* plan records produced (every GPU's) */
    int64_t plan_records_local;      /* ... of which executed by this process (rank mode: its GPU) */
    double host_issue_ms;            /* host wall time planning + issuing them (the per-call
                                        "creation and scheduling of dynamic tasks") */
    int64_t device_allocs;           /* new device tile buffers (not served by the free lists) */
    double device_alloc_ms;          /* host wall time spent obtaining them */
} xk_stats_t;
/* Counters since xk_init / the last xk_reset_stats: the per-link byte counts are the paper's
 * transfer breakdown (SecIV-E) and the evidence that the heuristics cut PCIe bytes
 * (P:181-183).  Errors: XK_ERR_NOT_INITIALIZED, XK_ERR_CONFIG (out == NULL). */
int xk_get_stats(xk_stats_t *out);
int xk_reset_stats(void);
/* 1 = time every tile-kernel launch with CUDA events (bench roofline); grouped launches are
 * then serialised on one kernel stream per GPU so each duration is its own.  0 = off. */
int xk_set_kernel_timing(int on);
/* Timeline tracing (paper: nvprof Gantt charts).  path != NULL: record
 * every copy and kernel launch with CUDA events from now on; path == NULL: stop and write the
 * Chrome-trace JSON (chrome://tracing / Perfetto) of everything recorded since to the path
 * given at start.  Waits for pending work.  XK_TRACE=path in the environment traces the whole
 * session and writes it at xk_finalize. */
int xk_trace(const char *path);

/* (G+1) x (G+1) link matrix in MB/s, row = source, column = destination, index G =
 * host; diagonal = device-local copy bandwidth.  Filled by xk_init (probe or defaults). */
typedef struct xk_topo {
    int ngpus;
    int64_t bw_MBps[(XK_MAX_GPUS + 1) * (XK_MAX_GPUS + 1)]; /* row-major, stride ngpus+1 */
    int perf_rank[XK_MAX_GPUS * XK_MAX_GPUS]; /* cuDeviceGetP2PAttribute PERFORMANCE_RANK, logged only (Q6) */
    int64_t task_rate_mflops;                 /* tile-task FP64 rate used by the planner */
    /* Host links with every GPU copying AT ONCE (xk_probe_host_links; 0 until it ran):
     * aggregate MB/s over all G GPUs for [0] H2D only, [1] D2H only, [2] full duplex (H2D and
     * D2H together, total bytes both ways / time).  Host DRAM and the root complexes are shared,
     * so these bound the PCIe term of the roofline (SecII-B, SecIV-D)
     * rather than G x the per-GPU entries of bw_MBps. */
    int64_t host_all_MBps[3];
    int64_t host_probe_bytes;                 /* bytes per GPU per direction of that probe */
} xk_topo_t;
int xk_get_topology(xk_topo_t *out);
/* Time the host links with all GPUs copying at once (SURVEY.md §8(d) "BW_h2d(G), BW_d2h(G),
 * full duplex"): every GPU copies bytes_per_gpu between its own pinned host region (distinct
 * per GPU, allocated here and freed before return) and device memory, H2D only, D2H only,
 * then both directions together; best of 2 after a warm-up, wall clock around the whole
 * group (rank mode: barrier-started, each rank's time in the session file, aggregate over
 * the slowest).  Results in xk_get_topology().host_all_MBps.  Untimed set-up, like the
 * init probe.  Waits for pending work first.  Rank mode: collective.  Returns
 * XK_ERR_OOM when neither the pinned host nor the device buffers can be allocated (the size
 * is halved down to 64 MiB before giving up), XK_ERR_CUDA on a copy failure. */
int xk_probe_host_links(int64_t bytes_per_gpu);

/* ------------------------------------------------------------------ planner (no GPU) */
/* The planner is a pure function of (call, topology, flags, directory state): tests run
 * it with G virtual GPUs and injected link matrices and compare it bit-exactly with the
 * independent CPU model tests/planmodel.py (SURVEY.md §8(c) "Plan oracle"). */
#define XK_REC_H2D 0
#define XK_REC_P2P 1
#define XK_REC_TASK 2
#define XK_REC_D2H 3

#define XK_SRC_NONE 0
#define XK_SRC_VALID 1    /* source copy valid at request time */
#define XK_SRC_INFLIGHT 2 /* source copy still arriving: optimistic forwarding */
#define XK_SRC_HOST 3

#define XK_ROUTINE_DGEMM 0
#define XK_ROUTINE_DSYRK 1
#define XK_ROUTINE_DSYR2K 2
#define XK_ROUTINE_DSYMM 3
#define XK_ROUTINE_DTRMM 4
#define XK_ROUTINE_DTRSM 5
#define XK_ROUTINE_COHERENT 100
#define XK_ROUTINE_SYNC 101
#define XK_ROUTINE_INVALIDATE 102
#define XK_ROUTINE_PREFETCH 103
#define XK_ROUTINE_DISTRIBUTE 104 /* view (m, n, C, ldc); grid_p x grid_q GPUs, blocks mb x nb tiles */

typedef struct xk_flags {
    int topo, optimistic, window;
    int grid_p, grid_q;
    int64_t tile;
    int64_t mem_bytes; /* device tile-cache capacity per GPU the plan must fit: a per-call
                          shadow (beta deferral Q12'', TRMM R15) is used only when every GPU's
                          resident tiles plus the call's tiles fit; 0 = unlimited */
} xk_flags_t;

/* Tile-task operations (TASK records, field op). */
#define XK_OP_GEMM 0      /* C = alpha*op(A)*op(B) + beta*C */
#define XK_OP_SCALE 1     /* C = beta*C (alpha == 0 or k == 0) */
#define XK_OP_GEMM_TRI 2  /* GEMM on a diagonal tile writing only its uplo triangle (SYRK/SYR2K) */
#define XK_OP_SYMM_DIAG 3 /* C = alpha*sym(A_ii)*B + beta*C or alpha*B*sym(A_jj) + beta*C */
#define XK_OP_TRMM_DIAG 4 /* B = alpha*op(A_kk)*B or alpha*B*op(A_kk), in place */
#define XK_OP_TRSM_DIAG 5 /* B = alpha*op(A_kk)^-1*B or alpha*B*op(A_kk)^-1, in place */

/* One API call as seen by the planner.  Matrix addresses are identities only (never
 * dereferenced by the planner).  The OUTPUT matrix is always (C, ldc): for TRMM/TRSM the
 * BLAS "B" (m x n, updated in place) is passed as C.  transA doubles as SYRK/SYR2K's
 * trans.  For XK_ROUTINE_COHERENT / INVALIDATE / PREFETCH the view is (m, n, C, ldc). */
typedef struct xk_call {
    int routine;
    char transA, transB, uplo, side, diag;
    int64_t m, n, k;
    double alpha, beta;
    uint64_t A, lda, B, ldb, C, ldc;
    int sync; /* 1 = synchronous routine: D2H of the output after its last writer */
    int grid_p, grid_q; /* XK_ROUTINE_DISTRIBUTE: GPU grid (P*Q <= G) */
    int64_t mb, nb;     /* XK_ROUTINE_DISTRIBUTE: block-cyclic block size in tiles */
} xk_call_t;

typedef struct xk_plan_rec {
    int64_t seq;       /* emission order, session-global */
    int32_t kind;      /* XK_REC_* */
    int32_t operand;   /* 0 = A, 1 = B, 2 = C of the call (coherent/prefetch: 2) */
    int64_t bi, bj;    /* tile coordinates in the STORED matrix (T x T grid at element 0,0) */
    int64_t tk;        /* TASK: k-tile / step index of the tiled algorithm (-1: scale-only) */
    int64_t version;   /* tile version the record moves / produces */
    int32_t dst, src;  /* node ids: GPU 0..G-1 or XK_HOST */
    int32_t src_state; /* XK_SRC_* (copies); XK_SRC_NONE for tasks */
    int32_t depth;     /* forwarding depth of the destination copy (host = 0, H2D = 1) */
    int32_t op;        /* TASK: XK_OP_*; copies: -1 */
    int32_t reserved;
    int64_t t_start, t_end; /* virtual time, integer ns */
    int64_t work;      /* bytes (copies) or flops (tasks) */
    int64_t dep[4];    /* seq of records this one waits on, one per task input in input order
                          (copies: dep[0] = producer of the source copy); -1 = none */
} xk_plan_rec_t;

/* Planner sessions: the directory, clocks and link occupancy persist across calls
 * (composition), exactly as inside the library. */
typedef struct xk_plan_session xk_plan_session_t;
int xk_plan_session_create(const xk_topo_t *topo, const xk_flags_t *flags, xk_plan_session_t **out);
int xk_plan_session_call(xk_plan_session_t *s, const xk_call_t *call,
                         xk_plan_rec_t *out, int64_t cap, int64_t *n_out);
void xk_plan_session_destroy(xk_plan_session_t *s);
/* One-shot: fresh session, one call. */
int xk_plan_dump(const xk_call_t *call, const xk_topo_t *topo, const xk_flags_t *flags,
                 xk_plan_rec_t *out, int64_t cap, int64_t *n_out);

/* ------------------------------------------------------------------ rank-mode session */
/* The host side of rank mode's synchronisation, without CUDA (for CPU tests and tools):
 * joins the session file `path` as `rank` of `world` (rank 0 creates it and removes it at
 * the end), passes `rounds` barriers, and writes into flags_out[r] (r < rounds) the number of
 * ranks that had arrived at round r when this rank left it (every rank must see `world`).
 * With abort_at >= 0 this rank marks the session aborted instead of arriving at round
 * abort_at; the others then fail.  Returns 0, XK_ERR_CONFIG (cannot create/join), or
 * XK_ERR_CUDA (a barrier failed: peer aborted or timeout_s elapsed). */
int xk_session_selftest(const char *path, int rank, int world, int rounds, int abort_at,
                        double timeout_s, int *flags_out);

/* ------------------------------------------------------------------ kernel-level entry */
/* One tile task on device memory, for kernel parity tests and the roofline bench:
 * D = alpha*op(A)*op(B) + beta*C on compact column-major tiles (ld = rows),
 * D may alias C.  Pointers are DEVICE pointers on the current device; stream is a
 * cudaStream_t (NULL = legacy default stream).  beta == 0: C not read. */
int xk_dgemm_tile_device(char transA, char transB, int64_t m, int64_t n, int64_t k,
                         double alpha, const double *A, int64_t lda, const double *B,
                         int64_t ldb, double beta, double *C, int64_t ldc, void *stream);

#ifdef __cplusplus
}
#endif
#endif /* XK_H */
