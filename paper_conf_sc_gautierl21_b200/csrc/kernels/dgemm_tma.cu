// dgemm_tma.cu -- FP64 tile GEMM for sm_100a with TMA loads and an mbarrier pipeline.
//
//   D = alpha * op(A) * op(B) + beta * C on column-major device tiles (same operation and
//   batching as dgemm_tile.cu).
//
// Why a second kernel: the cp.async kernel spends ~14% of its issue slots/time on per-thread
// address math, the per-k-block __syncthreads and cp.async waits (profiles/r01_*).  Here one
// thread streams whole operand boxes with the Tensor Memory Accelerator
// (cp.async.bulk.tensor.2d, zero-filled out of bounds so ragged tiles need no predication),
// each stage completes on a transaction-count mbarrier, and the last warp to finish reading a
// stage refills it (a shared-memory counter per stage): no CTA-wide barrier, no producer warp.
//
// Shared-memory layout: TMA 128-byte swizzle (16-byte chunk index XOR row % 8).  mn-contiguous
// operands are loaded as 16(mn) x 16(k) boxes (rows = k), k-contiguous operands as one
// 16(k) x BMN box (rows = mn).  The m8n8k4 fragments read k in a permuted order
// sigma(s, q) = X[s] ^ Q[q], X = {0,1,4,5}, Q = {0,3,12,15}: it partitions the 16 k of a
// stage into 4 steps and makes every 8-byte fragment read conflict-free for BOTH swizzled
// layouts.  A and B use the same permutation, so each step still sums over
// matching k; only the (legal) summation order changes.
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdlib.h>

#include "kernels/kernels.h"

namespace xk {
namespace {

constexpr int BK = 16;
#ifndef XK_CPF
#define XK_CPF 0  // extra k-blocks of lead for the epilogue's C prefetch (-1 = off)
#endif
constexpr int BM = 64, BN = 128;   // CTA tile
#ifndef XK_WN
#define XK_WN 32
#endif
constexpr int WM = 32, WN = XK_WN;  // warp tile (32 x 32: 8 warps; 32 x 64: 4 warps)
constexpr int NWM = BM / WM, NWN = BN / WN, NWARPS = NWM * NWN;
constexpr int NTHREADS = NWARPS * 32;
constexpr int STAGES = 4;
#ifndef XK_EPI_ROWS
#define XK_EPI_ROWS 1
#endif
constexpr int EPI_ROWS = XK_EPI_ROWS;  // row fragments per epilogue load batch
#ifndef XK_FB1
#define XK_FB1 1  // single-buffered B fragments (0: double-buffered, the round-2 A/B baseline)
#endif
static_assert((WM / 8) % EPI_ROWS == 0, "epilogue chunking");
constexpr int A_BYTES = BM * BK * 8, B_BYTES = BN * BK * 8, STAGE_BYTES = A_BYTES + B_BYTES;

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;\n" ::"r"(bar), "r"(count));
}
__device__ __forceinline__ void mbar_expect_tx(uint32_t bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
    asm volatile(
        "{\n"
        ".reg .pred p;\n"
        "WAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
        "@!p bra WAIT_%=;\n"
        "}\n" ::"r"(bar),
        "r"(parity)
        : "memory");
}
__device__ __forceinline__ void tma_load_2d(uint32_t dst, const CUtensorMap *map, int c0, int c1,
                                            uint32_t bar) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];\n" ::"r"(dst),
        "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(c1), "r"(bar)
        : "memory");
}
__device__ __forceinline__ void dmma(double (&c)[2], double a, double b) {
    asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
                 : "+d"(c[0]), "+d"(c[1])
                 : "d"(a), "d"(b));
}

// Byte offset of fragment element (mn = base8 + fr, k = x ^ qk) inside an operand region of
// one stage, split as lane_part ^ const_part: the two parts occupy disjoint bit ranges except
// where the swizzle XORs them, so each fragment address is one XOR with a compile-time
// constant (base8 = warp offset + 8*i is a multiple of 8; x in {0,1,4,5}; qk in {0,3,12,15}).
//   mn-contiguous (16 x 16 boxes, rows = k): off = (mn>>4)*2048 + k*128 + ((((mn&15)>>1) ^ (k&7))<<4) + (mn&1)*8
//   k-contiguous  (rows = mn)            : off = mn*128 + (((k>>1) ^ (mn&7))<<4) + (k&1)*8
template <bool MN_CONTIG>
__device__ __forceinline__ uint32_t lane_part(int fr, int qk) {
    if (MN_CONTIG) return (uint32_t)((qk << 7) | ((((fr >> 1) ^ (qk & 7)) & 7) << 4) | ((fr & 1) << 3));
    return (uint32_t)((fr << 7) | ((((qk >> 1) ^ fr) & 7) << 4) | ((qk & 1) << 3));
}
template <bool MN_CONTIG>
__device__ __forceinline__ uint32_t const_part(int base8, int x) {
    if (MN_CONTIG) return (uint32_t)(((base8 >> 4) << 11) | (x << 7) | (((((base8 & 8) >> 1) ^ x) & 7) << 4));
    return (uint32_t)((base8 << 7) | (((x >> 1) & 7) << 4) | ((x & 1) << 3));
}

__device__ __forceinline__ void tma_load_3d(uint32_t dst, const CUtensorMap *map, int c0, int c1, int c2,
                                            uint32_t bar) {
    asm volatile(
        "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], [%5];\n" ::"r"(dst),
        "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(c1), "r"(c2), "r"(bar)
        : "memory");
}

// One stage of an operand.  mn-contiguous: BMN/16 boxes of 16(mn) x 16(k) -- as ONE 3D box
// (16 mn, 16 k, BMN/16 chunks of 16 mn) when the map is 3D (same shared-memory image: chunk
// q at q * 2048, rows = k, 128-byte swizzle per row), else one 2D box per chunk.
template <bool MN_CONTIG, int BMN, bool D3>
__device__ __forceinline__ void issue_operand(uint32_t dst, const CUtensorMap *map, int mn0, int k0,
                                              uint32_t bar) {
    if (MN_CONTIG) {
        if (D3) {
            tma_load_3d(dst, map, 0, k0, mn0 >> 4, bar);
            return;
        }
#pragma unroll
        for (int q = 0; q < BMN / 16; ++q) tma_load_2d(dst + q * 2048, map, mn0 + 16 * q, k0, bar);
    } else {
        tma_load_2d(dst, map, k0, mn0, bar);
    }
}

template <bool TA, bool TB, bool D3>
__global__ void __launch_bounds__(NTHREADS, 2) dgemm_tma_kernel(const __grid_constant__ TmaBatch batch) {
    constexpr bool A_MN = !TA;  // op(A) M x K: 'N' -> m contiguous
    constexpr bool B_MN = TB;   // op(B) K x N: 'T' -> n contiguous
    int q = 0;
    const int bid = blockIdx.x;
#pragma unroll 1
    while (q + 1 < batch.n && bid >= batch.cta_start[q + 1]) ++q;
    const TmaTask &t = batch.t[q];
    const int local = bid - batch.cta_start[q];
    const int tiles_m = (int)((t.M + BM - 1) / BM);
    // grouped raster: CTAs run GROUP_M m-blocks at a time across all n-blocks, so the CTAs
    // resident together share A and B slabs in L2 instead of streaming all of A per column
    const int tiles_n = (int)((t.N + BN - 1) / BN);
    const int gm = batch.group_m > 0 ? batch.group_m : tiles_m;
    const int per_group = gm * tiles_n;
    const int grp = local / per_group, first = grp * gm;
    const int gsz = min(tiles_m - first, gm);
    const int in_group = local % per_group;
    // snake: odd groups walk the n-blocks backwards, so the first CTAs of a group read the
    // B panel the last CTAs of the previous group left in L2
    const int nblk = (batch.snake && (grp & 1)) ? tiles_n - 1 - in_group / gsz : in_group / gsz;
    const int m0 = (first + in_group % gsz) * BM, n0 = nblk * BN;
    const int64_t M = t.M, N = t.N;
    const int tri = t.tri;
    if ((tri == 1 && m0 + BM - 1 < n0) || (tri == 2 && n0 + BN - 1 < m0)) return;
    const int KB = (int)((t.K + BK - 1) / BK);

    extern __shared__ __align__(1024) unsigned char smem_raw[];
    // 1024-byte alignment of every stage (required by the 128-byte swizzle)
    const uint32_t sbase = (smem_u32(smem_raw) + 1023u) & ~1023u;
    unsigned char *sgen = smem_raw + (sbase - smem_u32(smem_raw));
    const uint32_t bars = sbase + STAGES * STAGE_BYTES;  // full[STAGES] mbarriers
    auto full = [&](int s) { return bars + 8u * s; };
    // per-stage count of warps done reading it; the last one refills the stage
    int *done_cnt = reinterpret_cast<int *>(sgen + STAGES * STAGE_BYTES + 8 * STAGES);

    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    if (tid == 0) {
        for (int s = 0; s < STAGES; ++s) {
            mbar_init(full(s), 1);
            done_cnt[s] = 0;
        }
        asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
        asm volatile("prefetch.tensormap [%0];\n" ::"l"(reinterpret_cast<uint64_t>(&t.mapA)) : "memory");
        asm volatile("prefetch.tensormap [%0];\n" ::"l"(reinterpret_cast<uint64_t>(&t.mapB)) : "memory");
    }
    __syncthreads();
    auto produce = [&](int kb) {
        const int s = kb % STAGES;
        const uint32_t dst = sbase + s * STAGE_BYTES;
        mbar_expect_tx(full(s), STAGE_BYTES);
        issue_operand<A_MN, BM, D3>(dst, &t.mapA, m0, kb * BK, full(s));
        issue_operand<B_MN, BN, D3>(dst + A_BYTES, &t.mapB, n0, kb * BK, full(s));
    };
    if (tid == 0)
        for (int kb = 0; kb < STAGES && kb < KB; ++kb) produce(kb);

    const int wm = (warp % NWM) * WM, wn = (warp / NWM) * WN;
    const int fr = lane >> 2, fc = lane & 3;
    constexpr int MF = WM / 8, NF = WN / 8;
    // permuted k of this lane for step s: X[s] ^ Q[fc], X = {0,1,4,5}, Q = {0,3,12,15}
    const int qk = (fc == 0) ? 0 : (fc == 1) ? 3 : (fc == 2) ? 12 : 15;
    const uint32_t laneA = lane_part<A_MN>(fr, qk), laneB = lane_part<B_MN>(fr, qk);

    double acc[MF][NF][2];
#pragma unroll
    for (int i = 0; i < MF; ++i)
#pragma unroll
        for (int j = 0; j < NF; ++j) acc[i][j][0] = acc[i][j][1] = 0.0;
#if XK_FB1
    // B fragments single-buffered (loaded right before their DMMAs; the other warps of the
    // scheduler cover the shared-load latency), A fragments double-buffered
    double fa[2][MF], fb[1][NF];
    auto load_b = [&](int stage, int s) {
        const unsigned char *sb = sgen + stage * STAGE_BYTES + A_BYTES;
        const int x = (s & 1) | ((s & 2) << 1);
#pragma unroll
        for (int j = 0; j < NF; ++j)
            fb[0][j] = *reinterpret_cast<const double *>(sb + (laneB ^ const_part<B_MN>(wn + j * 8, x)));
    };
    auto load_frags = [&](int buf, int stage, int s) {
        const unsigned char *sa = sgen + stage * STAGE_BYTES;
        const int x = (s & 1) | ((s & 2) << 1);
#pragma unroll
        for (int i = 0; i < MF; ++i)
            fa[buf][i] = *reinterpret_cast<const double *>(sa + (laneA ^ const_part<A_MN>(wm + i * 8, x)));
    };
#else
    double fa[2][MF], fb[2][NF];
    auto load_frags = [&](int buf, int stage, int s) {
        const unsigned char *sa = sgen + stage * STAGE_BYTES;
        const unsigned char *sb = sa + A_BYTES;
        const int x = (s & 1) | ((s & 2) << 1);
#pragma unroll
        for (int i = 0; i < MF; ++i)
            fa[buf][i] = *reinterpret_cast<const double *>(sa + (laneA ^ const_part<A_MN>(wm + i * 8, x)));
#pragma unroll
        for (int j = 0; j < NF; ++j)
            fb[buf][j] = *reinterpret_cast<const double *>(sb + (laneB ^ const_part<B_MN>(wn + j * 8, x)));
    };
#endif

    mbar_wait(full(0), 0);
    load_frags(0, 0, 0);
#pragma unroll 1
    for (int kb = 0; kb < KB; ++kb) {
        const int st = kb % STAGES;
        if (kb == KB - 2 - XK_CPF) {
            // the epilogue's C (and deferred-beta C2) reads are cold DRAM reads: pull this
            // warp's 32 x 32 block into L2 while the last k-blocks still run (one column of
            // 256 bytes per lane)
            const int64_t row = m0 + wm;
#pragma unroll
            for (int cg = 0; cg < WN / 32; ++cg) {
                const int64_t col = n0 + wn + cg * 32 + lane;
                if (col < t.N && row < t.M) {
                    if (t.beta != 0.0) {
                        const double *pc = t.C + row + col * t.ldc;
                        asm volatile("prefetch.global.L2 [%0];" ::"l"(pc));
                        if (row + 16 < t.M) asm volatile("prefetch.global.L2 [%0];" ::"l"(pc + 16));
                    }
                    if (t.beta2 != 0.0) {
                        const double *p2 = t.C2 + row + col * t.ldc2;
                        asm volatile("prefetch.global.L2 [%0];" ::"l"(p2));
                        if (row + 16 < t.M) asm volatile("prefetch.global.L2 [%0];" ::"l"(p2 + 16));
                    }
                }
            }
        }
        // this warp's last read of stage st is done; the last warp to get here refills the
        // stage with block kb + STAGES (no CTA-wide barrier, no dedicated producer warp).
        // The count is an acq_rel RMW: each warp's increment releases its reads of the stage
        // (ordered before lane 0's RMW by __syncwarp), and the last increment acquires all of
        // them (one release sequence), so the refill's async-proxy TMA write (after
        // fence.proxy.async) follows every read.
        auto release_stage = [&]() {
            __syncwarp();
            if (lane == 0) {
                uint32_t old;
                asm volatile("atom.acq_rel.cta.shared::cta.add.u32 %0, [%1], 1;\n"
                             : "=r"(old) : "r"(smem_u32(&done_cnt[st])) : "memory");
                if (old == NWARPS - 1) {
                    atomicExch(&done_cnt[st], 0);
                    if (kb + STAGES < KB) {
                        asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory");
                        produce(kb + STAGES);
                    }
                }
            }
        };
#pragma unroll
        for (int s = 0; s < BK / 4; ++s) {
            const int cur = s & 1;
#if XK_FB1
            load_b(st, s);
            // the last step's B fragments are this warp's last read of the stage (its A
            // fragments were loaded one step earlier)
            if (s + 1 == BK / 4) release_stage();
#endif
            if (s + 1 < BK / 4) {
                load_frags(cur ^ 1, st, s + 1);
#if !XK_FB1
                if (s + 2 == BK / 4) release_stage();  // the next step's A and B are loaded
#endif
            } else if (kb + 1 < KB) {
                const int nx = (kb + 1) % STAGES;
                mbar_wait(full(nx), (uint32_t)(((kb + 1) / STAGES) & 1));
                load_frags(cur ^ 1, nx, 0);
            }
#pragma unroll
            for (int i = 0; i < MF; ++i)
#pragma unroll
                for (int j = 0; j < NF; ++j) dmma(acc[i][j], fa[cur][i], fb[XK_FB1 ? 0 : cur][j]);
        }
    }

    // epilogue: D = alpha*acc + beta*C (+ beta2*C2) (C, C2 not read when their beta is 0).
    // Loads first, per chunk of EPI_ROWS row fragments, then the stores: the compiler cannot
    // prove that a store to C does not alias a later load of C, so loads interleaved with
    // stores would cost one L2 round trip per element (32 in a row per thread, ~6 us per CTA
    // -- 1.2% of a T=4096 tile's main loop, 5% of a T=1024 one); batched they cost one per chunk.
    const double alpha = t.alpha, beta = t.beta, beta2 = t.beta2;
    double *C = t.C;
    const int64_t ldc = t.ldc;
    const double *C2 = t.C2;
    const int64_t ldc2 = t.ldc2;
#pragma unroll
    for (int i0 = 0; i0 < MF; i0 += EPI_ROWS) {
        double cv[EPI_ROWS][NF][2], c2v[EPI_ROWS][NF][2];
#pragma unroll
        for (int ii = 0; ii < EPI_ROWS; ++ii) {
            const int64_t r = m0 + wm + (i0 + ii) * 8 + fr;
#pragma unroll
            for (int j = 0; j < NF; ++j)
#pragma unroll
                for (int h = 0; h < 2; ++h) {
                    const int64_t c = n0 + wn + j * 8 + fc * 2 + h;
                    const bool ok = r < M && c < N && !((tri == 1 && r < c) || (tri == 2 && r > c));
                    cv[ii][j][h] = (ok && beta != 0.0) ? C[r + c * ldc] : 0.0;
                    c2v[ii][j][h] = (ok && beta2 != 0.0) ? C2[r + c * ldc2] : 0.0;
                }
        }
#pragma unroll
        for (int ii = 0; ii < EPI_ROWS; ++ii) {
            const int64_t r = m0 + wm + (i0 + ii) * 8 + fr;
#pragma unroll
            for (int j = 0; j < NF; ++j)
#pragma unroll
                for (int h = 0; h < 2; ++h) {
                    const int64_t c = n0 + wn + j * 8 + fc * 2 + h;
                    if (r >= M || c >= N || (tri == 1 && r < c) || (tri == 2 && r > c)) continue;
                    double v = alpha * acc[i0 + ii][j][h];
                    if (beta != 0.0) v = fma(beta, cv[ii][j][h], v);
                    if (beta2 != 0.0) v = fma(beta2, c2v[ii][j][h], v);
                    C[r + c * ldc] = v;
                }
        }
    }
}

typedef CUresult (*EncodeTiledFn)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *,
                                  const cuuint64_t *, const cuuint64_t *, const cuuint32_t *,
                                  const cuuint32_t *, CUtensorMapInterleave, CUtensorMapSwizzle,
                                  CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

EncodeTiledFn encode_fn() {
    static EncodeTiledFn fn = nullptr;
    static bool tried = false;
    if (!tried) {
        tried = true;
        void *p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = reinterpret_cast<EncodeTiledFn>(p);
        cudaGetLastError();
    }
    return fn;
}

}  // namespace

// Tensor map of a stored column-major operand (rows x cols, ld) for the TMA kernel.
// mn_contig: the contiguous dimension is m/n (box 16 x 16); else it is k (box 16 x bmn).
bool make_tma_operand(CUtensorMap *map, const double *X, int64_t rows, int64_t cols, int64_t ld,
                      bool mn_contig, int bmn, int *is3d) {
    EncodeTiledFn fn = encode_fn();
    if (!fn) return false;
    if (((uintptr_t)X & 15) || ((ld * 8) & 15) || rows <= 0 || cols <= 0) return false;
    if (is3d) *is3d = 0;
    static int use3d = -1;
    if (use3d < 0) {
        const char *e = getenv("XK_TMA3D");
        use3d = (e && *e == '0') ? 0 : 1;
    }
    if (mn_contig && is3d && use3d && rows % 16 == 0) {
        // the same operand as (16 rows in a chunk, cols, rows/16 chunks): one box of
        // 16 x 16 x bmn/16 per stage instead of bmn/16 boxes (every chunk in bounds)
        cuuint64_t dims3[3] = {16u, (cuuint64_t)cols, (cuuint64_t)(rows / 16)};
        cuuint64_t strides3[2] = {(cuuint64_t)(ld * 8), 128u};
        cuuint32_t box3[3] = {16u, 16u, (cuuint32_t)(bmn / 16)};
        cuuint32_t estr3[3] = {1u, 1u, 1u};
        CUresult r3 = fn(map, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 3, const_cast<double *>(X), dims3, strides3, box3,
                         estr3, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                         CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
        if (r3 == CUDA_SUCCESS) {
            *is3d = 1;
            return true;
        }
    }
    cuuint64_t dims[2] = {(cuuint64_t)rows, (cuuint64_t)cols};
    cuuint64_t strides[1] = {(cuuint64_t)(ld * 8)};
    cuuint32_t box[2] = {16u, mn_contig ? 16u : (cuuint32_t)bmn};
    cuuint32_t estr[2] = {1u, 1u};
    CUresult r = fn(map, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 2, const_cast<double *>(X), dims, strides, box,
                    estr, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                    CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS;
}

int tma_bm() { return BM; }
int tma_bn() { return BN; }

cudaError_t launch_dgemm_tma(bool ta, bool tb, TmaBatch &b, cudaStream_t st) {
    if (b.n <= 0) return cudaSuccess;
    static int group_m = -1;
    if (group_m < 0) {
        const char *e = getenv("XK_GROUP_M");
        group_m = (e && *e) ? atoi(e) : 16;
    }
    b.group_m = group_m;
    static int snake = -1;
    if (snake < 0) {
        const char *e = getenv("XK_SNAKE");
        snake = (e && *e == '0') ? 0 : 1;
    }
    b.snake = snake;
    constexpr size_t smem = STAGES * STAGE_BYTES + STAGES * 8 + STAGES * 4 + 1024;
    int total = 0;
    for (int q = 0; q < b.n; ++q) {
        b.cta_start[q] = total;
        total += (int)(((b.t[q].M + BM - 1) / BM) * ((b.t[q].N + BN - 1) / BN));
    }
    b.cta_start[b.n] = total;
    if (total == 0) return cudaSuccess;
    static unsigned attr_set[8] = {0, 0, 0, 0, 0, 0, 0, 0};  // per kernel instance, one bit per device
    auto go = [&](void (*kern)(TmaBatch), int which) -> cudaError_t {
        int dev = 0;
        cudaGetDevice(&dev);
        if (!(attr_set[which] & (1u << dev))) {
            cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
            if (e != cudaSuccess) return e;
            attr_set[which] |= 1u << dev;
        }
        kern<<<total, NTHREADS, smem, st>>>(b);
        return cudaGetLastError();
    };
    // 3D maps for the mn-contiguous operands only if every task of the batch has them (the
    // caller builds all of a batch's maps 2D or all 3D; a mixed batch is an error)
    bool d3 = true, any3 = false;
    for (int q = 0; q < b.n; ++q) {
        d3 = d3 && (ta || b.t[q].a3d) && (!tb || b.t[q].b3d);
        any3 = any3 || b.t[q].a3d || b.t[q].b3d;
    }
    if (any3 && !d3) return cudaErrorInvalidValue;
    if (!ta && !tb) return d3 ? go(dgemm_tma_kernel<false, false, true>, 4) : go(dgemm_tma_kernel<false, false, false>, 0);
    if (!ta && tb) return d3 ? go(dgemm_tma_kernel<false, true, true>, 5) : go(dgemm_tma_kernel<false, true, false>, 1);
    if (ta && !tb) return go(dgemm_tma_kernel<true, false, false>, 2);
    return d3 ? go(dgemm_tma_kernel<true, true, true>, 7) : go(dgemm_tma_kernel<true, true, false>, 3);
}

}  // namespace xk
