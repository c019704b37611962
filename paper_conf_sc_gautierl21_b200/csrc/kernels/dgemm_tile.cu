// dgemm_tile.cu -- FP64 tile GEMM for sm_100a.
//
//   D = alpha * op(A) * op(B) + beta * C     on column-major device tiles,
//
// the operation every XKBlas GEMM tile task performs on its compact tiles (PAPER.md
// P:399-406 "the compact tile form is used as effective parameters for GPU kernels";
// tiled algorithms).  beta == 0: C is not read.
//
// B200 design (measured): sm_100a has no tcgen05 kind for f64; the
// FP64 tensor path is the warp-level mma.sync.m8n8k4.f64 which ptxas lowers to
// DMMA.8x8x4.  A probe on the box measured DMMA at 37.07 TFLOP/s (99.6% of the derived
// 37.2 = 148 SM x 64 FMA/clk x 2 x 1.965 GHz) vs 34.1 for DFMA, so the contraction runs
// on DMMA.  Operands are staged through a multi-stage cp.async (LDGSTS) shared-memory
// ring with zero-fill predication for ragged edges; fragments are read with
// conflict-free padded strides; alpha/beta are fused into the register epilogue.
//
// One launch runs a BATCH of up to kMaxBatch independent tile tasks (grouped GEMM): the
// executor groups ready tasks of one GPU so a launch is many waves long -- no per-task
// wave-quantization tail (a single T=2048 task is only 1.7 waves on 148 SMs) and one
// launch per batch instead of per task.
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdlib.h>

#include "kernels/kernels.h"

namespace xk {
namespace {

constexpr int PAD_MN = 4;  // [k][mn] layout: stride BMN+4 doubles (2*stride = 8 mod 32 words)

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

template <int VEC>
__device__ __forceinline__ void cp_async(uint32_t dst, const double *src, int valid) {
    // copy `valid` of VEC doubles, zero-fill the rest (src-size operand)
    if constexpr (VEC == 2) {
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;\n" ::"r"(dst), "l"(src), "r"(valid * 8));
    } else {
        asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;\n" ::"r"(dst), "l"(src), "r"(valid * 8));
    }
}
__device__ __forceinline__ void cp_commit() { asm volatile("cp.async.commit_group;\n" ::); }
template <int N>
__device__ __forceinline__ void cp_wait() { asm volatile("cp.async.wait_group %0;\n" ::"n"(N)); }

__device__ __forceinline__ void dmma(double (&c)[2], double a, double b) {
    asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
                 : "+d"(c[0]), "+d"(c[1])
                 : "d"(a), "d"(b));
}

// Shared-memory slab of op(X), BMN x BK doubles.  MN_CONTIG: stored [k][mn] (mn
// contiguous, stride BMN+4); else [mn][k] (k contiguous, stride BK+4).  Both strides give
// conflict-free 8-byte fragment reads for the m8n8k4 A/B fragments.
template <int BMN, bool MN_CONTIG, int BK>
struct Slab {
    static constexpr int kStride = MN_CONTIG ? (BMN + PAD_MN) : (BK + 4);
    static constexpr int kDoubles = MN_CONTIG ? BK * (BMN + PAD_MN) : BMN * (BK + 4);
    __device__ __forceinline__ static int idx(int mn, int k) {
        return MN_CONTIG ? k * kStride + mn : mn * kStride + k;
    }
};

// Loader of one operand slab: a thread's chunks keep the same (mn, k) slab coordinates
// every stage; interior blocks skip the ragged-edge predication entirely.
template <int BMN, bool MN_CONTIG, int BK, int VEC, int NTHREADS>
struct Loader {
    using S = Slab<BMN, MN_CONTIG, BK>;
    static constexpr int kChunks = BMN * BK / VEC / NTHREADS;  // chunks per thread
    static_assert(BMN * BK / VEC % NTHREADS == 0, "chunking");
    const double *base;
    int64_t ld, MN, K, mn0;

    __device__ __forceinline__ static void coords(int c, int &mn, int &k) {
        if (MN_CONTIG) {
            k = c / (BMN / VEC);
            mn = (c % (BMN / VEC)) * VEC;
        } else {
            mn = c / (BK / VEC);
            k = (c % (BK / VEC)) * VEC;
        }
    }
    __device__ __forceinline__ void init(const double *X, int64_t ld_, int64_t mn0_, int64_t MN_,
                                         int64_t K_) {
        base = X;
        ld = ld_;
        mn0 = mn0_;
        MN = MN_;
        K = K_;
    }
    // issue the copies of the k-block starting at k0 into the slab at shared address s
    __device__ __forceinline__ void load(uint32_t s, int64_t k0, int tid, bool interior) const {
#pragma unroll
        for (int q = 0; q < kChunks; ++q) {
            int mn, k;
            coords(tid + q * NTHREADS, mn, k);
            const int64_t gm = mn0 + mn, gk = k0 + k;
            int valid;
            if (interior) {
                valid = VEC;
            } else if (MN_CONTIG) {
                const int64_t rem = MN - gm;
                valid = (gk < K && rem > 0) ? (int)(rem < VEC ? rem : VEC) : 0;
            } else {
                const int64_t rem = K - gk;
                valid = (gm < MN && rem > 0) ? (int)(rem < VEC ? rem : VEC) : 0;
            }
            const double *src = valid ? (MN_CONTIG ? base + gm + gk * ld : base + gk + gm * ld) : base;
            cp_async<VEC>(s + 8u * (uint32_t)S::idx(mn, k), src, valid);
        }
    }
};

template <int BM, int BN, int WM, int WN, int BK, int STAGES, int MINB, bool TA, bool TB, int VEC>
__global__ void __launch_bounds__((BM / WM) * (BN / WN) * 32, MINB)
dgemm_tile_kernel(const __grid_constant__ TileBatch batch) {
    constexpr int NWM = BM / WM, NWN = BN / WN;
    constexpr int NTHREADS = NWM * NWN * 32;
    constexpr int MF = WM / 8, NF = WN / 8;
    // A: op(A) is M x K; 'N' -> m contiguous, 'T' -> k contiguous.
    // B: op(B) is K x N; 'N' -> k contiguous, 'T' -> n contiguous.
    constexpr bool A_MN = !TA;
    constexpr bool B_MN = TB;
    using SA = Slab<BM, A_MN, BK>;
    using SB = Slab<BN, B_MN, BK>;

    // which task of the batch, which CTA tile of it
    int q = 0;
    const int bid = blockIdx.x;
#pragma unroll 1
    while (q + 1 < batch.n && bid >= batch.cta_start[q + 1]) ++q;
    const TileTask &t = batch.t[q];
    const int local = bid - batch.cta_start[q];
    const int tiles_m = (int)((t.M + BM - 1) / BM);
    const int64_t m0 = (int64_t)(local % tiles_m) * BM, n0 = (int64_t)(local / tiles_m) * BN;
    const int64_t M = t.M, N = t.N, K = t.K;
    const int tri = t.tri;
    // diagonal tiles of SYRK/SYR2K: CTAs entirely outside the written triangle do nothing
    if ((tri == 1 && m0 + BM - 1 < n0) || (tri == 2 && n0 + BN - 1 < m0)) return;

    extern __shared__ __align__(128) double smem[];
    const uint32_t sA0 = smem_u32(smem);
    const uint32_t sB0 = sA0 + 8u * STAGES * SA::kDoubles;

    const int tid = threadIdx.x;
    const int lane = tid & 31, warp = tid >> 5;
    const int wm = (warp % NWM) * WM, wn = (warp / NWM) * WN;
    const int KB = (int)((K + BK - 1) / BK);
    const bool mn_interior = (m0 + BM <= M) && (n0 + BN <= N);

    Loader<BM, A_MN, BK, VEC, NTHREADS> la;
    Loader<BN, B_MN, BK, VEC, NTHREADS> lb;
    la.init(t.A, t.lda, m0, M, K);
    lb.init(t.B, t.ldb, n0, N, K);

    double acc[MF][NF][2];
#pragma unroll
    for (int i = 0; i < MF; ++i)
#pragma unroll
        for (int j = 0; j < NF; ++j) acc[i][j][0] = acc[i][j][1] = 0.0;

#pragma unroll
    for (int s = 0; s < STAGES - 1; ++s) {
        if (s < KB) {
            const int64_t k0 = (int64_t)s * BK;
            const bool in = mn_interior && (k0 + BK <= K);
            la.load(sA0 + 8u * s * SA::kDoubles, k0, tid, in);
            lb.load(sB0 + 8u * s * SB::kDoubles, k0, tid, in);
        }
        cp_commit();
    }

    const int fr = lane >> 2, fc = lane & 3;
    const double *sAd = smem;
    const double *sBd = smem + STAGES * SA::kDoubles;
    constexpr int KS = BK / 4;
    // Fragments are double-buffered in registers: the loads for step ks+1 (or for step 0
    // of the next k-block, right after the one barrier per block) are issued before the
    // DMMAs of step ks, so shared-memory latency hides behind 32 DMMAs.
    double fa[2][MF], fb[2][NF];
    auto load_frags = [&](int buf, const double *a, const double *b, int ks) {
#pragma unroll
        for (int i = 0; i < MF; ++i) fa[buf][i] = a[SA::idx(wm + i * 8 + fr, ks * 4 + fc)];
#pragma unroll
        for (int j = 0; j < NF; ++j) fb[buf][j] = b[SB::idx(wn + j * 8 + fr, ks * 4 + fc)];
    };
    cp_wait<STAGES - 2>();
    __syncthreads();
    load_frags(0, sAd, sBd, 0);
#pragma unroll 1
    for (int kb = 0; kb < KB; ++kb) {
        {
            // stage (kb-1) % STAGES was released by the barrier of the previous block
            const int nk = kb + STAGES - 1;
            if (nk < KB) {
                const int st = nk % STAGES;
                const int64_t k0 = (int64_t)nk * BK;
                const bool in = mn_interior && (k0 + BK <= K);
                la.load(sA0 + 8u * st * SA::kDoubles, k0, tid, in);
                lb.load(sB0 + 8u * st * SB::kDoubles, k0, tid, in);
            }
            cp_commit();
        }
        const double *a = sAd + (kb % STAGES) * SA::kDoubles;
        const double *b = sBd + (kb % STAGES) * SB::kDoubles;
#pragma unroll
        for (int ks = 0; ks < KS; ++ks) {
            const int cur = ks & 1;
            if (ks + 1 < KS) {
                load_frags(cur ^ 1, a, b, ks + 1);
            } else if (kb + 1 < KB) {
                // next block's stage has landed for every thread; this block's stage is
                // no longer read after this barrier
                cp_wait<STAGES - 2>();
                __syncthreads();
                const int nx = (kb + 1) % STAGES;
                load_frags(cur ^ 1, sAd + nx * SA::kDoubles, sBd + nx * SB::kDoubles, 0);
            }
#pragma unroll
            for (int i = 0; i < MF; ++i)
#pragma unroll
                for (int j = 0; j < NF; ++j) dmma(acc[i][j], fa[cur][i], fb[cur][j]);
        }
    }
    cp_wait<0>();

    // epilogue: D = alpha*acc + beta*C (+ beta2*C2) (C, C2 not read when their beta is 0);
    // one row fragment's loads are issued before its stores (see dgemm_tma.cu: interleaved,
    // every element would cost an L2 round trip, since a store may alias a later load)
    const double alpha = t.alpha, beta = t.beta, beta2 = t.beta2;
    double *C = t.C;
    const int64_t ldc = t.ldc;
    const double *C2 = t.C2;
    const int64_t ldc2 = t.ldc2;
#pragma unroll
    for (int i = 0; i < MF; ++i) {
        const int64_t r = m0 + wm + i * 8 + fr;
        double cv[NF][2], c2v[NF][2];
#pragma unroll
        for (int j = 0; j < NF; ++j)
#pragma unroll
            for (int h = 0; h < 2; ++h) {
                const int64_t c = n0 + wn + j * 8 + fc * 2 + h;
                const bool ok = r < M && c < N && !((tri == 1 && r < c) || (tri == 2 && r > c));
                cv[j][h] = (ok && beta != 0.0) ? C[r + c * ldc] : 0.0;
                c2v[j][h] = (ok && beta2 != 0.0) ? C2[r + c * ldc2] : 0.0;
            }
#pragma unroll
        for (int j = 0; j < NF; ++j)
#pragma unroll
            for (int h = 0; h < 2; ++h) {
                const int64_t c = n0 + wn + j * 8 + fc * 2 + h;
                if (r >= M || c >= N || (tri == 1 && r < c) || (tri == 2 && r > c)) continue;
                double v = alpha * acc[i][j][h];
                if (beta != 0.0) v = fma(beta, cv[j][h], v);
                if (beta2 != 0.0) v = fma(beta2, c2v[j][h], v);
                C[r + c * ldc] = v;
            }
    }
}

template <int BM, int BN, int WM, int WN, int BK, int STAGES, int MINB, bool TA, bool TB, int VEC>
cudaError_t launch_cfg(TileBatch &b, cudaStream_t st) {
    using SA = Slab<BM, !TA, BK>;
    using SB = Slab<BN, TB, BK>;
    constexpr size_t smem = (size_t)STAGES * (SA::kDoubles + SB::kDoubles) * sizeof(double);
    auto kern = dgemm_tile_kernel<BM, BN, WM, WN, BK, STAGES, MINB, TA, TB, VEC>;
    static unsigned attr_set = 0;  // per instantiation, one bit per device (idempotent)
    int dev = 0;
    cudaGetDevice(&dev);
    if (!(attr_set & (1u << dev))) {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
        attr_set |= 1u << dev;
    }
    int total = 0;
    for (int q = 0; q < b.n; ++q) {
        b.cta_start[q] = total;
        total += (int)(((b.t[q].M + BM - 1) / BM) * ((b.t[q].N + BN - 1) / BN));
    }
    b.cta_start[b.n] = total;
    if (total == 0) return cudaSuccess;
    kern<<<total, (BM / WM) * (BN / WN) * 32, smem, st>>>(b);
    return cudaGetLastError();
}

// Kernel configurations (tuning sweep via XK_KCFG; the default is the measured best).
//   0: 128x128 CTA, 8 warps of 64x32, BK 16, 4 stages, 1 CTA/SM
//   1: 128x64  CTA, 4 warps of 64x32, BK 16, 4 stages, 2 CTAs/SM (independent barriers)
//   2: 128x128 CTA, 8 warps of 64x32, BK 32, 3 stages
//   4: 128x64  CTA, 4 warps of 64x32, BK 16, 3 stages, 2 CTAs/SM
//   5: 128x64  CTA, 8 warps of 32x32, BK 16, 3 stages, 2 CTAs/SM (4 warps per scheduler)
//   6: 64x128  CTA, 8 warps of 32x32, BK 16, 3 stages, 2 CTAs/SM  (default: measured best,
//      32.0 TFLOP/s on a T=4096 tile vs 30.8 for cfg 4 and 31.1 for cfg 0)
//   7: 128x64  CTA, 8 warps of 32x32, BK 32, 2 stages, 2 CTAs/SM
int g_kcfg = -1;
int kcfg() {
    if (g_kcfg < 0) {
        const char *e = getenv("XK_KCFG");
        g_kcfg = (e && *e) ? atoi(e) : 6;
    }
    return g_kcfg;
}

template <bool TA, bool TB, int VEC>
cudaError_t launch_t(TileBatch &b, cudaStream_t st) {
    switch (kcfg()) {
    case 0:
        return launch_cfg<128, 128, 64, 32, 16, 4, 1, TA, TB, VEC>(b, st);
    case 1:
        return launch_cfg<128, 64, 64, 32, 16, 4, 2, TA, TB, VEC>(b, st);
    case 2:
        return launch_cfg<128, 128, 64, 32, 32, 3, 1, TA, TB, VEC>(b, st);
    case 5:
        return launch_cfg<128, 64, 32, 32, 16, 3, 2, TA, TB, VEC>(b, st);
    case 6:
        return launch_cfg<64, 128, 32, 32, 16, 3, 2, TA, TB, VEC>(b, st);
    case 7:
        return launch_cfg<128, 64, 32, 32, 32, 2, 2, TA, TB, VEC>(b, st);
    default:
        return launch_cfg<128, 64, 64, 32, 16, 3, 2, TA, TB, VEC>(b, st);
    }
}

__global__ void scale_tile_kernel(int64_t M, int64_t N, double beta, double *C, int64_t ldc) {
    int64_t total = M * N;
    for (int64_t q = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; q < total;
         q += (int64_t)gridDim.x * blockDim.x) {
        int64_t r = q % M, c = q / M;
        double *p = C + r + c * ldc;
        *p = (beta == 0.0) ? 0.0 : beta * *p;
    }
}

}  // namespace

bool tma_enabled() {
    static int on = -1;
    if (on < 0) {
        const char *e = getenv("XK_TMA");
        on = (e && *e) ? atoi(e) : 1;
    }
    return on != 0;
}

// Grouped launch: the TMA + mbarrier kernel when every operand can be described by a
// tensor map (16-byte aligned base and ld), else the cp.async kernel.
cudaError_t launch_dgemm_batch(bool ta, bool tb, TileBatch &b, cudaStream_t st) {
    if (b.n <= 0) return cudaSuccess;
    if (tma_enabled() && b.n <= kMaxTmaBatch) {
        static thread_local TmaBatch tb_;
        tb_.n = b.n;
        bool ok = true;
        // the mn-contiguous operands go as 3D maps (one TMA box per stage) only if every
        // task's can: the batch runs one kernel instance, 2D or 3D, for all of them
        bool all3d = true;
        for (int q = 0; q < b.n; ++q)
            all3d = all3d && (ta || b.t[q].M % 16 == 0) && (!tb || b.t[q].N % 16 == 0);
        for (int q = 0; q < b.n && ok; ++q) {
            const TileTask &t = b.t[q];
            TmaTask &u = tb_.t[q];
            u.a3d = u.b3d = 0;
            ok = make_tma_operand(&u.mapA, t.A, ta ? t.K : t.M, ta ? t.M : t.K, t.lda, !ta, tma_bm(),
                                  all3d ? &u.a3d : nullptr) &&
                 make_tma_operand(&u.mapB, t.B, tb ? t.N : t.K, tb ? t.K : t.N, t.ldb, tb, tma_bn(),
                                  all3d ? &u.b3d : nullptr);
            u.C = t.C;
            u.ldc = t.ldc;
            u.M = t.M;
            u.N = t.N;
            u.K = t.K;
            u.alpha = t.alpha;
            u.beta = t.beta;
            u.tri = t.tri;
            u.C2 = t.C2;
            u.ldc2 = t.ldc2;
            u.beta2 = t.beta2;
        }
        if (ok) return launch_dgemm_tma(ta, tb, tb_, st);
    }
    // 16-byte cp.async needs 16-byte aligned columns of both operands in every task
    bool v2 = true;
    for (int q = 0; q < b.n; ++q)
        v2 = v2 && ((b.t[q].lda | b.t[q].ldb) % 2 == 0) &&
             ((((uintptr_t)b.t[q].A) | ((uintptr_t)b.t[q].B)) % 16 == 0);
#define XK_DISPATCH(VEC)                                               \
    if (!ta && !tb) return launch_t<false, false, VEC>(b, st);          \
    if (!ta && tb) return launch_t<false, true, VEC>(b, st);            \
    if (ta && !tb) return launch_t<true, false, VEC>(b, st);            \
    return launch_t<true, true, VEC>(b, st);
    if (v2) {
        XK_DISPATCH(2)
    } else {
        XK_DISPATCH(1)
    }
#undef XK_DISPATCH
}

cudaError_t launch_dgemm_tile(bool ta, bool tb, int64_t M, int64_t N, int64_t K, double alpha,
                              const double *A, int64_t lda, const double *B, int64_t ldb,
                              double beta, double *C, int64_t ldc, cudaStream_t st) {
    if (M <= 0 || N <= 0) return cudaSuccess;
    if (alpha == 0.0 || K <= 0) return launch_scale_tile(M, N, beta, C, ldc, st);
    TileBatch b;
    b.n = 1;
    b.t[0] = TileTask{A, B, C, lda, ldb, ldc, M, N, K, alpha, beta, 0, nullptr, 0, 0.0};
    return launch_dgemm_batch(ta, tb, b, st);
}

cudaError_t launch_scale_tile(int64_t M, int64_t N, double beta, double *C, int64_t ldc,
                              cudaStream_t st) {
    if (M <= 0 || N <= 0 || beta == 1.0) return cudaSuccess;
    int64_t total = M * N;
    int blocks = (int)((total + 255) / 256);
    if (blocks > 148 * 8) blocks = 148 * 8;
    scale_tile_kernel<<<blocks, 256, 0, st>>>(M, N, beta, C, ldc);
    return cudaGetLastError();
}

}  // namespace xk
