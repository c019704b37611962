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
#include <cuda_runtime.h>
#include <stdint.h>

#include "kernels/kernels.h"

namespace xk {
namespace {

constexpr int BK = 16;          // k per pipeline stage
constexpr int PAD_MN = 4;       // [k][mn] layout: stride BM+4 doubles (2*stride = 8 mod 32 words)
constexpr int STRIDE_K = 20;    // [mn][k] layout: stride 16+4 doubles

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

template <int VEC>
__device__ __forceinline__ void cp_async(double *dst, const double *src, int valid) {
    // copy `valid` of VEC doubles, zero-fill the rest (src-size operand)
    uint32_t d = smem_u32(dst);
    if constexpr (VEC == 2) {
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;\n" ::"r"(d), "l"(src),
                     "r"(valid * 8));
    } else {
        asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;\n" ::"r"(d), "l"(src),
                     "r"(valid * 8));
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

// Shared-memory footprint of one operand slab (BMN x BK) in doubles.
template <int BMN, bool MN_CONTIG>
struct Slab {
    static constexpr int kStride = MN_CONTIG ? (BMN + PAD_MN) : STRIDE_K;
    static constexpr int kDoubles = MN_CONTIG ? BK * (BMN + PAD_MN) : BMN * STRIDE_K;
    __device__ __forceinline__ static int idx(int mn, int k) {
        return MN_CONTIG ? k * kStride + mn : mn * kStride + k;
    }
};

// Load a BMN x BK slab of op(X) into shared memory.  Global element (mn, k) of op(X) is
// X[mn + k*ld] when MN_CONTIG (mn contiguous) else X[k + mn*ld].
template <int BMN, bool MN_CONTIG, int VEC, int NTHREADS>
__device__ __forceinline__ void load_slab(double *s, const double *X, int64_t ld, int64_t mn0,
                                          int64_t k0, int64_t MN, int64_t K, int tid) {
    using S = Slab<BMN, MN_CONTIG>;
    constexpr int kChunks = BMN * BK / VEC;
    static_assert(kChunks % NTHREADS == 0, "chunking");
#pragma unroll
    for (int q = 0; q < kChunks / NTHREADS; ++q) {
        int c = tid + q * NTHREADS;
        int mn, k;
        int64_t gm, gk;
        int valid;
        if (MN_CONTIG) {
            k = c / (BMN / VEC);
            mn = (c % (BMN / VEC)) * VEC;
            gm = mn0 + mn;
            gk = k0 + k;
            int64_t rem = MN - gm;
            valid = (gk < K && rem > 0) ? (int)(rem < VEC ? rem : VEC) : 0;
        } else {
            mn = c / (BK / VEC);
            k = (c % (BK / VEC)) * VEC;
            gm = mn0 + mn;
            gk = k0 + k;
            int64_t rem = K - gk;
            valid = (gm < MN && rem > 0) ? (int)(rem < VEC ? rem : VEC) : 0;
        }
        const double *src = valid ? (MN_CONTIG ? X + gm + gk * ld : X + gk + gm * ld) : X;
        cp_async<VEC>(s + S::idx(mn, k), src, valid);
    }
}

template <int BM, int BN, int WM, int WN, int STAGES, bool TA, bool TB, int VEC>
__global__ void __launch_bounds__((BM / WM) * (BN / WN) * 32, 1)
dgemm_tile_kernel(int64_t M, int64_t N, int64_t K, double alpha, const double *__restrict__ A,
                  int64_t lda, const double *__restrict__ B, int64_t ldb, double beta,
                  double *__restrict__ C, int64_t ldc) {
    constexpr int NWM = BM / WM, NWN = BN / WN;
    constexpr int NTHREADS = NWM * NWN * 32;
    constexpr int MF = WM / 8, NF = WN / 8;
    // A: op(A) is M x K; 'N' -> m contiguous, 'T' -> k contiguous.
    // B: op(B) is K x N; 'N' -> k contiguous, 'T' -> n contiguous.
    constexpr bool A_MN = !TA;
    constexpr bool B_MN = TB;
    using SA = Slab<BM, A_MN>;
    using SB = Slab<BN, B_MN>;

    extern __shared__ __align__(128) double smem[];
    double *sA = smem;
    double *sB = smem + STAGES * SA::kDoubles;

    const int tid = threadIdx.x;
    const int lane = tid & 31, warp = tid >> 5;
    const int wm = (warp % NWM) * WM, wn = (warp / NWM) * WN;
    const int64_t m0 = (int64_t)blockIdx.x * BM, n0 = (int64_t)blockIdx.y * BN;
    const int KB = (int)((K + BK - 1) / BK);

    double acc[MF][NF][2];
#pragma unroll
    for (int i = 0; i < MF; ++i)
#pragma unroll
        for (int j = 0; j < NF; ++j) acc[i][j][0] = acc[i][j][1] = 0.0;

#pragma unroll
    for (int s = 0; s < STAGES - 1; ++s) {
        if (s < KB) {
            load_slab<BM, A_MN, VEC, NTHREADS>(sA + s * SA::kDoubles, A, lda, m0, (int64_t)s * BK, M, K, tid);
            load_slab<BN, B_MN, VEC, NTHREADS>(sB + s * SB::kDoubles, B, ldb, n0, (int64_t)s * BK, N, K, tid);
        }
        cp_commit();
    }

    const int fr = lane >> 2, fc = lane & 3;
    for (int kb = 0; kb < KB; ++kb) {
        cp_wait<STAGES - 2>();
        __syncthreads();
        {
            int nk = kb + STAGES - 1;
            if (nk < KB) {
                int st = nk % STAGES;
                load_slab<BM, A_MN, VEC, NTHREADS>(sA + st * SA::kDoubles, A, lda, m0, (int64_t)nk * BK, M, K, tid);
                load_slab<BN, B_MN, VEC, NTHREADS>(sB + st * SB::kDoubles, B, ldb, n0, (int64_t)nk * BK, N, K, tid);
            }
            cp_commit();
        }
        const double *a = sA + (kb % STAGES) * SA::kDoubles;
        const double *b = sB + (kb % STAGES) * SB::kDoubles;
#pragma unroll
        for (int ks = 0; ks < BK; ks += 4) {
            double fa[MF], fb[NF];
#pragma unroll
            for (int i = 0; i < MF; ++i) fa[i] = a[SA::idx(wm + i * 8 + fr, ks + fc)];
#pragma unroll
            for (int j = 0; j < NF; ++j) fb[j] = b[SB::idx(wn + j * 8 + fr, ks + fc)];
#pragma unroll
            for (int i = 0; i < MF; ++i)
#pragma unroll
                for (int j = 0; j < NF; ++j) dmma(acc[i][j], fa[i], fb[j]);
        }
    }
    cp_wait<0>();

    // epilogue: D = alpha*acc + beta*C (C not read when beta == 0)
#pragma unroll
    for (int i = 0; i < MF; ++i) {
        int64_t r = m0 + wm + i * 8 + fr;
        if (r >= M) continue;
#pragma unroll
        for (int j = 0; j < NF; ++j) {
#pragma unroll
            for (int h = 0; h < 2; ++h) {
                int64_t c = n0 + wn + j * 8 + fc * 2 + h;
                if (c >= N) continue;
                double *p = C + r + c * ldc;
                double v = alpha * acc[i][j][h];
                if (beta != 0.0) v = fma(beta, *p, v);
                *p = v;
            }
        }
    }
}

template <int BM, int BN, int WM, int WN, int STAGES, bool TA, bool TB, int VEC>
cudaError_t launch_cfg(int64_t M, int64_t N, int64_t K, double alpha, const double *A,
                       int64_t lda, const double *B, int64_t ldb, double beta, double *C,
                       int64_t ldc, cudaStream_t st) {
    using SA = Slab<BM, !TA>;
    using SB = Slab<BN, TB>;
    constexpr size_t smem = (size_t)STAGES * (SA::kDoubles + SB::kDoubles) * sizeof(double);
    auto kern = dgemm_tile_kernel<BM, BN, WM, WN, STAGES, TA, TB, VEC>;
    static unsigned attr_set = 0;  // per instantiation, one bit per device (idempotent)
    int dev = 0;
    cudaGetDevice(&dev);
    if (!(attr_set & (1u << dev))) {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
        attr_set |= 1u << dev;
    }
    dim3 grid((unsigned)((M + BM - 1) / BM), (unsigned)((N + BN - 1) / BN));
    dim3 block((BM / WM) * (BN / WN) * 32);
    kern<<<grid, block, smem, st>>>(M, N, K, alpha, A, lda, B, ldb, beta, C, ldc);
    return cudaGetLastError();
}

template <bool TA, bool TB, int VEC>
cudaError_t launch_t(int64_t M, int64_t N, int64_t K, double alpha, const double *A, int64_t lda,
                     const double *B, int64_t ldb, double beta, double *C, int64_t ldc,
                     cudaStream_t st) {
    return launch_cfg<128, 128, 64, 32, 4, TA, TB, VEC>(M, N, K, alpha, A, lda, B, ldb, beta, C,
                                                        ldc, st);
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

cudaError_t launch_dgemm_tile(bool ta, bool tb, int64_t M, int64_t N, int64_t K, double alpha,
                              const double *A, int64_t lda, const double *B, int64_t ldb,
                              double beta, double *C, int64_t ldc, cudaStream_t st) {
    if (M <= 0 || N <= 0) return cudaSuccess;
    if (alpha == 0.0 || K <= 0) return launch_scale_tile(M, N, beta, C, ldc, st);
    // 16-byte cp.async needs 16-byte aligned columns of both operands
    bool v2 = ((lda | ldb) % 2 == 0) && (((uintptr_t)A | (uintptr_t)B) % 16 == 0);
#define XK_DISPATCH(VEC)                                                                       \
    if (!ta && !tb) return launch_t<false, false, VEC>(M, N, K, alpha, A, lda, B, ldb, beta, C, ldc, st); \
    if (!ta && tb) return launch_t<false, true, VEC>(M, N, K, alpha, A, lda, B, ldb, beta, C, ldc, st);   \
    if (ta && !tb) return launch_t<true, false, VEC>(M, N, K, alpha, A, lda, B, ldb, beta, C, ldc, st);   \
    return launch_t<true, true, VEC>(M, N, K, alpha, A, lda, B, ldb, beta, C, ldc, st);
    if (v2) {
        XK_DISPATCH(2)
    } else {
        XK_DISPATCH(1)
    }
#undef XK_DISPATCH
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
