// kernels.h -- internal launch interface of the sm_100a tile kernels (no torch types).
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>

namespace xk {

// One tile task D = alpha*op(A)*op(B) + beta*C on column-major device tiles.
struct TileTask {
    const double *A;
    const double *B;
    double *C;
    int64_t lda, ldb, ldc;
    int64_t M, N, K;
    double alpha, beta;
    int tri;  // 0 full tile; 1 / 2: write only the lower / upper triangle (SYRK diagonal tiles)
    const double *C2 = nullptr;  // deferred beta: D += beta2 * C2 (beta2 == 0: C2 not read)
    int64_t ldc2 = 0;
    double beta2 = 0.0;
};

// A batch of independent tile tasks launched as one grid (grouped GEMM); passed by value
// as a __grid_constant__ kernel parameter (32 * 88 + 136 bytes < 4 KB).
constexpr int kMaxBatch = 32;
struct TileBatch {
    int n = 0;
    int cta_start[kMaxBatch + 1] = {};
    TileTask t[kMaxBatch];
};

// TMA variant (dgemm_tma.cu): operands described by tensor maps (128-byte swizzle).
struct TmaTask {
    CUtensorMap mapA, mapB;  // stored A / B tiles (make_tma_operand)
    int a3d = 0, b3d = 0;    // mn-contiguous operand mapped as a 3D tensor: one box per stage
    double *C;
    int64_t ldc, M, N, K;
    double alpha, beta;
    int tri;
    const double *C2;
    int64_t ldc2;
    double beta2;
};
constexpr int kMaxTmaBatch = 16;
struct TmaBatch {
    int n = 0;
    int group_m = 16;  // CTA raster: m-blocks per group (L2 reuse); 0 = column-major raster
    int snake = 1;     // odd groups walk the n-blocks backwards (the B panel at a group boundary is reused)
    int cta_start[kMaxTmaBatch + 1] = {};
    TmaTask t[kMaxTmaBatch];
};
bool make_tma_operand(CUtensorMap *map, const double *X, int64_t rows, int64_t cols, int64_t ld,
                      bool mn_contig, int bmn, int *is3d = nullptr);
int tma_bm();
int tma_bn();
cudaError_t launch_dgemm_tma(bool ta, bool tb, TmaBatch &b, cudaStream_t st);
bool tma_enabled();

// All tasks of a batch share transA / transB (dgemm_tile.cu).
cudaError_t launch_dgemm_batch(bool ta, bool tb, TileBatch &b, cudaStream_t st);
// Single task (batch of one).
cudaError_t launch_dgemm_tile(bool ta, bool tb, int64_t M, int64_t N, int64_t K, double alpha,
                              const double *A, int64_t lda, const double *B, int64_t ldb,
                              double beta, double *C, int64_t ldc, cudaStream_t st);
// C = beta*C (beta == 0: C = 0, C not read).
cudaError_t launch_scale_tile(int64_t M, int64_t N, double beta, double *C, int64_t ldc,
                              cudaStream_t st);
// Diagonal-tile TRSM (solve) / TRMM (multiply) in place on B (trxm_tile.cu):
//   side 'L': B = alpha*op(A)^-1*B or alpha*op(A)*B;  'R': B*op(A)^-1 / B*op(A).
cudaError_t launch_trxm_tile(bool solve, char side, char uplo, char transA, char diag, int64_t M,
                             int64_t N, double alpha, const double *A, int64_t lda, double *B,
                             int64_t ldb, cudaStream_t st);
// The same on up to kMaxBatch B tiles that share the diagonal tile A (order = the extent
// along the triangle; other[q] = tile q's extent along the untouched dimension): one
// recursion whose GEMMs are grouped launches and whose base kernels cover every tile.
cudaError_t launch_trxm_batch(bool solve, char side, char uplo, char transA, char diag, int64_t order,
                              double alpha, const double *A, int64_t lda, int n, double *const *B,
                              const int64_t *ldb, const int64_t *other, cudaStream_t st);
// S = sym(A) (n x n) from the uplo triangle of A.
cudaError_t launch_symm_expand(int64_t n, const double *A, int64_t lda, char uplo, double *S,
                               int64_t lds, cudaStream_t st);
// C = beta*C on the tri triangle only (tri 0: whole tile).
cudaError_t launch_scale_tri(int64_t M, int64_t N, double beta, double *C, int64_t ldc, int tri,
                             cudaStream_t st);
}  // namespace xk
