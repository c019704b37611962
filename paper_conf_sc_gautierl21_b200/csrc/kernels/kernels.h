// kernels.h -- internal launch interface of the sm_100a tile kernels (no torch types).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace xk {
// D = alpha*op(A)*op(B) + beta*C on column-major device tiles (dgemm_tile.cu).
cudaError_t launch_dgemm_tile(bool ta, bool tb, int64_t M, int64_t N, int64_t K, double alpha,
                              const double *A, int64_t lda, const double *B, int64_t ldb,
                              double beta, double *C, int64_t ldc, cudaStream_t st);
// C = beta*C (beta == 0: C = 0, C not read).
cudaError_t launch_scale_tile(int64_t M, int64_t N, double beta, double *C, int64_t ldc,
                              cudaStream_t st);
}  // namespace xk
