// trxm_tile.cu -- diagonal-tile kernels of the BLAS-3 tile algorithms (SURVEY.md §8(f),
// K2-K5): triangular solve / multiply of one B tile by a diagonal tile of A (TRSM/TRMM),
// the symmetric expansion of a SYMM diagonal tile, and the triangle-masked C = beta*C.
//
// TRSM/TRMM tile (PLASMA's dtrsm/dtrmm on a tile): recursive blocking on the
// order of the triangular matrix -- the two half-size triangles recurse, the off-diagonal
// block is one GEMM on the sm_100a DMMA tile kernel (dgemm_tile.cu), and below 64 a base
// kernel solves (or multiplies) one vector per thread against the small triangle held in
// shared memory.  Recursive blocking keeps the substitution backward stable (no explicit
// inverse), so the componentwise residual bound of DESIGN.md reading Q13 holds.
//
// Only the triangle op(A) references is read; with diag == 'U' the diagonal is not read.
#include <cuda_runtime.h>
#include <stdint.h>

#include "kernels/kernels.h"

namespace xk {
namespace {

constexpr int NB = 64;  // base-case order

// op(A)(r, c) of a diagonal tile stored at A (column-major, ld), trans = op is A^T
__device__ __forceinline__ double opa(const double *A, int64_t lda, bool trans, int r, int c) {
    return trans ? A[c + (int64_t)r * lda] : A[r + (int64_t)c * lda];
}

// One thread per vector.  The system (or product) is on vectors v of length n (n <= NB):
//   left  side: v = a column of B (element stride 1, vectors ldb apart), matrix M = op(A)
//   right side: v = a row of B (element stride ldb, vectors 1 apart),   matrix M = op(A)^T
// LOWER: M is lower triangular (forward substitution / bottom-up product).
template <bool SOLVE, bool LOWER>
__global__ void __launch_bounds__(NB) trxm_base_kernel(int n, int64_t nvec, double alpha,
                                                       const double *A, int64_t lda, bool mtrans,
                                                       bool unit, double *B, int64_t es,
                                                       int64_t vs) {
    extern __shared__ double sm[];
    double(*Ms)[NB + 1] = reinterpret_cast<double(*)[NB + 1]>(sm);
    double(*V)[NB + 1] = reinterpret_cast<double(*)[NB + 1]>(sm + NB * (NB + 1));  // V[element][vector]
    const int tid = threadIdx.x;
    const int64_t v0 = (int64_t)blockIdx.x * NB;
    // triangle of M into shared memory (only the referenced part is read)
    for (int q = tid; q < n * n; q += NB) {
        int r = q % n, c = q / n;
        bool in = LOWER ? (r > c) : (r < c);
        double x = 0.0;
        if (in) x = opa(A, lda, mtrans, r, c);
        else if (r == c) x = unit ? 1.0 : opa(A, lda, mtrans, r, c);
        Ms[r][c] = x;
    }
    // vectors of this CTA (coalesced along the contiguous direction)
    const int nv = (int)((nvec - v0) < NB ? (nvec - v0) : NB);
    if (es == 1) {
        for (int q = tid; q < n * nv; q += NB) {
            int e = q % n, v = q / n;
            V[e][v] = B[e + (v0 + v) * vs];
        }
    } else {
        for (int q = tid; q < n * nv; q += NB) {
            int v = q % nv, e = q / nv;
            V[e][v] = B[(v0 + v) * vs + e * es];
        }
    }
    __syncthreads();
    if (tid < nv) {
        const int v = tid;
        if (SOLVE) {
            if (LOWER) {
                for (int i = 0; i < n; ++i) {
                    double s = alpha * V[i][v];
                    for (int l = 0; l < i; ++l) s -= Ms[i][l] * V[l][v];
                    V[i][v] = unit ? s : s / Ms[i][i];
                }
            } else {
                for (int i = n - 1; i >= 0; --i) {
                    double s = alpha * V[i][v];
                    for (int l = i + 1; l < n; ++l) s -= Ms[i][l] * V[l][v];
                    V[i][v] = unit ? s : s / Ms[i][i];
                }
            }
        } else {
            if (LOWER) {  // bottom-up keeps the inputs of later rows intact
                for (int i = n - 1; i >= 0; --i) {
                    double s = 0.0;
                    for (int l = 0; l <= i; ++l) s += Ms[i][l] * V[l][v];
                    V[i][v] = alpha * s;
                }
            } else {
                for (int i = 0; i < n; ++i) {
                    double s = 0.0;
                    for (int l = i; l < n; ++l) s += Ms[i][l] * V[l][v];
                    V[i][v] = alpha * s;
                }
            }
        }
    }
    __syncthreads();
    if (es == 1) {
        for (int q = tid; q < n * nv; q += NB) {
            int e = q % n, v = q / n;
            B[e + (v0 + v) * vs] = V[e][v];
        }
    } else {
        for (int q = tid; q < n * nv; q += NB) {
            int v = q % nv, e = q / nv;
            B[(v0 + v) * vs + e * es] = V[e][v];
        }
    }
}

struct TriOp {
    bool solve, left, elow, trans, unit;
};

// op(A) block (rows R0.., cols C0..) as a GEMM operand: pointer + transposition
inline const double *opa_block(const double *A, int64_t lda, bool trans, int64_t r0, int64_t c0,
                               bool *t) {
    *t = trans;
    return trans ? A + c0 + r0 * lda : A + r0 + c0 * lda;
}

cudaError_t base(const TriOp &o, int64_t M, int64_t N, double alpha, const double *A, int64_t lda,
                 double *B, int64_t ldb, cudaStream_t st) {
    const int n = (int)(o.left ? M : N);
    const int64_t nvec = o.left ? N : M;
    const int64_t es = o.left ? 1 : ldb, vs = o.left ? ldb : 1;
    // right side: the matrix acting on row vectors is op(A)^T
    const bool mtrans = o.left ? o.trans : !o.trans;
    const bool mlow = o.left ? o.elow : !o.elow;
    const unsigned grid = (unsigned)((nvec + NB - 1) / NB);
    constexpr size_t smem = 2 * NB * (NB + 1) * sizeof(double);
    static unsigned attr_set = 0;  // one bit per device
    int dev = 0;
    cudaGetDevice(&dev);
    if (!(attr_set & (1u << dev))) {
        cudaError_t e;
        if ((e = cudaFuncSetAttribute(trxm_base_kernel<true, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem))) return e;
        if ((e = cudaFuncSetAttribute(trxm_base_kernel<true, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem))) return e;
        if ((e = cudaFuncSetAttribute(trxm_base_kernel<false, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem))) return e;
        if ((e = cudaFuncSetAttribute(trxm_base_kernel<false, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem))) return e;
        attr_set |= 1u << dev;
    }
    if (o.solve) {
        if (mlow) trxm_base_kernel<true, true><<<grid, NB, smem, st>>>(n, nvec, alpha, A, lda, mtrans, o.unit, B, es, vs);
        else trxm_base_kernel<true, false><<<grid, NB, smem, st>>>(n, nvec, alpha, A, lda, mtrans, o.unit, B, es, vs);
    } else {
        if (mlow) trxm_base_kernel<false, true><<<grid, NB, smem, st>>>(n, nvec, alpha, A, lda, mtrans, o.unit, B, es, vs);
        else trxm_base_kernel<false, false><<<grid, NB, smem, st>>>(n, nvec, alpha, A, lda, mtrans, o.unit, B, es, vs);
    }
    return cudaGetLastError();
}

cudaError_t rec(const TriOp &o, int64_t M, int64_t N, double alpha, const double *A, int64_t lda,
                double *B, int64_t ldb, cudaStream_t st) {
    const int64_t n = o.left ? M : N;
    if (n <= NB) return base(o, M, N, alpha, A, lda, B, ldb, st);
    const int64_t n1 = ((n / 2 + NB - 1) / NB) * NB, n2 = n - n1;
    const double *A11 = A, *A22 = A + n1 + n1 * lda;
    // B halves along the triangular dimension
    double *B1 = B, *B2 = o.left ? B + n1 : B + n1 * ldb;
    const int64_t M1 = o.left ? n1 : M, M2 = o.left ? n2 : M;
    const int64_t N1 = o.left ? N : n1, N2 = o.left ? N : n2;
    bool t;
    cudaError_t e;
    // For the solve the first block solved is the one op(A) maps without coupling:
    //   left & elow, right & upper: block 1 first; otherwise block 2 first.
    const bool first1 = (o.left == o.elow);
    if (o.solve) {
        if (first1) {
            if ((e = rec(o, M1, N1, alpha, A11, lda, B1, ldb, st))) return e;
            if (o.left) {  // B2 = -op(A)21 X1 + alpha B2
                const double *P = opa_block(A, lda, o.trans, n1, 0, &t);
                e = launch_dgemm_tile(t, false, n2, N, n1, -1.0, P, lda, B1, ldb, alpha, B2, ldb, st);
            } else {       // B2 = -X1 op(A)12 + alpha B2
                const double *P = opa_block(A, lda, o.trans, 0, n1, &t);
                e = launch_dgemm_tile(false, t, M, n2, n1, -1.0, B1, ldb, P, lda, alpha, B2, ldb, st);
            }
            if (e) return e;
            return rec(o, M2, N2, 1.0, A22, lda, B2, ldb, st);
        }
        if ((e = rec(o, M2, N2, alpha, A22, lda, B2, ldb, st))) return e;
        if (o.left) {      // B1 = -op(A)12 X2 + alpha B1
            const double *P = opa_block(A, lda, o.trans, 0, n1, &t);
            e = launch_dgemm_tile(t, false, n1, N, n2, -1.0, P, lda, B2, ldb, alpha, B1, ldb, st);
        } else {           // B1 = -X2 op(A)21 + alpha B1
            const double *P = opa_block(A, lda, o.trans, n1, 0, &t);
            e = launch_dgemm_tile(false, t, M, n1, n2, -1.0, B2, ldb, P, lda, alpha, B1, ldb, st);
        }
        if (e) return e;
        return rec(o, M1, N1, 1.0, A11, lda, B1, ldb, st);
    }
    // TRMM (in place): update the block whose inputs must stay old last
    //   left & elow : B2 <- a A22 B2 ; B2 += a A21 B1 ; B1 <- a A11 B1
    //   left & eup  : B1 <- a A11 B1 ; B1 += a A12 B2 ; B2 <- a A22 B2
    //   right & elow: B1 <- a B1 A11 ; B1 += a B2 A21 ; B2 <- a B2 A22
    //   right & eup : B2 <- a B2 A22 ; B2 += a B1 A12 ; B1 <- a B1 A11
    const bool two_first = (o.left == o.elow);
    if (two_first) {
        if ((e = rec(o, M2, N2, alpha, A22, lda, B2, ldb, st))) return e;
        if (o.left) {
            const double *P = opa_block(A, lda, o.trans, n1, 0, &t);
            e = launch_dgemm_tile(t, false, n2, N, n1, alpha, P, lda, B1, ldb, 1.0, B2, ldb, st);
        } else {
            const double *P = opa_block(A, lda, o.trans, 0, n1, &t);
            e = launch_dgemm_tile(false, t, M, n2, n1, alpha, B1, ldb, P, lda, 1.0, B2, ldb, st);
        }
        if (e) return e;
        return rec(o, M1, N1, alpha, A11, lda, B1, ldb, st);
    }
    if ((e = rec(o, M1, N1, alpha, A11, lda, B1, ldb, st))) return e;
    if (o.left) {
        const double *P = opa_block(A, lda, o.trans, 0, n1, &t);
        e = launch_dgemm_tile(t, false, n1, N, n2, alpha, P, lda, B2, ldb, 1.0, B1, ldb, st);
    } else {
        const double *P = opa_block(A, lda, o.trans, n1, 0, &t);
        e = launch_dgemm_tile(false, t, M, n1, n2, alpha, B2, ldb, P, lda, 1.0, B1, ldb, st);
    }
    if (e) return e;
    return rec(o, M2, N2, alpha, A22, lda, B2, ldb, st);
}

__global__ void symm_expand_kernel(int64_t n, const double *A, int64_t lda, bool lower, double *S,
                                   int64_t lds) {
    for (int64_t q = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; q < n * n;
         q += (int64_t)gridDim.x * blockDim.x) {
        int64_t r = q % n, c = q / n;
        bool in = lower ? (r >= c) : (r <= c);
        S[r + c * lds] = in ? A[r + c * lda] : A[c + r * lda];
    }
}

__global__ void scale_tri_kernel(int64_t M, int64_t N, double beta, double *C, int64_t ldc, int tri) {
    for (int64_t q = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; q < M * N;
         q += (int64_t)gridDim.x * blockDim.x) {
        int64_t r = q % M, c = q / M;
        if (tri == 1 && r < c) continue;
        if (tri == 2 && r > c) continue;
        double *p = C + r + c * ldc;
        *p = (beta == 0.0) ? 0.0 : beta * *p;
    }
}

}  // namespace

cudaError_t launch_trxm_tile(bool solve, char side, char uplo, char transA, char diag, int64_t M,
                             int64_t N, double alpha, const double *A, int64_t lda, double *B,
                             int64_t ldb, cudaStream_t st) {
    if (M <= 0 || N <= 0) return cudaSuccess;
    TriOp o;
    o.solve = solve;
    o.left = (side == 'L' || side == 'l');
    o.trans = (transA == 'T' || transA == 't' || transA == 'C' || transA == 'c');
    o.elow = ((uplo == 'L' || uplo == 'l') != o.trans);
    o.unit = (diag == 'U' || diag == 'u');
    return rec(o, M, N, alpha, A, lda, B, ldb, st);
}

cudaError_t launch_symm_expand(int64_t n, const double *A, int64_t lda, char uplo, double *S,
                               int64_t lds, cudaStream_t st) {
    if (n <= 0) return cudaSuccess;
    int blocks = (int)((n * n + 255) / 256);
    if (blocks > 148 * 8) blocks = 148 * 8;
    symm_expand_kernel<<<blocks, 256, 0, st>>>(n, A, lda, uplo == 'L' || uplo == 'l', S, lds);
    return cudaGetLastError();
}

cudaError_t launch_scale_tri(int64_t M, int64_t N, double beta, double *C, int64_t ldc, int tri,
                             cudaStream_t st) {
    if (M <= 0 || N <= 0 || beta == 1.0) return cudaSuccess;
    int blocks = (int)((M * N + 255) / 256);
    if (blocks > 148 * 8) blocks = 148 * 8;
    scale_tri_kernel<<<blocks, 256, 0, st>>>(M, N, beta, C, ldc, tri);
    return cudaGetLastError();
}

}  // namespace xk
