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
// One launch covers the vectors of every B tile of a batch (all share the triangle).
struct BaseBatch {
    int n;                            // tiles
    int cta_start[kMaxBatch + 1];     // CTAs per tile: ceil(nvec / NB)
    double *B[kMaxBatch];
    int64_t ldb[kMaxBatch], nvec[kMaxBatch];
};

constexpr int LDM = NB + 2;  // triangle stride in shared memory (16-byte aligned rows)

template <bool SOLVE, bool LOWER, bool LEFT>
__global__ void __launch_bounds__(NB) trxm_base_kernel(const __grid_constant__ BaseBatch bb, int n,
                                                       double alpha, const double *A, int64_t lda,
                                                       bool mtrans, bool unit) {
    extern __shared__ double sm[];
    // SOLVE: Ms[c * LDM + i] = M(i, c) (columns contiguous: column-oriented substitution);
    // multiply: Ms[i * LDM + c] = M(i, c) (rows contiguous: row dot products).  Either way
    // the inner loop reads two consecutive entries with one 16-byte shared load, and every
    // thread of the warp reads the same address (broadcast).
    double *Ms = sm;
    double(*V)[NB + 1] = reinterpret_cast<double(*)[NB + 1]>(sm + NB * LDM);  // V[element][vector]
    double *rd = sm + NB * LDM + NB * (NB + 1);                               // 1 / M(l, l)
    int q = 0;
#pragma unroll 1
    while (q + 1 < bb.n && (int)blockIdx.x >= bb.cta_start[q + 1]) ++q;
    double *B = bb.B[q];
    const int64_t ldb = bb.ldb[q], nvec = bb.nvec[q];
    const int64_t es = LEFT ? 1 : ldb, vs = LEFT ? ldb : 1;
    const int tid = threadIdx.x;
    const int64_t v0 = (int64_t)(blockIdx.x - bb.cta_start[q]) * NB;
    // triangle of M into shared memory, padded to NB with the identity (only the referenced
    // part of A is read).  The kernel is latency-bound, so every load of a phase is issued
    // before the first shared store (fully unrolled, one element per thread per column:
    // coalesced along the stored-contiguous direction of A for either transposition).
    const int nv = (int)((nvec - v0) < NB ? (nvec - v0) : NB);
    {
        double t[NB];
#pragma unroll
        for (int k = 0; k < NB; ++k) {
            const int i = mtrans ? k : tid, c = mtrans ? tid : k;  // M(i, c); A contiguous in tid
            const bool in = LOWER ? (i > c) : (i < c);
            double x = (i == c) ? 1.0 : 0.0;
            if (i < n && c < n && (in || (i == c && !unit))) x = opa(A, lda, mtrans, i, c);
            t[k] = x;
        }
#pragma unroll
        for (int k = 0; k < NB; ++k) {
            const int i = mtrans ? k : tid, c = mtrans ? tid : k;
            Ms[SOLVE ? c * LDM + i : i * LDM + c] = t[k];
            if (SOLVE && i == c) rd[i] = 1.0 / t[k];
        }
        // vectors of this CTA (coalesced along the contiguous direction of B), zero-padded
#pragma unroll
        for (int k = 0; k < NB; ++k) {
            if (LEFT) {  // element e = tid of vector k
                t[k] = (tid < n && k < nv) ? B[tid + (v0 + k) * vs] : 0.0;
            } else {     // vector tid, element k
                t[k] = (k < n && tid < nv) ? B[(v0 + tid) * vs + k * es] : 0.0;
            }
        }
#pragma unroll
        for (int k = 0; k < NB; ++k) {
            if (LEFT) V[tid][k] = t[k];
            else V[k][tid] = t[k];
        }
    }
    __syncthreads();
    {
        // one vector per thread, held in registers; every loop is fully unrolled so the
        // indices are compile-time and independent updates interleave (ILP)
        const int v = tid;
        double x[NB];
#pragma unroll
        for (int i = 0; i < NB; ++i) x[i] = V[i][v];
        if (SOLVE) {
#pragma unroll
            for (int i = 0; i < NB; ++i) x[i] *= alpha;
            if (LOWER) {  // column-oriented forward substitution: x_i -= M_il x_l, l ascending
#pragma unroll
                for (int l = 0; l < NB; ++l) {
                    if (!unit) x[l] *= rd[l];
                    const double2 *col = reinterpret_cast<const double2 *>(Ms + l * LDM);
#pragma unroll
                    for (int p = (l + 1) / 2; p < NB / 2; ++p) {
                        const double2 m2 = col[p];
                        if (2 * p > l) x[2 * p] -= m2.x * x[l];
                        x[2 * p + 1] -= m2.y * x[l];
                    }
                }
            } else {      // back substitution, l descending
#pragma unroll
                for (int l = NB - 1; l >= 0; --l) {
                    if (!unit) x[l] *= rd[l];
                    const double2 *col = reinterpret_cast<const double2 *>(Ms + l * LDM);
#pragma unroll
                    for (int p = 0; 2 * p < l; ++p) {
                        const double2 m2 = col[p];
                        x[2 * p] -= m2.x * x[l];
                        if (2 * p + 1 < l) x[2 * p + 1] -= m2.y * x[l];
                    }
                }
            }
        } else {
            if (LOWER) {  // bottom-up: row i only reads x_0..x_i, still unmodified
#pragma unroll
                for (int i = NB - 1; i >= 0; --i) {
                    const double2 *row = reinterpret_cast<const double2 *>(Ms + i * LDM);
                    double s = 0.0;
#pragma unroll
                    for (int p = 0; 2 * p <= i; ++p) {
                        const double2 m2 = row[p];
                        s += m2.x * x[2 * p];
                        if (2 * p + 1 <= i) s += m2.y * x[2 * p + 1];
                    }
                    x[i] = alpha * s;
                }
            } else {      // top-down: row i only reads x_i..x_NB-1, still unmodified
#pragma unroll
                for (int i = 0; i < NB; ++i) {
                    const double2 *row = reinterpret_cast<const double2 *>(Ms + i * LDM);
                    double s = 0.0;
#pragma unroll
                    for (int p = i / 2; p < NB / 2; ++p) {
                        const double2 m2 = row[p];
                        if (2 * p >= i) s += m2.x * x[2 * p];
                        s += m2.y * x[2 * p + 1];
                    }
                    x[i] = alpha * s;
                }
            }
        }
#pragma unroll
        for (int i = 0; i < NB; ++i) V[i][v] = x[i];
    }
    __syncthreads();
    if (LEFT) {
#pragma unroll 16
        for (int r = tid; r < n * nv; r += NB) {
            int e = r % n, v = r / n;
            B[e + (v0 + v) * vs] = V[e][v];
        }
    } else {
#pragma unroll 16
        for (int r = tid; r < n * nv; r += NB) {
            int v = r % nv, e = r / nv;
            B[(v0 + v) * vs + e * es] = V[e][v];
        }
    }
}

struct TriOp {
    bool solve, left, elow, trans, unit;
};

// The B tiles of one diagonal op: all share the triangle (order n along the triangular
// dimension); `other` is each tile's extent along the untouched dimension.
struct Tiles {
    int n = 0;
    double *B[kMaxBatch];
    int64_t ldb[kMaxBatch], other[kMaxBatch];
};

// op(A) block (rows R0.., cols C0..) as a GEMM operand: pointer + transposition
inline const double *opa_block(const double *A, int64_t lda, bool trans, int64_t r0, int64_t c0,
                               bool *t) {
    *t = trans;
    return trans ? A + c0 + r0 * lda : A + r0 + c0 * lda;
}

template <bool SOLVE, bool LOWER, bool LEFT>
cudaError_t base_launch(const BaseBatch &bb, unsigned grid, int n, double alpha, const double *A,
                        int64_t lda, bool mtrans, bool unit, cudaStream_t st) {
    constexpr size_t smem = (NB * LDM + NB * (NB + 1) + NB) * sizeof(double);
    auto kern = trxm_base_kernel<SOLVE, LOWER, LEFT>;
    static unsigned attr_set = 0;  // per instantiation, one bit per device
    int dev = 0;
    cudaGetDevice(&dev);
    if (!(attr_set & (1u << dev))) {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
        attr_set |= 1u << dev;
    }
    kern<<<grid, NB, smem, st>>>(bb, n, alpha, A, lda, mtrans, unit);
    return cudaGetLastError();
}

cudaError_t base(const TriOp &o, int64_t n, const Tiles &T, double alpha, const double *A, int64_t lda,
                 cudaStream_t st) {
    BaseBatch bb;
    bb.n = T.n;
    int total = 0;
    for (int q = 0; q < T.n; ++q) {
        bb.cta_start[q] = total;
        bb.B[q] = T.B[q];
        bb.ldb[q] = T.ldb[q];
        bb.nvec[q] = T.other[q];
        total += (int)((T.other[q] + NB - 1) / NB);
    }
    bb.cta_start[T.n] = total;
    if (total == 0) return cudaSuccess;
    // right side: the matrix acting on row vectors is op(A)^T
    const bool mtrans = o.left ? o.trans : !o.trans;
    const bool mlow = o.left ? o.elow : !o.elow;
    const int ni = (int)n;
#define XK_BASE(S, L, LE) return base_launch<S, L, LE>(bb, (unsigned)total, ni, alpha, A, lda, mtrans, o.unit, st)
    if (o.solve) {
        if (mlow) { if (o.left) XK_BASE(true, true, true); else XK_BASE(true, true, false); }
        else { if (o.left) XK_BASE(true, false, true); else XK_BASE(true, false, false); }
    } else {
        if (mlow) { if (o.left) XK_BASE(false, true, true); else XK_BASE(false, true, false); }
        else { if (o.left) XK_BASE(false, false, true); else XK_BASE(false, false, false); }
    }
#undef XK_BASE
}

// Sub-tiles of every tile: the first n1 (half 1) or the rest (half 2) along the triangle.
Tiles half(const Tiles &T, bool left, int64_t off) {
    Tiles H = T;
    for (int q = 0; q < T.n; ++q) H.B[q] = left ? T.B[q] + off : T.B[q] + off * T.ldb[q];
    return H;
}

// One grouped GEMM over the tiles: left  Y = a*opA(blk)*X + b*Y  (Y, X sub-tiles)
//                                   right Y = a*X*opA(blk) + b*Y
cudaError_t gemm_all(const TriOp &o, const Tiles &X, const Tiles &Y, const double *P, bool t, int64_t lda,
                     int64_t ny, int64_t nk, double a, double b, cudaStream_t st) {
    TileBatch tb;
    tb.n = X.n;
    for (int q = 0; q < X.n; ++q) {
        if (o.left)
            tb.t[q] = TileTask{P, X.B[q], Y.B[q], lda, X.ldb[q], Y.ldb[q], ny, X.other[q], nk, a, b, 0, nullptr, 0, 0.0};
        else
            tb.t[q] = TileTask{X.B[q], P, Y.B[q], X.ldb[q], lda, Y.ldb[q], X.other[q], ny, nk, a, b, 0, nullptr, 0, 0.0};
    }
    return o.left ? launch_dgemm_batch(t, false, tb, st) : launch_dgemm_batch(false, t, tb, st);
}

cudaError_t rec(const TriOp &o, int64_t n, const Tiles &T, double alpha, const double *A, int64_t lda,
                cudaStream_t st) {
    if (n <= NB) return base(o, n, T, alpha, A, lda, st);
    const int64_t n1 = ((n / 2 + NB - 1) / NB) * NB, n2 = n - n1;
    const double *A11 = A, *A22 = A + n1 + n1 * lda;
    const Tiles B1 = half(T, o.left, 0), B2 = half(T, o.left, n1);
    bool t;
    cudaError_t e;
    // blocks of op(A): (1,2) = rows 0..n1, cols n1..; (2,1) = rows n1.., cols 0..n1
    const double *P21 = opa_block(A, lda, o.trans, n1, 0, &t);
    const double *P12 = opa_block(A, lda, o.trans, 0, n1, &t);
    // left: Y = op(A)_yx X ; right: Y = X op(A)_xy.  Coupling block for "1 then 2" is
    // (2,1) on the left and (1,2) on the right, and the reverse for "2 then 1".
    if (o.solve) {
        // solve first the block op(A) maps without coupling:
        //   left & elow, right & upper: block 1 first; otherwise block 2 first.
        if (o.left == o.elow) {
            if ((e = rec(o, n1, B1, alpha, A11, lda, st))) return e;
            if ((e = gemm_all(o, B1, B2, o.left ? P21 : P12, t, lda, n2, n1, -1.0, alpha, st))) return e;
            return rec(o, n2, B2, 1.0, A22, lda, st);
        }
        if ((e = rec(o, n2, B2, alpha, A22, lda, st))) return e;
        if ((e = gemm_all(o, B2, B1, o.left ? P12 : P21, t, lda, n1, n2, -1.0, alpha, st))) return e;
        return rec(o, n1, B1, 1.0, A11, lda, st);
    }
    // TRMM (in place): update the block whose inputs must stay old last
    //   left & elow : B2 <- a A22 B2 ; B2 += a A21 B1 ; B1 <- a A11 B1
    //   left & eup  : B1 <- a A11 B1 ; B1 += a A12 B2 ; B2 <- a A22 B2
    //   right & elow: B1 <- a B1 A11 ; B1 += a B2 A21 ; B2 <- a B2 A22
    //   right & eup : B2 <- a B2 A22 ; B2 += a B1 A12 ; B1 <- a B1 A11
    if (o.left == o.elow) {
        if ((e = rec(o, n2, B2, alpha, A22, lda, st))) return e;
        if ((e = gemm_all(o, B1, B2, o.left ? P21 : P12, t, lda, n2, n1, alpha, 1.0, st))) return e;
        return rec(o, n1, B1, alpha, A11, lda, st);
    }
    if ((e = rec(o, n1, B1, alpha, A11, lda, st))) return e;
    if ((e = gemm_all(o, B2, B1, o.left ? P12 : P21, t, lda, n1, n2, alpha, 1.0, st))) return e;
    return rec(o, n2, B2, alpha, A22, lda, st);
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

static TriOp make_op(bool solve, char side, char uplo, char transA, char diag) {
    TriOp o;
    o.solve = solve;
    o.left = (side == 'L' || side == 'l');
    o.trans = (transA == 'T' || transA == 't' || transA == 'C' || transA == 'c');
    o.elow = ((uplo == 'L' || uplo == 'l') != o.trans);
    o.unit = (diag == 'U' || diag == 'u');
    return o;
}

cudaError_t launch_trxm_tile(bool solve, char side, char uplo, char transA, char diag, int64_t M,
                             int64_t N, double alpha, const double *A, int64_t lda, double *B,
                             int64_t ldb, cudaStream_t st) {
    if (M <= 0 || N <= 0) return cudaSuccess;
    TriOp o = make_op(solve, side, uplo, transA, diag);
    Tiles T;
    T.n = 1;
    T.B[0] = B;
    T.ldb[0] = ldb;
    T.other[0] = o.left ? N : M;
    return rec(o, o.left ? M : N, T, alpha, A, lda, st);
}

cudaError_t launch_trxm_batch(bool solve, char side, char uplo, char transA, char diag, int64_t order,
                              double alpha, const double *A, int64_t lda, int n, double *const *B,
                              const int64_t *ldb, const int64_t *other, cudaStream_t st) {
    if (order <= 0 || n <= 0) return cudaSuccess;
    TriOp o = make_op(solve, side, uplo, transA, diag);
    Tiles T;
    T.n = n;
    for (int q = 0; q < n; ++q) {
        T.B[q] = B[q];
        T.ldb[q] = ldb[q];
        T.other[q] = other[q];
    }
    return rec(o, order, T, alpha, A, lda, st);
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
