// trxm_tile.cu -- diagonal-tile kernels of the BLAS-3 tile algorithms (SURVEY.md §8(f),
// K2-K5): triangular solve / multiply of one B tile by a diagonal tile of A (TRSM/TRMM),
// the symmetric expansion of a SYMM diagonal tile, and the triangle-masked C = beta*C.
//
// TRSM/TRMM tile (PLASMA's dtrsm/dtrmm on a tile): recursive blocking on the
// order of the triangular matrix -- the two half-size triangles recurse, the off-diagonal
// block is one GEMM on the sm_100a DMMA tile kernel (dgemm_tile.cu), and below 64 a base
// kernel solves (or multiplies) one vector per thread, held in registers, against the small
// triangle held in shared memory (128 vectors per CTA share one triangle load).  Recursive blocking keeps the substitution backward stable (no explicit
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
#ifndef XK_VPC
#define XK_VPC 128
#endif
constexpr int VPC = XK_VPC;  // vectors (threads) per CTA: the triangle load is shared by all
static_assert(VPC % 32 == 0 && (NB * NB) % VPC == 0, "VPC: whole warps, triangle split evenly");
struct BaseBatch {
    int n;                            // tiles
    int cta_start[kMaxBatch + 1];     // CTAs per tile: ceil(nvec / VPC)
    double *B[kMaxBatch];
    int64_t ldb[kMaxBatch], nvec[kMaxBatch];
};

constexpr int LDM = NB + 2;  // triangle stride in shared memory (16-byte aligned rows)

constexpr int LDV = NB + 2;  // staged vector stride (left side): 16-byte rows, odd in 16-byte units
constexpr size_t kBaseSmemLeft = (size_t)(NB * LDM + NB + VPC * LDV) * sizeof(double);

template <bool SOLVE, bool LOWER, bool LEFT>
__global__ void __launch_bounds__(VPC) trxm_base_kernel(const __grid_constant__ BaseBatch bb, int n,
                                                        double alpha, const double *A, int64_t lda,
                                                        bool mtrans, bool unit) {
    // SOLVE: Ms[c * LDM + i] = M(i, c) (columns contiguous: column-oriented substitution);
    // multiply: Ms[i * LDM + c] = M(i, c) (rows contiguous: row dot products).  Either way
    // the inner loop reads two consecutive entries with one 16-byte shared load, and every
    // thread of the warp reads the same address (broadcast).
    extern __shared__ __align__(16) double smem_base[];
    double *Ms = smem_base;
    double *rd = Ms + NB * LDM;  // 1 / M(l, l)
    double *V = rd + NB;         // left side: the CTA's vectors, V[v * LDV + e]
    int q = 0;
#pragma unroll 1
    while (q + 1 < bb.n && (int)blockIdx.x >= bb.cta_start[q + 1]) ++q;
    double *B = bb.B[q];
    const int64_t ldb = bb.ldb[q], nvec = bb.nvec[q];
    const int tid = threadIdx.x;
    const int64_t v0 = (int64_t)(blockIdx.x - bb.cta_start[q]) * VPC;
    const int nv = (int)((nvec - v0) < VPC ? (nvec - v0) : VPC);
    // triangle of M into shared memory, padded to NB with the identity (only the referenced
    // part of A is read); consecutive threads read along the stored-contiguous direction,
    // every load in flight before the first shared store (latency-bound phase)
    {
        double t[NB * NB / VPC];
#pragma unroll
        for (int k = 0; k < NB * NB / VPC; ++k) {
            const int e = tid + k * VPC, f = e % NB, s2 = e / NB;
            const int i = mtrans ? s2 : f, c = mtrans ? f : s2;  // M(i, c); A contiguous in f
            const bool in = LOWER ? (i > c) : (i < c);
            double v = (i == c) ? 1.0 : 0.0;
            if (i < n && c < n && (in || (i == c && !unit))) v = opa(A, lda, mtrans, i, c);
            t[k] = v;
        }
#pragma unroll
        for (int k = 0; k < NB * NB / VPC; ++k) {
            const int e = tid + k * VPC, f = e % NB, s2 = e / NB;
            const int i = mtrans ? s2 : f, c = mtrans ? f : s2;
            Ms[SOLVE ? c * LDM + i : i * LDM + c] = t[k];
            if (SOLVE && i == c) rd[i] = 1.0 / t[k];
        }
    }
    double x[NB];
    if (LEFT) {
        // vectors are columns of B (contiguous): a warp loads whole columns, 16 bytes per
        // lane (fully coalesced), into the staging area; each thread then takes its own
        const int w = tid >> 5, lane = tid & 31;
        double2 u[32];  // VPC / 32 warps x 32 columns each = VPC vectors
#pragma unroll
        for (int k = 0; k < 32; ++k) {
            const int v = w * 32 + k, e = 2 * lane;
            double2 z = make_double2(0.0, 0.0);
            if (v < nv && e < n) {
                const double *src = B + (v0 + v) * ldb + e;
                if (e + 1 < n) z = *reinterpret_cast<const double2 *>(src);
                else z.x = src[0];
            }
            u[k] = z;
        }
#pragma unroll
        for (int k = 0; k < 32; ++k) {
            const int v = w * 32 + k;
            *reinterpret_cast<double2 *>(V + v * LDV + 2 * lane) = u[k];
        }
        __syncthreads();
#pragma unroll
        for (int p = 0; p < NB / 2; ++p) {
            const double2 z = *reinterpret_cast<const double2 *>(V + tid * LDV + 2 * p);
            x[2 * p] = z.x;
            x[2 * p + 1] = z.y;
        }
    } else {
        // vectors are rows of B: consecutive threads read consecutive addresses
        const bool active = tid < nv;
        const double *p = B + (v0 + tid);
#pragma unroll
        for (int i = 0; i < NB; ++i, p += ldb) x[i] = (active && i < n) ? *p : 0.0;
    }
    __syncthreads();
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
    if (LEFT) {
        // back through the staging area so that every warp stores whole columns
#pragma unroll
        for (int p = 0; p < NB / 2; ++p)
            *reinterpret_cast<double2 *>(V + tid * LDV + 2 * p) = make_double2(x[2 * p], x[2 * p + 1]);
        __syncthreads();
        const int w = tid >> 5, lane = tid & 31;
#pragma unroll
        for (int k = 0; k < 32; ++k) {
            const int v = w * 32 + k, e = 2 * lane;
            if (v < nv && e < n) {
                const double2 z = *reinterpret_cast<const double2 *>(V + v * LDV + e);
                double *dst = B + (v0 + v) * ldb + e;
                if (e + 1 < n) *reinterpret_cast<double2 *>(dst) = z;
                else dst[0] = z.x;
            }
        }
    } else if (tid < nv) {
        double *p = B + (v0 + tid);
        asm volatile("mov.b64 %0, %0;" : "+l"(p));  // opaque: no CSE with the load addresses
#pragma unroll
        for (int i = 0; i < NB; ++i, p += ldb)
            if (i < n) *p = x[i];
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
    auto kern = trxm_base_kernel<SOLVE, LOWER, LEFT>;
    const size_t smem = LEFT ? kBaseSmemLeft : (size_t)(NB * LDM + NB) * sizeof(double);
    static unsigned attr_set = 0;  // per instantiation, one bit per device
    int dev = 0;
    cudaGetDevice(&dev);
    if (!(attr_set & (1u << dev))) {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kBaseSmemLeft);
        if (e != cudaSuccess) return e;
        attr_set |= 1u << dev;
    }
    kern<<<grid, VPC, smem, st>>>(bb, n, alpha, A, lda, mtrans, unit);
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
        total += (int)((T.other[q] + VPC - 1) / VPC);
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
