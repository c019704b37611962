// trxm_tile.cu -- diagonal-tile kernels of the BLAS-3 tile algorithms (SURVEY.md §8(f),
// K2-K5): triangular solve / multiply of one B tile by a diagonal tile of A (TRSM/TRMM),
// the symmetric expansion of a SYMM diagonal tile, and the triangle-masked C = beta*C.
//
// TRSM/TRMM tile (PLASMA's dtrsm/dtrmm on a tile): recursive blocking on the
// order of the triangular matrix -- the two half-size triangles recurse, the off-diagonal
// block is one GEMM on the sm_100a DMMA tile kernel (dgemm_tile.cu), and at order <= 64 a
// base kernel works on 64 vectors per CTA staged in shared memory next to the triangle:
// 16 x 16 diagonal blocks one thread per vector, the updates between blocks on DMMA (see
// trxm_base_kernel).  Blocking keeps the substitution backward stable (no explicit inverse),
// so the componentwise residual bound of DESIGN.md reading Q13 holds.
//
// Only the triangle op(A) references is read; with diag == 'U' the diagonal is not read.
#include <cuda_runtime.h>
#include <stdint.h>

#include "kernels/kernels.h"

namespace xk {
namespace {

constexpr int NB = 64;  // base-case order


// Base case (order n <= NB = 64) on the vectors of every B tile of a batch (all share the
// triangle): left side, the vectors are the columns of B and the matrix is M = op(A); right
// side, the vectors are the rows of B and M = op(A)^T.  A CTA takes NVB = 64 vectors (2 NVB
// threads) and stages them in shared memory as X (one vector per padded row), next to M.  The
// triangle is processed in diagonal blocks of BS = 16:
//   TRSM (lower, forward): for each block kb in order, one thread per vector solves the
//     16 x 16 diagonal block against its 16 entries (reciprocal diagonal, no inverse of the
//     triangle), then the 4 warps update the rows below with the solved block on the FP64
//     tensor path: X(rows > kb, :) -= M(rows > kb, kb) X(kb, :), 8 x 8 output tiles of
//     mma.sync.m8n8k4.f64 (DMMA), 4 k-steps each.  Upper: the mirror image, blocks backward.
//   TRMM (lower, bottom-up): for each block kb from the last, one thread per vector forms
//     M(kb, kb) X(kb) in place (rows bottom-up), then the warps add M(kb, < kb) X(< kb, :) --
//     blocks < kb are still unmodified.  Upper: top-down, adding M(kb, > kb) X(> kb, :).
// Straight-line code stays small (the old one-vector-per-thread substitution over all 64
// rows was ~3k instructions and instruction-fetch bound, profiles/r01_trsm_base_v2_ncu.txt).
// Blocked substitution with GEMM updates is the standard backward-stable form; it is the
// same algorithm the recursion above applies at larger orders (Q13 bounds hold).
#ifndef XK_NVB
#define XK_NVB 64
#endif
#ifndef XK_BS
#define XK_BS 16
#endif
constexpr int BS = XK_BS;   // diagonal block of the base case
constexpr int NVB = XK_NVB; // vectors per CTA
constexpr int BT = 2 * NVB; // threads per CTA
constexpr int NW = BT / 32; // warps per CTA
constexpr int LDM = 68;   // M stride in doubles: 68 = 4 mod 16 -> conflict-free DMMA A fragments
constexpr int LDV = 68;   // X stride per vector: conflict-free DMMA B fragments
static_assert(NB % BS == 0 && BS % 8 == 0 && NVB % 8 == 0 && NVB <= BT, "base-case blocking");
struct BaseBatch {
    int n;                            // tiles
    int cta_start[kMaxBatch + 1];     // CTAs per tile: ceil(nvec / NVB)
    double *B[kMaxBatch];
    int64_t ldb[kMaxBatch], nvec[kMaxBatch];
    bool al16;                        // every B and ldb 16-byte aligned: 16-byte async copies
};
constexpr size_t kBaseSmem = (size_t)(NB * LDM + NB + NVB * LDV) * sizeof(double);

__device__ __forceinline__ void dmma884(double (&c)[2], double a, double b) {
    asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
                 : "+d"(c[0]), "+d"(c[1])
                 : "d"(a), "d"(b));
}

// X(r0..r1, :) += sign * M(r0..r1, k0..k0+nk) X(k0..k0+nk, :) on 8 x 8 output tiles dealt to
// the CTA's warps (sign = -1: TRSM update, +1: TRMM contribution).  A warp keeps UT tiles in
// flight at once (independent accumulators), so the DMMA latency of one tile's k-chain is
// hidden behind the others'.
constexpr int UT = 4;
__device__ __forceinline__ void block_update(const double *Ms, double *X, int r0, int r1, int k0, int nk,
                                             double sign, int warp, int lane, int nwarps = NW) {
    const int nrt = (r1 - r0) / 8, tiles = nrt * (NVB / 8);
    const int fr = lane >> 2, fc = lane & 3;
    for (int t0 = warp * UT; t0 < tiles; t0 += nwarps * UT) {
        int rr[UT], vv[UT];
        double d[UT][2];
#pragma unroll
        for (int u = 0; u < UT; ++u) {
            const int t = t0 + u < tiles ? t0 + u : t0;  // past the end: redo tile t0, not stored
            rr[u] = r0 + (t % nrt) * 8;
            vv[u] = (t / nrt) * 8;
            d[u][0] = X[(vv[u] + 2 * fc) * LDV + rr[u] + fr];
            d[u][1] = X[(vv[u] + 2 * fc + 1) * LDV + rr[u] + fr];
        }
        for (int k = 0; k < nk; k += 4) {
#pragma unroll
            for (int u = 0; u < UT; ++u) {
                const double a = sign * Ms[(k0 + k + fc) * LDM + rr[u] + fr];
                const double b = X[(vv[u] + fr) * LDV + k0 + k + fc];
                dmma884(d[u], a, b);
            }
        }
#pragma unroll
        for (int u = 0; u < UT; ++u) {
            if (t0 + u >= tiles) break;
            X[(vv[u] + 2 * fc) * LDV + rr[u] + fr] = d[u][0];
            X[(vv[u] + 2 * fc + 1) * LDV + rr[u] + fr] = d[u][1];
        }
    }
}

__device__ __forceinline__ void cp_async8(double *dst, const double *src, bool ok) {
    const uint32_t d = static_cast<uint32_t>(__cvta_generic_to_shared(dst));
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;\n" ::"r"(d), "l"(src), "r"(ok ? 8 : 0) : "memory");
}
__device__ __forceinline__ void cp_async16(double *dst, const double *src, bool ok) {
    const uint32_t d = static_cast<uint32_t>(__cvta_generic_to_shared(dst));
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;\n" ::"r"(d), "l"(src), "r"(ok ? 16 : 0) : "memory");
}

template <bool SOLVE, bool LOWER, bool LEFT>
__global__ void __launch_bounds__(BT) trxm_base_kernel(const __grid_constant__ BaseBatch bb, int n,
                                                       double alpha, const double *A, int64_t lda,
                                                       bool mtrans, bool unit) {
    extern __shared__ __align__(16) double smem_base[];
    double *Ms = smem_base;      // Ms[c * LDM + i] = M(i, c)
    double *rd = Ms + NB * LDM;  // 1 / M(l, l)
    double *X = rd + NB;         // X[v * LDV + l] = entry l of vector v
    int q = 0;
#pragma unroll 1
    while (q + 1 < bb.n && (int)blockIdx.x >= bb.cta_start[q + 1]) ++q;
    double *B = bb.B[q];
    const int64_t ldb = bb.ldb[q], nvec = bb.nvec[q];
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int64_t v0 = (int64_t)(blockIdx.x - bb.cta_start[q]) * NVB;
    const int nv = (int)((nvec - v0) < NVB ? (nvec - v0) : NVB);
    // Every global load is an asynchronous copy straight into shared memory (cp.async,
    // zero-filled when predicated off), all in flight at once: the referenced triangle of M
    // (consecutive threads along A's stored-contiguous direction; the other triangle, the
    // unit diagonal and the padding to NB are never read from A) as one group, then the
    // CTA's vectors block by block in the order the blocks are processed (one group each),
    // so the first diagonal block starts while the later ones are still arriving.
    constexpr int NBLK = NB / BS;
    auto order = [&](int step) { return (SOLVE == LOWER) ? step : NBLK - 1 - step; };
#pragma unroll 4
    for (int k = 0; k < NB * NB / BT; ++k) {
        const int e = tid + k * BT, f = e % NB, s2 = e / NB;
        const int i = mtrans ? s2 : f, c = mtrans ? f : s2;  // M(i, c); A contiguous in f
        const bool in = LOWER ? (i > c) : (i < c);
        const bool rd_a = i < n && c < n && (in || (i == c && !unit));
        cp_async8(Ms + c * LDM + i, rd_a ? (mtrans ? A + c + (int64_t)i * lda : A + i + (int64_t)c * lda) : A, rd_a);
    }
    asm volatile("cp.async.commit_group;\n" ::: "memory");
#pragma unroll 1
    for (int step = 0; step < NBLK; ++step) {
        const int o = order(step) * BS;
        if (LEFT) {  // BS entries of every column: 16-byte chunks, 128 contiguous bytes per column
#pragma unroll
            for (int k = 0; k < NVB * BS / 2 / BT; ++k) {
                const int c = tid + k * BT, v = c / (BS / 2), e = o + 2 * (c % (BS / 2));
                const bool ok = v < nv && e < n;
                const double *src = ok ? B + (v0 + v) * ldb + e : B;
                if (bb.al16 && (e + 1 < n || !ok)) {
                    cp_async16(X + v * LDV + e, src, ok);
                } else {
                    cp_async8(X + v * LDV + e, src, ok);
                    cp_async8(X + v * LDV + e + 1, ok && e + 1 < n ? src + 1 : B, ok && e + 1 < n);
                }
            }
        } else {     // rows of B: consecutive threads read consecutive rows of one column
#pragma unroll
            for (int k = 0; k < NVB * BS / BT; ++k) {
                const int e = tid + k * BT, v = e % NVB, l = o + e / NVB;
                const bool ok = v < nv && l < n;
                cp_async8(X + v * LDV + l, ok ? B + (v0 + v) + (int64_t)l * ldb : B, ok);
            }
        }
        asm volatile("cp.async.commit_group;\n" ::: "memory");
    }
    static_assert(NBLK == 4, "the cp.async group waits below assume 4 blocks");
    // M and the first block: the diagonal fix-up (1 where A's is not read: unit, padding)
    asm volatile("cp.async.wait_group 3;\n" ::: "memory");
    __syncthreads();
    if (tid < NB) {
        if (unit || tid >= n) Ms[tid * LDM + tid] = 1.0;
        rd[tid] = 1.0 / Ms[tid * LDM + tid];
    }
    __syncthreads();
    // one thread per vector: solve / multiply the vector's BS entries of diagonal block kb
    auto diag = [&](int kb) {
        const int o = kb * BS;
        double *xv = X + tid * LDV + o;
        double x[BS];
#pragma unroll
        for (int p = 0; p < BS / 2; ++p) {
            const double2 z = *reinterpret_cast<const double2 *>(xv + 2 * p);
            x[2 * p] = z.x;
            x[2 * p + 1] = z.y;
        }
        if (SOLVE && LOWER) {         // forward, column-oriented
#pragma unroll
            for (int l = 0; l < BS; ++l) {
                if (!unit) x[l] *= rd[o + l];
#pragma unroll
                for (int i = l + 1; i < BS; ++i) x[i] -= Ms[(o + l) * LDM + o + i] * x[l];
            }
        } else if (SOLVE) {           // backward
#pragma unroll
            for (int l = BS - 1; l >= 0; --l) {
                if (!unit) x[l] *= rd[o + l];
#pragma unroll
                for (int i = 0; i < l; ++i) x[i] -= Ms[(o + l) * LDM + o + i] * x[l];
            }
        } else if (LOWER) {           // bottom-up: row i reads x_0..x_i, still unmodified
#pragma unroll
            for (int i = BS - 1; i >= 0; --i) {
                double s = 0.0;
#pragma unroll
                for (int l = 0; l <= i; ++l) s += Ms[(o + l) * LDM + o + i] * x[l];
                x[i] = s;
            }
        } else {                      // top-down: row i reads x_i..x_BS-1
#pragma unroll
            for (int i = 0; i < BS; ++i) {
                double s = 0.0;
#pragma unroll
                for (int l = i; l < BS; ++l) s += Ms[(o + l) * LDM + o + i] * x[l];
                x[i] = s;
            }
        }
#pragma unroll
        for (int p = 0; p < BS / 2; ++p)
            *reinterpret_cast<double2 *>(xv + 2 * p) = make_double2(x[2 * p], x[2 * p + 1]);
    };
#ifndef XK_BASE_NULL
    if (SOLVE) {
        // TRSM with a one-block lookahead: after block kb is solved, the rows of the next
        // block are updated first (all warps); then warps 0-1 solve that next block while
        // warps 2-3 update the remaining rows with block kb -- the diagonal chain and the
        // bulk of the updates overlap instead of alternating
        if (tid < NVB) diag(order(0));
#pragma unroll 1
        for (int step = 0; step + 1 < NBLK; ++step) {
            const int kb = order(step), kn = order(step + 1);
            if (step == 0) asm volatile("cp.async.wait_group 2;\n" ::: "memory");
            __syncthreads();
            block_update(Ms, X, kn * BS, kn * BS + BS, kb * BS, BS, -1.0, warp, lane);
            if (step == 0) asm volatile("cp.async.wait_group 0;\n" ::: "memory");
            __syncthreads();
            if (tid < NVB) {
                diag(kn);
            } else if (LOWER) {
                if (kn + 1 < NBLK) block_update(Ms, X, (kn + 1) * BS, NB, kb * BS, BS, -1.0, warp - 2, lane, NW - 2);
            } else {
                if (kn > 0) block_update(Ms, X, 0, kn * BS, kb * BS, BS, -1.0, warp - 2, lane, NW - 2);
            }
        }
        __syncthreads();
    } else {
        asm volatile("cp.async.wait_group 0;\n" ::: "memory");
        __syncthreads();
#pragma unroll 1
        for (int step = 0; step < NBLK; ++step) {
            // TRMM: lower bottom-up (blocks above still unmodified), upper top-down
            const int kb = order(step);
            const int o = kb * BS;
            if (tid < NVB) diag(kb);
            __syncthreads();
            if (LOWER) block_update(Ms, X, o, o + BS, 0, o, 1.0, warp, lane);
            else block_update(Ms, X, o, o + BS, o + BS, NB - o - BS, 1.0, warp, lane);
            __syncthreads();
        }
    }
#else
    asm volatile("cp.async.wait_group 0;\n" ::: "memory");
    __syncthreads();
#endif
    // X back to B, times alpha (TRSM: op(A)^-1 (alpha B) = alpha op(A)^-1 B)
    const double so = alpha;
    if (LEFT) {
#pragma unroll
        for (int k = 0; k < NVB / NW; ++k) {
            const int v = warp + NW * k, e = 2 * lane;
            if (v < nv && e < n) {
                const double2 z = *reinterpret_cast<const double2 *>(X + v * LDV + e);
                double *dst = B + (v0 + v) * ldb + e;
                if (e + 1 < n) *reinterpret_cast<double2 *>(dst) = make_double2(so * z.x, so * z.y);
                else dst[0] = so * z.x;
            }
        }
    } else {
#pragma unroll
        for (int k = 0; k < NB * NVB / BT; ++k) {
            const int e = tid + k * BT, v = e % NVB, l = e / NVB;
            if (v < nv && l < n) B[(v0 + v) + (int64_t)l * ldb] = so * X[v * LDV + l];
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
    auto kern = trxm_base_kernel<SOLVE, LOWER, LEFT>;
    static unsigned attr_set = 0;  // per instantiation, one bit per device
    int dev = 0;
    cudaGetDevice(&dev);
    if (!(attr_set & (1u << dev))) {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kBaseSmem);
        if (e != cudaSuccess) return e;
        attr_set |= 1u << dev;
    }
    kern<<<grid, BT, kBaseSmem, st>>>(bb, n, alpha, A, lda, mtrans, unit);
    return cudaGetLastError();
}

cudaError_t base(const TriOp &o, int64_t n, const Tiles &T, double alpha, const double *A, int64_t lda,
                 cudaStream_t st) {
    BaseBatch bb;
    bb.n = T.n;
    bb.al16 = true;
    int total = 0;
    for (int q = 0; q < T.n; ++q) {
        bb.cta_start[q] = total;
        bb.B[q] = T.B[q];
        bb.ldb[q] = T.ldb[q];
        bb.nvec[q] = T.other[q];
        bb.al16 = bb.al16 && ((uintptr_t)T.B[q] % 16 == 0) && (T.ldb[q] % 2 == 0);
        total += (int)((T.other[q] + NVB - 1) / NVB);
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
