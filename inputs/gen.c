/*
 * inputs/gen.c -- seeded, counter-based synthetic input generator (SURVEY.md §8(d)
 * "Generator"; readings Q9/Q10 in DESIGN.md).  Shared by the oracle side (tests,
 * bench cpu_baseline) and the product side (bench, GPU parity tests) as the ONLY common
 * module; it holds none of the method's arithmetic -- it only fills host arrays.
 *
 *   x  = splitmix64_mix(seed * 0x9E3779B97F4A7C15 + idx),  idx = i + j*m (logical
 *        column-major index, independent of ld)
 *   u  = (x >> 11) * 2^-53 in [0,1)
 *   real inputs   : a = 2u - 1 in [-1,1)
 *   integer inputs: a = floor(span*u) + lo  (default span 17, lo -8 -> [-8,8])
 *   triangular    : Q9 diagonally dominant factor, off-diagonal (2u-1)/(2*n),
 *                   diagonal 1 + u; the other triangle gets `fill`.
 * Counter-based, so any thread count and any language produce identical matrices.
 */
#include <stdint.h>
#include <math.h>

typedef int64_t i64;

static inline uint64_t mix(uint64_t z)
{
    z ^= z >> 30; z *= 0xBF58476D1CE4E5B9ULL;
    z ^= z >> 27; z *= 0x94D049BB133111EBULL;
    z ^= z >> 31;
    return z;
}
static inline double u01(uint64_t seed, uint64_t idx)
{
    return (double)(mix(seed * 0x9E3779B97F4A7C15ULL + idx) >> 11) * 0x1.0p-53;
}

uint64_t xkgen_mix(uint64_t z) { return mix(z); }

/* threads of the fills (torchrun sets OMP_NUM_THREADS=1 in every rank; the one rank that
 * generates the shared matrices asks for all of its cores) -- never affects the values */
#ifdef _OPENMP
#include <omp.h>
void xkgen_set_threads(int n) { if (n > 0) omp_set_num_threads(n); }
#else
void xkgen_set_threads(int n) { (void)n; }
#endif

void xkgen_uniform(uint64_t seed, i64 m, i64 n, double *out, i64 ld)
{
#pragma omp parallel for schedule(static)
    for (i64 j = 0; j < n; ++j)
        for (i64 i = 0; i < m; ++i)
            out[i + j * ld] = 2.0 * u01(seed, (uint64_t)(i + j * m)) - 1.0;
}

void xkgen_int(uint64_t seed, i64 m, i64 n, double *out, i64 ld, int lo, int span)
{
#pragma omp parallel for schedule(static)
    for (i64 j = 0; j < n; ++j)
        for (i64 i = 0; i < m; ++i)
            out[i + j * ld] = floor((double)span * u01(seed, (uint64_t)(i + j * m))) + (double)lo;
}

void xkgen_tri_dd(uint64_t seed, i64 n, double *out, i64 ld, int lower, double fill)
{
#pragma omp parallel for schedule(static)
    for (i64 j = 0; j < n; ++j)
        for (i64 i = 0; i < n; ++i) {
            double u = u01(seed, (uint64_t)(i + j * n));
            double v;
            if (i == j) v = 1.0 + u;
            else if (lower ? (i > j) : (i < j)) v = (2.0 * u - 1.0) / (2.0 * (double)n);
            else v = fill;
            out[i + j * ld] = v;
        }
}
