/* examples/xk_dgemm_example.c -- using libxk.so from plain C through include/xk.h.
 *
 * Host-resident column-major matrices, a synchronous DGEMM, then two asynchronous calls that
 * compose through the GPU tile cache (D = A*B; E = D*B) with only E made coherent
 * (PAPER.md P:947-958), and a BLAS argument error.  Checks a few entries against a plain
 * triple-loop and prints the library's transfer statistics.  Exit status 0 on success.
 *
 *   gcc -O2 -I include examples/xk_dgemm_example.c -L paper_conf_sc_gautierl21_b200 -lxk \
 *       -Wl,-rpath,$PWD/paper_conf_sc_gautierl21_b200 -o xk_example && ./xk_example
 */
#include <math.h>
#include <stdio.h>
#include <stdlib.h>

#include "xk.h"

static double ref_entry(int64_t n, const double *X, const double *Y, int64_t i, int64_t j) {
    double s = 0.0;
    for (int64_t l = 0; l < n; ++l) s += X[i + l * n] * Y[l + j * n];
    return s;
}

int main(void) {
    const int64_t n = 1500;
    double *A = malloc(sizeof(double) * n * n), *B = malloc(sizeof(double) * n * n);
    double *C = malloc(sizeof(double) * n * n), *D = malloc(sizeof(double) * n * n);
    double *E = malloc(sizeof(double) * n * n);
    for (int64_t q = 0; q < n * n; ++q) {
        A[q] = (double)((q * 7919) % 17) - 8.0;
        B[q] = (double)((q * 104729) % 13) - 6.0;
        C[q] = 1.0;
    }
    xk_config_t cfg;
    xk_config_default(&cfg);
    cfg.tile = 512;
    cfg.probe = 0;
    int rc = xk_init(&cfg);
    if (rc) {
        fprintf(stderr, "xk_init: %d %s\n", rc, xk_last_error());
        return 1;
    }
    /* BLAS argument check: lda < m is argument 8 */
    if (xk_dgemm('N', 'N', n, n, n, 1.0, A, n - 1, B, n, 0.0, C, n) != -8) return 2;
    rc = xk_dgemm('N', 'N', n, n, n, 2.0, A, n, B, n, -1.0, C, n);
    if (rc) {
        fprintf(stderr, "xk_dgemm: %d %s\n", rc, xk_last_error());
        return 3;
    }
    rc = xk_dgemm_async('N', 'N', n, n, n, 1.0, A, n, B, n, 0.0, D, n);
    rc |= xk_dgemm_async('N', 'N', n, n, n, 1.0, D, n, B, n, 0.0, E, n);
    rc |= xk_memory_coherent_sync(n, n, E, n);
    rc |= xk_memory_coherent_sync(n, n, D, n);
    if (rc) {
        fprintf(stderr, "async: %d %s\n", rc, xk_last_error());
        return 4;
    }
    int64_t probes[4][2] = {{0, 0}, {n - 1, n - 1}, {17, 1234}, {999, 3}};
    for (int p = 0; p < 4; ++p) {
        int64_t i = probes[p][0], j = probes[p][1];
        double c = 2.0 * ref_entry(n, A, B, i, j) - 1.0;      /* exact: integer data */
        double e = ref_entry(n, D, B, i, j);
        if (C[i + j * n] != c || E[i + j * n] != e) {
            fprintf(stderr, "mismatch at (%ld,%ld): %g vs %g, %g vs %g\n", (long)i, (long)j,
                    C[i + j * n], c, E[i + j * n], e);
            return 5;
        }
    }
    xk_stats_t st;
    xk_get_stats(&st);
    printf("xk example ok: %lld tile tasks, H2D %.1f MB, D2H %.1f MB, %lld kernel launches\n",
           (long long)st.tasks[0], st.h2d_bytes[0] / 1e6, st.d2h_bytes[0] / 1e6,
           (long long)st.kernel_launches);
    xk_finalize();
    free(A); free(B); free(C); free(D); free(E);
    return 0;
}
