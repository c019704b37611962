// api_kernel.cpp -- kernel-level C entry (device pointers) and the error slot.
#include <cuda_runtime.h>

#include <mutex>
#include <string>

#include "api/common.h"
#include "kernels/kernels.h"
#include "xk.h"

namespace xk {
static std::mutex g_err_mu;
static std::string g_err;
void set_error(const std::string &msg) {
    std::lock_guard<std::mutex> lk(g_err_mu);
    g_err = msg;
}
}  // namespace xk

extern "C" {

const char *xk_last_error(void) {
    static thread_local std::string copy;
    std::lock_guard<std::mutex> lk(xk::g_err_mu);
    copy = xk::g_err;
    return copy.c_str();
}

int xk_dgemm_tile_device(char transA, char transB, int64_t m, int64_t n, int64_t k,
                         double alpha, const double *A, int64_t lda, const double *B,
                         int64_t ldb, double beta, double *C, int64_t ldc, void *stream) {
    auto up = [](char c) { return (char)((c >= 'a' && c <= 'z') ? c - 32 : c); };
    char ta = up(transA), tb = up(transB);
    if (ta != 'N' && ta != 'T' && ta != 'C') return -1;
    if (tb != 'N' && tb != 'T' && tb != 'C') return -2;
    if (m < 0) return -3;
    if (n < 0) return -4;
    if (k < 0) return -5;
    int64_t nra = (ta == 'N') ? m : k, nrb = (tb == 'N') ? k : n;
    if (lda < (nra > 1 ? nra : 1)) return -8;
    if (ldb < (nrb > 1 ? nrb : 1)) return -10;
    if (ldc < (m > 1 ? m : 1)) return -13;
    if (m == 0 || n == 0 || ((alpha == 0.0 || k == 0) && beta == 1.0)) return XK_OK;
    cudaError_t e = xk::launch_dgemm_tile(ta != 'N', tb != 'N', m, n, k, alpha, A, lda, B, ldb,
                                          beta, C, ldc, (cudaStream_t)stream);
    if (e != cudaSuccess) {
        xk::set_error(std::string("dgemm_tile launch: ") + cudaGetErrorString(e));
        return XK_ERR_CUDA;
    }
    return XK_OK;
}

}  // extern "C"
