// lf_tridiag.cu -- step (4) of PAPER.md §3.3 (L219) / §4.3 (L297): copy the coefficients
// of the linear forest into the three diagonals of Q^T A Q.
//
// The paper converts A to COO and scatters one thread per stored entry, checking forest
// membership (L297).  Here the signed forest coefficients and the diagonal were captured
// by lf_factor while it streamed the rows (pi_val, diag), so the pass is one thread per
// vertex over O(N) bytes and never re-reads the CSR.
#include <cuda_runtime.h>

#include <cstdint>

#include "lf_common.cuh"
#include "lf_internal.h"

namespace lf {

__global__ void __launch_bounds__(256) k_tridiag(int64_t N, const int2* __restrict__ forest,
                                                 const int32_t* __restrict__ iperm,
                                                 const int2* __restrict__ pi2,
                                                 const float2* __restrict__ pi2_val,
                                                 const float* __restrict__ diag, float* a, float* b,
                                                 float* c) {
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < N;
         v += (int64_t)gridDim.x * blockDim.x) {
        const int32_t r = __ldg(iperm + v);
        const int2 f = __ldg(forest + v);
        const int2 pn = __ldg(pi2 + v);
        const float2 pv = __ldg(pi2_val + v);
        float ar = 0.0f, cr = 0.0f;
        if (f.x >= 0) {
            const float x = (pn.x == f.x) ? pv.x : pv.y;
            const int32_t rw = __ldg(iperm + f.x);
            if (rw == r - 1) ar = x;
            else if (rw == r + 1) cr = x;
        }
        if (f.y >= 0) {
            const float x = (pn.x == f.y) ? pv.x : pv.y;
            const int32_t rw = __ldg(iperm + f.y);
            if (rw == r - 1) ar = x;
            else if (rw == r + 1) cr = x;
        }
        a[r] = ar;
        b[r] = __ldg(diag + v);
        c[r] = cr;
    }
}

int tridiag_run(int64_t N, const int32_t* forest, const int32_t* iperm, const int32_t* pi2,
                const float* pi2_val, const float* diag, float* a, float* b, float* c,
                cudaStream_t s) {
    if (N == 0) return LF_OK;
    LF_PROF("tridiag", -1, s);
    k_tridiag<<<persistent_grid((const void*)k_tridiag, 256), 256, 0, s>>>(
        N, (const int2*)forest, iperm, (const int2*)pi2, (const float2*)pi2_val, diag, a, b, c);
    LF_CUDA(cudaGetLastError());
    return LF_OK;
}

}  // namespace lf
