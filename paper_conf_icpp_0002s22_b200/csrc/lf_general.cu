// lf_general.cu -- general (non-symmetric) inputs, SURVEY.md §8(f) f3.
//
// PAPER.md §4: "constructing pi from an underlying undirected graph and extracting the
// coefficients from the original graph is a better alternative for general graphs", and
// §5.1: "When A' is not symmetric, the [0,n]-factor computations use A' + A'^T".
// Two calls:
//   lf_symmetrize   S = A' + A'^T (A' = |A| - diag|A|): the union of the patterns of A and
//                   A^T without the diagonal, s_ij = fl32(|a_ij| + |a_ji|) (a missing entry
//                   counts 0).  The factor and the linear forest then run on S unchanged.
//   lf_orig_coeffs  the signed coefficients of the ORIGINAL A on the factor's slots and its
//                   diagonal (pi_val[v n + s] = a_{v, pi[v n + s]}, 0 if A does not store the
//                   entry; diag[v] = a_vv): the input of lf_tridiag / lf_linear_forest_tridiag.
// B200 design: S is built by one radix sort of the 2 nnz directed entries keyed row n + col
// -- every entry (i,j) contributes (i,j) and (j,i) -- and one reduce-by-key that adds the
// (at most two) |values| of a key; fl32 addition of two operands is commutative, so the sum
// does not depend on which of the two the sort puts first.  Diagonal entries get the
// largest key and are dropped.  The row pointers follow from the sorted keys.
#include <cuda_runtime.h>

#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_reduce.cuh>

#include <cstdint>

#include "lf_common.cuh"
#include "lf_internal.h"

namespace lf {

namespace {

constexpr uint64_t kDiagKey = ~0ull;  // sorts last, dropped

// the two directed keys of every stored entry (a thread per row: rows are short)
__global__ void k_sym_keys(int64_t n, const int64_t* __restrict__ rowptr, const int32_t* __restrict__ col,
                           const float* __restrict__ val, uint64_t* __restrict__ keys, float* __restrict__ vals) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t e0 = rowptr[i], e1 = rowptr[i + 1];
        for (int64_t e = e0; e < e1; e++) {
            const int64_t j = col[e];
            const float w = fabsf(val[e]);  // A' = |A| (L231)
            const bool d = j == i;           // - diag|A|
            keys[2 * e] = d ? kDiagKey : (uint64_t)i * (uint64_t)n + (uint64_t)j;  // (row, col) as i n + j:
            keys[2 * e + 1] = d ? kDiagKey : (uint64_t)j * (uint64_t)n + (uint64_t)i;  // fewer radix passes
            vals[2 * e] = w;
            vals[2 * e + 1] = w;
        }
    }
}

// unique sorted keys -> column indices and row pointers of S; s_nnz = the non-diagonal runs
__global__ void k_sym_rows(int64_t n, const uint64_t* __restrict__ ukeys, const int* __restrict__ nruns,
                           int32_t* __restrict__ s_col, int64_t* __restrict__ s_rowptr, int64_t* __restrict__ s_nnz) {
    const int64_t nr = *nruns;
    const int64_t m = (nr > 0 && ukeys[nr - 1] == kDiagKey) ? nr - 1 : nr;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    const int64_t t0 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t0 == 0) {
        *s_nnz = m;
        s_rowptr[n] = m;
    }
    for (int64_t r = t0; r < m; r += stride) {
        const uint64_t k = ukeys[r];
        const int64_t i = (int64_t)(k / (uint64_t)n);
        s_col[r] = (int32_t)(k - (uint64_t)i * (uint64_t)n);
        // rows prev+1 .. i start at r (prev = the row of run r-1, -1 before the first run)
        const int64_t prev = r > 0 ? (int64_t)(ukeys[r - 1] / (uint64_t)n) : -1;
        for (int64_t q = prev + 1; q <= i; q++) s_rowptr[q] = r;
    }
    // rows after the last run's row
    const int64_t last = m > 0 ? (int64_t)(ukeys[m - 1] / (uint64_t)n) : -1;
    for (int64_t q = last + 1 + t0; q < n; q += stride) s_rowptr[q] = m;
}

// signed coefficients of A on the factor's slots, and its diagonal (a thread per row)
__global__ void k_orig_coeffs(int64_t n, int nn, const int64_t* __restrict__ rowptr, const int32_t* __restrict__ col,
                              const float* __restrict__ val, const int32_t* __restrict__ pi, float* __restrict__ pi_val,
                              float* __restrict__ diag) {
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        int32_t p[4] = {-1, -1, -1, -1};
        float o[4] = {0.f, 0.f, 0.f, 0.f};
        for (int s = 0; s < nn; s++) p[s] = pi[v * nn + s];
        float dv = 0.f;
        const int64_t e0 = rowptr[v], e1 = rowptr[v + 1];
        for (int64_t e = e0; e < e1; e++) {
            const int32_t j = col[e];
            const float a = val[e];
            if (j == v) dv = a;
            for (int s = 0; s < nn; s++)
                if (p[s] >= 0 && p[s] == j) o[s] = a;
        }
        if (pi_val)
            for (int s = 0; s < nn; s++) pi_val[v * nn + s] = o[s];
        if (diag) diag[v] = dv;
    }
}

struct SymWs {
    uint64_t *k0, *k1, *uk;
    float *v0, *v1;
    int* nruns;
    void* tmp;
    size_t tmp_bytes;
};

size_t sym_temp_bytes(int64_t m) {
    size_t a = 0, b = 0;
    const int mi = (int)(m > 0 ? m : 1);
    cub::DeviceRadixSort::SortPairs(nullptr, a, (const uint64_t*)nullptr, (uint64_t*)nullptr, (const float*)nullptr,
                                    (float*)nullptr, mi);
    cub::DeviceReduce::ReduceByKey(nullptr, b, (const uint64_t*)nullptr, (uint64_t*)nullptr, (const float*)nullptr,
                                   (float*)nullptr, (int*)nullptr, cub::Sum(), mi);
    (void)cudaGetLastError();
    return (a > b ? a : b) + 4096;
}

size_t sym_carve(Carve& c, int64_t nnz, SymWs* w) {
    SymWs t;
    const size_t m = (size_t)(2 * (nnz > 0 ? nnz : 1));
    t.k0 = c.take<uint64_t>(m);
    t.k1 = c.take<uint64_t>(m);
    t.uk = c.take<uint64_t>(m);
    t.v0 = c.take<float>(m);
    t.v1 = c.take<float>(m);
    t.nruns = c.take<int>(64);
    t.tmp_bytes = sym_temp_bytes((int64_t)m);
    t.tmp = c.take<char>(t.tmp_bytes);
    if (w) *w = t;
    return c.off;
}

bool csr_args_ok(const lf_csr_t* A) {
    if (!A || A->n < 0 || A->n >= ((int64_t)1 << 31) || A->nnz < 0) return false;
    if (A->n > 0 && !A->rowptr) return false;
    if (A->nnz > 0 && (!A->col || !A->val)) return false;
    return true;
}

}  // namespace

}  // namespace lf

using namespace lf;

extern "C" size_t lf_symmetrize_workspace_size(int64_t n, int64_t nnz) {
    (void)n;
    if (nnz < 0 || nnz >= ((int64_t)1 << 30)) return 0;
    Carve c(nullptr, 0);
    return sym_carve(c, nnz, nullptr) + 256;
}

extern "C" int lf_symmetrize(const lf_csr_t* A, int64_t* s_rowptr, int32_t* s_col, float* s_val, int64_t* s_nnz,
                             void* ws, size_t ws_bytes, void* stream) {
    g_err_clear();
    if (!csr_args_ok(A)) return set_error(LF_EINVAL, "lf_symmetrize: bad CSR descriptor");
    if (A->nnz >= ((int64_t)1 << 30)) return set_error(LF_EINVAL, "lf_symmetrize: nnz must be < 2^30");
    if (!s_rowptr || !s_nnz || (A->nnz > 0 && (!s_col || !s_val)))
        return set_error(LF_EINVAL, "lf_symmetrize: NULL output");
    cudaStream_t s = (cudaStream_t)stream;
    const int64_t n = A->n, m = 2 * A->nnz;
    if (m == 0) {
        LF_CUDA(cudaMemsetAsync(s_rowptr, 0, sizeof(int64_t) * (size_t)(n + 1), s));
        LF_CUDA(cudaMemsetAsync(s_nnz, 0, sizeof(int64_t), s));
        return LF_OK;
    }
    Carve c(ws, ws_bytes);
    SymWs w;
    sym_carve(c, A->nnz, &w);
    if (!ws || !c.ok() || ((uintptr_t)ws & 255)) return set_error(LF_ENOMEM, "lf_symmetrize: workspace too small");
    const int grid = persistent_grid((const void*)k_sym_keys, 256);
    k_sym_keys<<<grid, 256, 0, s>>>(n, A->rowptr, A->col, A->val, w.k0, w.v0);
    LF_CUDA(cudaGetLastError());
    size_t tb = w.tmp_bytes;
    // keys below n^2 - 1 (the diagonal key, all ones, still sorts last on these bits)
    int end_bit = 1;
    while (end_bit < 64 && ((uint64_t)1 << end_bit) < (uint64_t)n * (uint64_t)n) end_bit++;
    LF_CUDA(cub::DeviceRadixSort::SortPairs(w.tmp, tb, w.k0, w.k1, w.v0, w.v1, (int)m, 0, end_bit, s));
    tb = w.tmp_bytes;
    LF_CUDA(cub::DeviceReduce::ReduceByKey(w.tmp, tb, w.k1, w.uk, w.v1, s_val, w.nruns, cub::Sum(), (int)m, s));
    k_sym_rows<<<persistent_grid((const void*)k_sym_rows, 256), 256, 0, s>>>(n, w.uk, w.nruns, s_col, s_rowptr, s_nnz);
    LF_CUDA(cudaGetLastError());
    return LF_OK;
}

extern "C" int lf_orig_coeffs(const lf_csr_t* A, int n, const int32_t* pi, float* pi_val, float* diag, void* stream) {
    g_err_clear();
    if (!csr_args_ok(A)) return set_error(LF_EINVAL, "lf_orig_coeffs: bad CSR descriptor");
    if (n < 1 || n > 4) return set_error(LF_EINVAL, "lf_orig_coeffs: n must be in [1,4]");
    if (A->n > 0 && (!pi || (!pi_val && !diag))) return set_error(LF_EINVAL, "lf_orig_coeffs: NULL argument");
    if (A->n == 0) return LF_OK;
    k_orig_coeffs<<<persistent_grid((const void*)k_orig_coeffs, 256), 256, 0, (cudaStream_t)stream>>>(
        A->n, n, A->rowptr, A->col, A->val, pi, pi_val, diag);
    LF_CUDA(cudaGetLastError());
    return LF_OK;
}
