// lfgen_gpu.cu -- seeded synthetic input generator on the device (liblfgen_gpu.so).
//
// INPUT GENERATION ONLY: this file holds none of the method's arithmetic (no proposal,
// confirmation, scan or permutation).  It writes, on the GPU, the rows of the same 27-point
// graph that lfgen.grid3d_27pt_rows builds with numpy (SURVEY.md §8(d) C5 recipe: n x n x nz
// grid, natural order, |w| = 1 - u with u the splitmix64 edge hash on a 24-bit grid,
// a_uv = -w, a_vv = sum |w| + 1), so the 512^3 graph (3.6e9 entries, 30 GB) can be built
// in HBM slab by slab without a host round trip.  tests/test_gpu_c5.py checks it against
// the numpy generator (sha256, small n and the full C5) -- it shares no code with the
// product library (paper_conf_icpp_0002s22_b200/csrc) or the oracle.
#include <cuda_runtime.h>

#include <cstdint>

namespace {

constexpr uint64_t kGolden = 0x9E3779B97F4A7C15ull;

__device__ __forceinline__ uint64_t splitmix64(uint64_t z) {
    z += kGolden;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

// 2^24 * w for the edge {s, t}: w = 1 - h 2^-24 with h the top 24 bits of the hash
__device__ __forceinline__ uint32_t weight24(uint64_t s, uint64_t t, uint64_t N, uint64_t seed) {
    const uint64_t lo = s < t ? s : t, hi = s < t ? t : s;
    const uint64_t h = splitmix64(seed ^ ((lo * N + hi) * kGolden)) >> 40;
    return (uint32_t)((1ull << 24) - h);
}

// entries stored by a coordinate with `c` neighbours per axis: 3 minus the missing sides
__device__ __forceinline__ int64_t cnt(int64_t x, int64_t n) { return n == 1 ? 1 : 3 - (x == 0) - (x == n - 1); }
// sum of cnt over [0, x)
__device__ __forceinline__ int64_t pre(int64_t x, int64_t n) {
    if (n == 1) return x;
    return x == 0 ? 0 : 2 + 3 * (x - 1);
}

// one thread per row of the slab: closed-form row offset, 26 hashes, ascending columns
__global__ void k_grid27_rows(int64_t n, int64_t nz, int64_t z_lo, int64_t z_hi, uint64_t seed,
                              int64_t* __restrict__ rowptr, int32_t* __restrict__ col,
                              float* __restrict__ val) {
    const int64_t plane = n * n;
    const int64_t rows = (z_hi - z_lo) * plane;
    const uint64_t N = (uint64_t)(plane * nz);
    const int64_t S = n == 1 ? 1 : 3 * n - 2;  // sum of cnt over one axis
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < rows;
         i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t v = z_lo * plane + i;
        const int64_t x = v % n, y = (v / n) % n, z = v / plane;
        const int64_t cz = cnt(z, nz), cy = cnt(y, n), cx = cnt(x, n);
        const int64_t off = S * S * (pre(z, nz) - pre(z_lo, nz)) + cz * (S * pre(y, n) + cy * pre(x, n));
        rowptr[i] = off;
        if (i == rows - 1) rowptr[rows] = off + cz * cy * cx;
        uint32_t w[27];
        uint64_t wsum = 1ull << 24;  // the +1 of the diagonal, in units of 2^-24
#pragma unroll
        for (int k = 0; k < 27; k++) {
            const int dx = k % 3 - 1, dy = (k / 3) % 3 - 1, dz = k / 9 - 1;
            const bool ok = x + dx >= 0 && x + dx < n && y + dy >= 0 && y + dy < n && z + dz >= 0 && z + dz < nz;
            w[k] = 0;
            if (ok && k != 13) {
                const int64_t j = v + dx + n * (dy + n * dz);
                w[k] = weight24((uint64_t)v, (uint64_t)j, N, seed);
                wsum += w[k];
            }
        }
        // exact: every w is a multiple of 2^-24 and the sum < 2^29; one rounding to fp32
        const float diag = __ll2float_rn((long long)wsum) * 0x1p-24f;
        int64_t e = off;
#pragma unroll
        for (int k = 0; k < 27; k++) {
            const int dx = k % 3 - 1, dy = (k / 3) % 3 - 1, dz = k / 9 - 1;
            const bool ok = x + dx >= 0 && x + dx < n && y + dy >= 0 && y + dy < n && z + dz >= 0 && z + dz < nz;
            if (!ok) continue;
            col[e] = (int32_t)(v + dx + n * (dy + n * dz));
            val[e] = k == 13 ? diag : -((float)w[k] * 0x1p-24f);
            e++;
        }
    }
}

}  // namespace

extern "C" {

// stored entries of the planes [z_lo, z_hi) (closed form, host)
int64_t lfg_grid27_nnz(int64_t n, int64_t nz, int64_t z_lo, int64_t z_hi) {
    auto c = [](int64_t x, int64_t m) -> int64_t { return m == 1 ? 1 : 3 - (x == 0) - (x == m - 1); };
    const int64_t S = n == 1 ? 1 : 3 * n - 2;
    int64_t cz = 0;
    for (int64_t z = z_lo; z < z_hi; z++) cz += c(z, nz);
    return S * S * cz;
}

// rows of the planes [z_lo, z_hi) of the n x n x nz 27-point graph, GLOBAL column ids:
// rowptr[(z_hi - z_lo) n^2 + 1] (rebased to 0), col/val[lfg_grid27_nnz(...)], device
// pointers, asynchronous on `stream`.  Returns 0 or a cudaError_t.
int lfg_grid27_rows(int64_t n, int64_t nz, int64_t z_lo, int64_t z_hi, uint64_t seed, int64_t* rowptr,
                    int32_t* col, float* val, void* stream) {
    if (n < 1 || nz < 1 || z_lo < 0 || z_hi > nz || z_lo > z_hi || n * n * nz >= (1ll << 31)) return -1;
    const int64_t rows = (z_hi - z_lo) * n * n;
    if (rows == 0) {
        return (int)cudaMemsetAsync(rowptr, 0, sizeof(int64_t), (cudaStream_t)stream);
    }
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    int64_t blocks = (rows + 255) / 256;
    if (blocks > (int64_t)sms * 32) blocks = (int64_t)sms * 32;
    k_grid27_rows<<<(int)blocks, 256, 0, (cudaStream_t)stream>>>(n, nz, z_lo, z_hi, seed, rowptr, col, val);
    return (int)cudaGetLastError();
}

}  // extern "C"
