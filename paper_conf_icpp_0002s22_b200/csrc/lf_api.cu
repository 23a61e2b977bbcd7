// lf_api.cu -- the extern "C" boundary of liblf.so (include/lf.h): argument checks,
// workspace carving, error reporting, and the host-buffer end-to-end entry.
#include <cuda_runtime.h>

#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <unordered_map>
#include <vector>

#include "lf_common.cuh"
#include "lf_internal.h"

namespace lf {

static thread_local char g_err[512] = "";

void g_err_clear() { g_err[0] = 0; }

int set_error(int code, const char* msg) {
    snprintf(g_err, sizeof(g_err), "%s", msg);
    return code;
}

int set_cuda_error(cudaError_t e, const char* where) {
    snprintf(g_err, sizeof(g_err), "CUDA error %s (%s) in %s", cudaGetErrorName(e),
             cudaGetErrorString(e), where);
    return LF_ECUDA;
}

// ---------------------------------------------------------------------------
// per-kernel event timing
// ---------------------------------------------------------------------------
struct ProfRec {
    char name[40];
    cudaEvent_t a, b;
};
static std::mutex g_prof_mu;
static bool g_prof = false;
static std::vector<ProfRec> g_recs;
static std::vector<std::pair<cudaEvent_t, cudaEvent_t>> g_pool;

// inside a stream capture a plain record only orders streams; an "external" record
// becomes an event-record node that fires on every graph replay
static void record_event(cudaEvent_t e, cudaStream_t s) {
    cudaStreamCaptureStatus st = cudaStreamCaptureStatusNone;
    cudaStreamIsCapturing(s, &st);
    if (st == cudaStreamCaptureStatusActive) cudaEventRecordWithFlags(e, s, cudaEventRecordExternal);
    else cudaEventRecord(e, s);
}

int prof_begin(const char* name, int k, cudaStream_t s) {
    if (!g_prof) return -1;
    std::lock_guard<std::mutex> lk(g_prof_mu);
    const size_t i = g_recs.size();
    if (i >= g_pool.size()) {
        cudaEvent_t a, b;
        cudaEventCreate(&a);
        cudaEventCreate(&b);
        g_pool.push_back({a, b});
    }
    ProfRec r;
    if (k >= 0) snprintf(r.name, sizeof(r.name), "%s[%d]", name, k);
    else snprintf(r.name, sizeof(r.name), "%s", name);
    r.a = g_pool[i].first;
    r.b = g_pool[i].second;
    g_recs.push_back(r);
    record_event(r.a, s);
    return (int)i;
}

// closes record `idx` (scopes nest: an outer stage around per-kernel records)
void prof_end(cudaStream_t s, int idx) {
    if (!g_prof || idx < 0) return;
    std::lock_guard<std::mutex> lk(g_prof_mu);
    if ((size_t)idx < g_recs.size()) record_event(g_recs[idx].b, s);
}

int sm_count() {
    static int n = 0;
    if (n == 0) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
        if (n <= 0) n = 148;
    }
    return n;
}

bool pdl_enabled() {
    static const bool on = getenv("LF_NO_PDL") == nullptr;
    return on;
}

int persistent_grid(const void* kernel, int block, size_t smem) {
    static std::mutex mu;
    static std::unordered_map<const void*, int> cache;
    std::lock_guard<std::mutex> lk(mu);
    auto it = cache.find(kernel);
    if (it != cache.end()) return it->second;
    int per_sm = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kernel, block, smem) != cudaSuccess ||
        per_sm <= 0)
        per_sm = 1;
    const int g = per_sm * sm_count();
    cache[kernel] = g;
    return g;
}

size_t factor_ws_carve(Carve& c, int64_t N, int n, FactorWs* w) {
    FactorWs t;
    const size_t nn = (size_t)(N > 0 ? N : 1);
    t.state = c.take<uint8_t>(nn + 4);  // + 4: word-sized state fetches past the last vertex
    t.prop_j = c.take<int32_t>(nn * n);
    t.prop_v = c.take<float>(nn * n);
    t.wl[0] = c.take<int32_t>(nn);
    t.wl[1] = c.take<int32_t>(nn);
    // control block, contiguous so that one memset clears it: counts | flags | long_count |
    // live_part (the factor zeroes up to live_part + 128 M)
    t.counts = c.take<int32_t>(4);
    t.flags = c.take<int>(kMaxFlagRounds);
    t.long_count = c.take<int32_t>(kMaxFlagRounds);
    t.live_part = c.take<unsigned long long>((size_t)kMaxFlagRounds * 128);
    t.long_rows = c.take<int32_t>(nn);
    if (w) *w = t;
    return c.off;
}

static bool csr_ok(const lf_csr_t* A) {
    if (!A) return false;
    if (A->n < 0 || A->n >= ((int64_t)1 << 31) || A->nnz < 0) return false;
    if (A->n > 0 && (!A->rowptr)) return false;
    if (A->nnz > 0 && (!A->col || !A->val)) return false;
    return true;
}

// ---------------------------------------------------------------------------
// validation kernel
// ---------------------------------------------------------------------------
// pass 1: row pointers, column range, finite values; per row: strictly ascending columns
// (sorted[v] = 1), else a duplicate search within the row (O(deg^2), unsorted rows only)
__global__ void k_validate(int64_t N, int64_t nnz, const int64_t* rowptr, const int32_t* col,
                           const float* val, int* bad, uint8_t* sorted) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v <= N; v += stride) {
        const int64_t r = rowptr[v];
        if (v == 0 && r != 0) atomicOr(bad, 1);
        if (v == N && r != nnz) atomicOr(bad, 1);
        if (v < N && (rowptr[v + 1] < r || r < 0 || r > nnz)) atomicOr(bad, 1);
    }
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < nnz; e += stride) {
        const int32_t j = col[e];
        if (j < 0 || (int64_t)j >= N) atomicOr(bad, 2);
        if (!isfinite(val[e])) atomicOr(bad, 4);
    }
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < N; v += stride) {
        const int64_t r0 = min(max(rowptr[v], (int64_t)0), nnz), r1 = min(max(rowptr[v + 1], r0), nnz);
        bool asc = true;
        for (int64_t e = r0 + 1; e < r1 && asc; e++) asc = col[e] > col[e - 1];
        sorted[v] = asc ? 1 : 0;
        if (asc) continue;
        bool dup = false;
        for (int64_t e = r0; e < r1 && !dup; e++)
            for (int64_t f = e + 1; f < r1; f++)
                if (col[e] == col[f]) { dup = true; break; }
        if (dup) atomicOr(bad, 8);
    }
}

// pass 2 (a warp per row): every edge (i, j) -- j != i, a_ij != 0, PAPER.md:L31, L231 --
// needs the entry (j, i) with the same |a| (an undirected weighted graph, L315)
__global__ void k_validate_sym(int64_t N, int64_t nnz, const int64_t* rowptr, const int32_t* col,
                               const float* val, int* bad, const uint8_t* sorted) {
    const int lane = threadIdx.x & 31;
    const int64_t w0 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t i = w0; i < N; i += nw) {
        const int64_t r0 = min(max(rowptr[i], (int64_t)0), nnz), r1 = min(max(rowptr[i + 1], r0), nnz);
        for (int64_t e = r0 + lane; e < r1; e += 32) {
            const int32_t j = col[e];
            const uint32_t x = __float_as_uint(val[e]) & 0x7FFFFFFFu;
            if (j < 0 || (int64_t)j >= N || (int64_t)j == i || x == 0u) continue;
            const int64_t s0 = min(max(rowptr[j], (int64_t)0), nnz), s1 = min(max(rowptr[j + 1], s0), nnz);
            int64_t hit = -1;
            if (sorted[j]) {
                int64_t lo = s0, hi = s1;
                while (lo < hi) {
                    const int64_t m = (lo + hi) >> 1;
                    if ((int64_t)col[m] < i) lo = m + 1; else hi = m;
                }
                if (lo < s1 && (int64_t)col[lo] == i) hit = lo;
            } else {
                for (int64_t f = s0; f < s1; f++)
                    if ((int64_t)col[f] == i) { hit = f; break; }
            }
            if (hit < 0) atomicOr(bad, 16);
            else if ((__float_as_uint(val[hit]) & 0x7FFFFFFFu) != x) atomicOr(bad, 32);
        }
    }
}

// a [0,n]-factor in lf_factor's canonical form: ids in range, no self loop, valid slots
// first and -1 padding last, no repeated neighbour, symmetric (w in pi(v) <=> v in pi(w))
__global__ void k_validate_factor(int64_t N, int n, const int32_t* pi, int* bad) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < N; v += stride) {
        bool pad = false;
        for (int s = 0; s < n; s++) {
            const int32_t w = pi[v * n + s];
            if (w < -1 || (int64_t)w >= N || (int64_t)w == v) { atomicOr(bad, 64); break; }
            if (w < 0) { pad = true; continue; }
            if (pad) { atomicOr(bad, 64); break; }  // a neighbour after padding
            bool back = false;
            for (int t = 0; t < n; t++) {
                if (t != s && pi[v * n + t] == w) atomicOr(bad, 64);
                back |= pi[(int64_t)w * n + t] == (int32_t)v;
            }
            if (!back) atomicOr(bad, 128);
        }
    }
}

}  // namespace lf

using namespace lf;

extern "C" {

void lf_factor_opts_default(lf_factor_opts_t* o) {
    if (!o) return;
    o->M = 5;
    o->m = 5;
    o->k_m = 0;
    o->p = 0.5f;
    o->seed = 0;
    o->until_maximal = 0;
}

const char* lf_last_error(void) { return g_err; }

int lf_profile_enable(int on) {
    std::lock_guard<std::mutex> lk(g_prof_mu);
    g_prof = on != 0;
    if (g_prof) g_recs.clear();  // turning off keeps the records for lf_profile_collect
    return LF_OK;
}

int lf_profile_collect(char* names, int name_stride, float* ms, int cap) {
    std::lock_guard<std::mutex> lk(g_prof_mu);
    int n = 0;
    for (auto& r : g_recs) {
        if (n >= cap) break;
        float t = -1.0f;
        if (cudaEventSynchronize(r.b) == cudaSuccess) cudaEventElapsedTime(&t, r.a, r.b);
        if (ms) ms[n] = t;
        if (names && name_stride > 0) snprintf(names + (size_t)n * name_stride, name_stride, "%s", r.name);
        n++;
    }
    (void)cudaGetLastError();  // an unrecorded event must not leak into a later launch check
    return n;
}

const char* lf_version(void) { return "liblf 0.1 sm_100a"; }

size_t lf_factor_workspace_size(int64_t N, int n) {
    if (n < 1 || n > 4) return 0;
    Carve c(nullptr, 0);
    return factor_ws_carve(c, N, n, nullptr) + 256;
}

int lf_factor(const lf_csr_t* A, int n, const lf_factor_opts_t* opts, int32_t* pi, float* pi_w,
              float* pi_val, float* diag, int32_t* rounds_dev, int64_t* live, void* ws,
              size_t ws_bytes, void* stream) {
    g_err[0] = 0;
    if (!csr_ok(A)) return set_error(LF_EINVAL, "lf_factor: invalid CSR descriptor");
    if (n < 1 || n > 4) return set_error(LF_EINVAL, "lf_factor: n must be in [1,4]");
    if (A->n > 0 && (!pi || !pi_w)) return set_error(LF_EINVAL, "lf_factor: pi and pi_w are required");
    lf_factor_opts_t o;
    if (opts) o = *opts; else lf_factor_opts_default(&o);
    if (o.m < 1 || o.M < 0) return set_error(LF_EINVAL, "lf_factor: need m >= 1 and M >= 0");
    if (o.until_maximal && (o.k_m < 0 || o.k_m >= o.m))
        return set_error(LF_EINVAL, "lf_factor: until_maximal needs 0 <= k_m < m");
    if (!o.until_maximal && o.M > kMaxFlagRounds)
        return set_error(LF_EINVAL, "lf_factor: M > 1024 (use until_maximal)");
    if (!(o.p >= 0.0f && o.p <= 1.0f)) return set_error(LF_EINVAL, "lf_factor: p must be in [0,1]");
    Carve c(ws, ws_bytes);
    FactorWs w;
    factor_ws_carve(c, A->n, n, &w);
    if (!ws || !c.ok()) return set_error(LF_ENOMEM, "lf_factor: workspace too small");
    return factor_dispatch(A, n, &o, pi, pi_w, pi_val, diag, rounds_dev, live, w, (cudaStream_t)stream);
}

size_t lf_linear_forest_workspace_size(int64_t N) {
    Carve c(nullptr, 0);
    return forest_ws_carve(c, N, nullptr) + 256;
}

int lf_linear_forest(int64_t N, const int32_t* pi2, const float* pi2_w, int32_t* forest,
                     int32_t* path_id, int32_t* pos, int32_t* perm, int32_t* iperm, int64_t* n_cycles,
                     void* ws, size_t ws_bytes, void* stream) {
    g_err[0] = 0;
    if (N < 0 || N >= ((int64_t)1 << 31)) return set_error(LF_EINVAL, "lf_linear_forest: bad N");
    if (N > 0 && (!pi2 || !pi2_w || !forest || !path_id || !pos || !perm || !iperm))
        return set_error(LF_EINVAL, "lf_linear_forest: NULL argument");
    if (((uintptr_t)pi2 | (uintptr_t)pi2_w | (uintptr_t)forest) & 7)
        return set_error(LF_EINVAL, "lf_linear_forest: pi2, pi2_w and forest must be 8-byte aligned");
    Carve c(ws, ws_bytes);
    ForestWs w;
    forest_ws_carve(c, N, &w);
    if (N > 0 && (!ws || !c.ok())) return set_error(LF_ENOMEM, "lf_linear_forest: workspace too small");
    return forest_run(N, pi2, pi2_w, forest, path_id, pos, perm, iperm, n_cycles, w, (cudaStream_t)stream);
}

int lf_linear_forest_tridiag(int64_t N, const int32_t* pi2, const float* pi2_w, const float* pi2_val,
                             const float* diag, int32_t* forest, int32_t* path_id, int32_t* pos,
                             int32_t* perm, int32_t* iperm, float* a, float* b, float* c, int64_t* n_cycles,
                             void* ws, size_t ws_bytes, void* stream) {
    g_err[0] = 0;
    if (N < 0 || N >= ((int64_t)1 << 31)) return set_error(LF_EINVAL, "lf_linear_forest_tridiag: bad N");
    if (N > 0 && (!pi2 || !pi2_w || !pi2_val || !diag || !forest || !path_id || !pos || !perm || !iperm || !a ||
                  !b || !c))
        return set_error(LF_EINVAL, "lf_linear_forest_tridiag: NULL argument");
    if (((uintptr_t)pi2 | (uintptr_t)pi2_w | (uintptr_t)pi2_val | (uintptr_t)forest) & 7)
        return set_error(LF_EINVAL, "lf_linear_forest_tridiag: pi2, pi2_w, pi2_val and forest must be 8-byte aligned");
    Carve cv(ws, ws_bytes);
    ForestWs w;
    forest_ws_carve(cv, N, &w);
    if (N > 0 && (!ws || !cv.ok())) return set_error(LF_ENOMEM, "lf_linear_forest_tridiag: workspace too small");
    const TriOut tri{pi2_val, diag, a, b, c};
    return forest_run(N, pi2, pi2_w, forest, path_id, pos, perm, iperm, n_cycles, w, (cudaStream_t)stream, &tri);
}

int lf_forest_stats(int64_t N, void* ws, size_t ws_bytes, int32_t* out, int cap) {
    g_err[0] = 0;
    Carve c(ws, ws_bytes);
    ForestWs w;
    forest_ws_carve(c, N, &w);
    if (!ws || !c.ok()) return set_error(LF_ENOMEM, "lf_forest_stats: workspace too small");
    return forest_stats(w, out, cap);
}

int lf_tridiag(int64_t N, const int32_t* forest, const int32_t* iperm, const int32_t* pi2,
               const float* pi2_val, const float* diag, float* a, float* b, float* c, void* stream) {
    g_err[0] = 0;
    if (N < 0 || N >= ((int64_t)1 << 31)) return set_error(LF_EINVAL, "lf_tridiag: bad N");
    if (N > 0 && (!forest || !iperm || !pi2 || !pi2_val || !diag || !a || !b || !c))
        return set_error(LF_EINVAL, "lf_tridiag: NULL argument");
    if (((uintptr_t)forest | (uintptr_t)pi2 | (uintptr_t)pi2_val) & 7)
        return set_error(LF_EINVAL, "lf_tridiag: forest, pi2 and pi2_val must be 8-byte aligned");
    return tridiag_run(N, forest, iperm, pi2, pi2_val, diag, a, b, c, (cudaStream_t)stream);
}

// device scratch of the host-buffer pipeline: A, factor outputs, forest outputs, stage ws
struct PipeWs {
    int64_t* rowptr;
    int32_t* col;
    float* val;
    int32_t* pi;
    float* pi_w;
    float* pi_val;
    float* diag;
    int32_t* forest;
    int32_t* path_id;
    int32_t* pos;
    int32_t* perm;
    int32_t* iperm;
    float* a;
    float* b;
    float* c;
    void* ws;
    size_t ws_bytes;
};

static size_t pipe_carve(Carve& c, int64_t N, int64_t nnz, PipeWs* p) {
    PipeWs t;
    const size_t n = (size_t)(N > 0 ? N : 1);
    t.rowptr = c.take<int64_t>(n + 1);
    t.col = c.take<int32_t>((size_t)(nnz > 0 ? nnz : 1));
    t.val = c.take<float>((size_t)(nnz > 0 ? nnz : 1));
    t.pi = c.take<int32_t>(2 * n);
    t.pi_w = c.take<float>(2 * n);
    t.pi_val = c.take<float>(2 * n);
    t.diag = c.take<float>(n);
    t.forest = c.take<int32_t>(2 * n);
    t.path_id = c.take<int32_t>(n);
    t.pos = c.take<int32_t>(n);
    t.perm = c.take<int32_t>(n);
    t.iperm = c.take<int32_t>(n);
    t.a = c.take<float>(n);
    t.b = c.take<float>(n);
    t.c = c.take<float>(n);
    const size_t fw = lf_factor_workspace_size(N, 2);
    const size_t lw = lf_linear_forest_workspace_size(N);
    t.ws_bytes = fw > lw ? fw : lw;
    t.ws = c.take<char>(t.ws_bytes);
    if (p) *p = t;
    return c.off;
}

size_t lf_tri_solve_workspace_size(int64_t N) { return N > 0 ? trisolve_ws_bytes(N) : 0; }

int lf_tri_solve(int64_t N, const float* a, const float* b, const float* c, const float* x, float* y,
                 void* ws, size_t ws_bytes, void* stream) {
    g_err[0] = 0;
    if (N < 0 || N >= ((int64_t)1 << 31)) return set_error(LF_EINVAL, "lf_tri_solve: bad N");
    if (N == 0) return LF_OK;
    if (!a || !b || !c || !x || !y) return set_error(LF_EINVAL, "lf_tri_solve: NULL argument");
    if (!ws || ws_bytes < trisolve_ws_bytes(N) || ((uintptr_t)ws & 255))
        return set_error(LF_ENOMEM, "lf_tri_solve: workspace too small or not 256-byte aligned");
    // y is written while a, b, c, x are still being read (other blocks, other segments):
    // any overlap of [y, y+N) with one of them is rejected, not just y == x
    {
        const uintptr_t y0 = (uintptr_t)y, y1 = y0 + (uintptr_t)N * sizeof(float);
        const float* ins[4] = {a, b, c, x};
        for (const float* q : ins) {
            const uintptr_t q0 = (uintptr_t)q, q1 = q0 + (uintptr_t)N * sizeof(float);
            if (q0 < y1 && y0 < q1) return set_error(LF_EINVAL, "lf_tri_solve: y overlaps a, b, c or x");
        }
    }
    return trisolve_run(N, a, b, c, x, y, ws, (cudaStream_t)stream);
}

size_t lf_pipeline_workspace_size(int64_t N, int64_t nnz) {
    Carve c(nullptr, 0);
    return pipe_carve(c, N, nnz, nullptr) + 256;
}

int lf_pipeline_host(const lf_csr_t* Ah, const lf_factor_opts_t* opts, int32_t* perm_h,
                     int32_t* path_id_h, int32_t* pos_h, float* a_h, float* b_h, float* c_h, void* ws,
                     size_t ws_bytes, void* stream) {
    g_err[0] = 0;
    if (!csr_ok(Ah)) return set_error(LF_EINVAL, "lf_pipeline_host: invalid CSR descriptor");
    const int64_t N = Ah->n;
    Carve cv(ws, ws_bytes);
    PipeWs p;
    pipe_carve(cv, N, Ah->nnz, &p);
    if (!ws || !cv.ok()) return set_error(LF_ENOMEM, "lf_pipeline_host: workspace too small");
    cudaStream_t s = (cudaStream_t)stream;
    LF_CUDA(cudaMemcpyAsync(p.rowptr, Ah->rowptr, sizeof(int64_t) * (N + 1), cudaMemcpyHostToDevice, s));
    if (Ah->nnz > 0) {
        LF_CUDA(cudaMemcpyAsync(p.col, Ah->col, sizeof(int32_t) * Ah->nnz, cudaMemcpyHostToDevice, s));
        LF_CUDA(cudaMemcpyAsync(p.val, Ah->val, sizeof(float) * Ah->nnz, cudaMemcpyHostToDevice, s));
    }
    lf_csr_t Ad{N, Ah->nnz, p.rowptr, p.col, p.val};
    int rc = lf_factor(&Ad, 2, opts, p.pi, p.pi_w, p.pi_val, p.diag, nullptr, nullptr, p.ws, p.ws_bytes, stream);
    if (rc) return rc;
    rc = lf_linear_forest_tridiag(N, p.pi, p.pi_w, p.pi_val, p.diag, p.forest, p.path_id, p.pos, p.perm,
                                  p.iperm, p.a, p.b, p.c, nullptr, p.ws, p.ws_bytes, stream);
    if (rc) return rc;
    struct {
        void* h;
        const void* d;
        size_t bytes;
    } outs[6] = {{perm_h, p.perm, 4}, {path_id_h, p.path_id, 4}, {pos_h, p.pos, 4},
                 {a_h, p.a, 4},       {b_h, p.b, 4},             {c_h, p.c, 4}};
    for (auto& o : outs)
        if (o.h && N > 0) LF_CUDA(cudaMemcpyAsync(o.h, o.d, o.bytes * N, cudaMemcpyDeviceToHost, s));
    LF_CUDA(cudaStreamSynchronize(s));
    return LF_OK;
}

int lf_validate_csr(const lf_csr_t* A, void* ws, size_t ws_bytes, void* stream) {
    g_err[0] = 0;
    if (!csr_ok(A)) return set_error(LF_EINVAL, "lf_validate_csr: invalid CSR descriptor");
    if (!ws || ws_bytes < sizeof(int)) return set_error(LF_ENOMEM, "lf_validate_csr: workspace too small");
    cudaStream_t s = (cudaStream_t)stream;
    if (!ws || ws_bytes < lf_validate_workspace_size(A->n) || ((uintptr_t)ws & 255))
        return set_error(LF_ENOMEM, "lf_validate_csr: workspace smaller than lf_validate_workspace_size(N)");
    int* bad = (int*)ws;
    uint8_t* sorted = (uint8_t*)ws + 256;
    LF_CUDA(cudaMemsetAsync(bad, 0, sizeof(int), s));
    k_validate<<<persistent_grid((const void*)k_validate, 256), 256, 0, s>>>(A->n, A->nnz, A->rowptr, A->col,
                                                                         A->val, bad, sorted);
    LF_CUDA(cudaGetLastError());
    k_validate_sym<<<persistent_grid((const void*)k_validate_sym, 256), 256, 0, s>>>(A->n, A->nnz, A->rowptr,
                                                                                 A->col, A->val, bad, sorted);
    LF_CUDA(cudaGetLastError());
    int h = 0;
    LF_CUDA(cudaMemcpyAsync(&h, bad, sizeof(int), cudaMemcpyDeviceToHost, s));
    LF_CUDA(cudaStreamSynchronize(s));
    if (h & 1) return set_error(LF_EINPUT, "lf_validate_csr: rowptr not monotone or wrong ends");
    if (h & 2) return set_error(LF_EINPUT, "lf_validate_csr: column index out of range");
    if (h & 4) return set_error(LF_EINPUT, "lf_validate_csr: NaN or Inf value");
    if (h & 8) return set_error(LF_EINPUT, "lf_validate_csr: duplicate (i,j) entry");
    if (h & 16) return set_error(LF_EINPUT, "lf_validate_csr: pattern not symmetric (edge (i,j) without (j,i))");
    if (h & 32) return set_error(LF_EINPUT, "lf_validate_csr: |a_ij| != |a_ji| (values not symmetric)");
    return LF_OK;
}

size_t lf_validate_workspace_size(int64_t N) { return 256 + (size_t)(N > 0 ? N : 0) + 256; }

int lf_validate_factor(int64_t N, int n, const int32_t* pi, void* ws, size_t ws_bytes, void* stream) {
    g_err[0] = 0;
    cudaStream_t s = (cudaStream_t)stream;
    if (N < 0 || N >= ((int64_t)1 << 31)) return set_error(LF_EINVAL, "lf_validate_factor: bad N");
    if (n < 1 || n > 4) return set_error(LF_EINVAL, "lf_validate_factor: n must be in [1,4]");
    if (N == 0) return LF_OK;
    if (!pi) return set_error(LF_EINVAL, "lf_validate_factor: NULL pi");
    if (!ws || ws_bytes < 256 || ((uintptr_t)ws & 255))
        return set_error(LF_ENOMEM, "lf_validate_factor: workspace smaller than 256 bytes");
    int* bad = (int*)ws;
    LF_CUDA(cudaMemsetAsync(bad, 0, sizeof(int), s));
    k_validate_factor<<<persistent_grid((const void*)k_validate_factor, 256), 256, 0, s>>>(N, n, pi, bad);
    LF_CUDA(cudaGetLastError());
    int h = 0;
    LF_CUDA(cudaMemcpyAsync(&h, bad, sizeof(int), cudaMemcpyDeviceToHost, s));
    LF_CUDA(cudaStreamSynchronize(s));
    if (h & 64) return set_error(LF_EINPUT, "lf_validate_factor: bad slot (id range, self loop, order or repeat)");
    if (h & 128) return set_error(LF_EINPUT, "lf_validate_factor: not symmetric (w in pi(v) but v not in pi(w))");
    return LF_OK;
}

}  // extern "C"

// Diagnostics only (not part of include/lf.h): per-kernel timeline of LF_TIMELINE builds.
// out[0..15] factor kernels, out[16..47] forest kernels; reset != 0 clears.  -1 otherwise.
extern "C" int lf_debug_timeline(unsigned long long* out, int reset) {
    if (reset) return lf::timeline_factor(nullptr, 1) | lf::timeline_forest(nullptr, 1);
    return lf::timeline_factor(out, 0) | lf::timeline_forest(out + 16, 0);
}
