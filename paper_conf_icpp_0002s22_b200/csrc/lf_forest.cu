// lf_forest.cu -- linear forest from a [0,2]-factor (§3.3,
// Algorithm 3, §4.2, §4.3).
//
// Both scans are the paper's bidirectional pointer-jumping scan (no orientation, no
// random-access iterator), run as ONE cooperative persistent kernel each instead of
// ceil(log2 N) launches: the grid iterates stride-doubling steps separated by grid-wide
// barriers over ping-pong buffers (L249) and leaves as soon as every vertex is done,
// i.e. after ceil(log2 L_max)+O(1) steps for the longest component L_max rather than
// ceil(log2 N).
//   cycle scan (step (1), L225, L245-L247): per direction the stride pointer and the
//     minimum edge key seen.  A path vertex is done when both pointers are path-end
//     markers -(e+1) (L245).  A cycle vertex is done when its two windows share the
//     cycle's weakest edge (equal minima) or both pointers coincide: then the union of
//     its windows is the whole cycle.  Every cycle vertex then knows the weakest edge;
//     its two endpoints drop it.
//   rank scan (step (2), Alg. 3): per direction the pointer and the position sum r.
//     l(v) = smaller end ID, p(v) = r toward that end (L223).
//   permutation (step (3)): path length at the path-ID vertex, exclusive scan (CUB),
//     new(v) = off[l(v)] + p(v) - 1 -- the same order as sorting by (l, p) (L297).
#include <cooperative_groups.h>
#include <cuda_runtime.h>

#include <cub/device/device_scan.cuh>
#include <cstdint>

#include "lf_common.cuh"
#include "lf_internal.h"

namespace cg = cooperative_groups;

namespace lf {

constexpr uint64_t KEY_INF = ~0ull;
constexpr int kCtlCycle = 0;    // ctl[0..63]  per-step not-done counts of the cycle scan
constexpr int kCtlRank = 64;    // ctl[64..127] rank scan
constexpr int kMaxSteps = 62;

__device__ __forceinline__ int block_reduce_add(int x, int* sh) {
    // sh: 32 ints of shared memory
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
#pragma unroll
    for (int o = 16; o; o >>= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
    if (lane == 0) sh[wid] = x;
    __syncthreads();
    int t = 0;
    if (threadIdx.x < 32) {
        t = (threadIdx.x < (blockDim.x >> 5)) ? sh[threadIdx.x] : 0;
#pragma unroll
        for (int o = 16; o; o >>= 1) t += __shfl_xor_sync(0xffffffffu, t, o);
    }
    __syncthreads();
    return t;  // valid in thread 0
}

// key of the edge {u,x} for the weakest-edge search: minimise (|w| bits, -rank), where
// rank orders edges by (min, max) lexicographically: rank = 2*min + c, c = 1 iff max is
// the larger of min's two higher neighbours (DESIGN.md §3 reading c9).
__device__ __forceinline__ uint64_t edge_key(const int2* __restrict__ nb, int32_t v, int32_t w,
                                             float wabs, int2 nbv) {
    const int32_t u = v < w ? v : w;
    const int32_t x = v < w ? w : v;
    const int2 nu = (u == v) ? nbv : nb[u];
    const int32_t y = (nu.x == x) ? nu.y : nu.x;  // u's other neighbour
    const uint32_t c = (y > u && y < x) ? 1u : 0u;
    const uint32_t rank = 2u * (uint32_t)u + c;
    return ((uint64_t)__float_as_uint(wabs) << 32) | (uint64_t)(0xFFFFFFFFu - rank);
}

__device__ __forceinline__ uint64_t umin64(uint64_t a, uint64_t b) { return a < b ? a : b; }

struct CycleArgs {
    int64_t N;
    const int2* __restrict__ pi2;     // [N] slots as int2
    const float2* __restrict__ pi2_w;
    int2* q0;
    int2* q1;
    ulonglong2* m0;
    ulonglong2* m1;
    ulonglong2* ekey;                 // [N] key of each slot's edge
    int2* forest;
    int* ctl;
    unsigned long long* n_cycles;     // may be NULL
    int max_steps;
};

__global__ void __launch_bounds__(256) k_cycle_scan(CycleArgs a) {
    __shared__ int sh[32];
    cg::grid_group grid = cg::this_grid();
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    const int64_t t0 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    // init (Alg. 3 L1-L4 analogue): stride-1 neighbours or end markers, edge keys
    for (int64_t v = t0; v < a.N; v += stride) {
        const int2 nb = a.pi2[v];
        const float2 wv = a.pi2_w[v];
        ulonglong2 k;
        k.x = nb.x >= 0 ? edge_key(a.pi2, (int32_t)v, nb.x, wv.x, nb) : KEY_INF;
        k.y = nb.y >= 0 ? edge_key(a.pi2, (int32_t)v, nb.y, wv.y, nb) : KEY_INF;
        a.ekey[v] = k;
        int2 q;
        q.x = nb.x >= 0 ? nb.x : -(int32_t)(v + 1);
        q.y = nb.y >= 0 ? nb.y : -(int32_t)(v + 1);
        a.q0[v] = q;
        a.m0[v] = k;
        a.q1[v] = q;   // a vertex final from the start must be final in both buffers
        a.m1[v] = k;
    }
    grid.sync();
    int step = 0;
    for (; step < a.max_steps; step++) {
        const int2* qs = (step & 1) ? a.q1 : a.q0;
        const ulonglong2* ms = (step & 1) ? a.m1 : a.m0;
        int2* qd = (step & 1) ? a.q0 : a.q1;
        ulonglong2* md = (step & 1) ? a.m0 : a.m1;
        int notdone = 0;
        for (int64_t v = t0; v < a.N; v += stride) {
            const int2 q = qs[v];
            if (q.x < 0 && q.y < 0) {
                // path vertex, final: make sure the other buffer holds the same values
                const int2 qo = qd[v];
                if (qo.x != q.x || qo.y != q.y) {
                    qd[v] = q;
                    md[v] = ms[v];
                }
                continue;
            }
            ulonglong2 m = ms[v];
            int2 nq = q;
            ulonglong2 nm = m;
            if (q.x >= 0) {  // Alg. 3 L12-L20 with the min operator
                const int2 qw = qs[q.x];
                const ulonglong2 mw = ms[q.x];
                if (qw.x != (int32_t)v) { nq.x = qw.x; nm.x = umin64(m.x, mw.x); }
                else if (qw.y != (int32_t)v) { nq.x = qw.y; nm.x = umin64(m.x, mw.y); }
            }
            if (q.y >= 0) {
                const int2 qw = qs[q.y];
                const ulonglong2 mw = ms[q.y];
                if (qw.x != (int32_t)v) { nq.y = qw.x; nm.y = umin64(m.y, mw.x); }
                else if (qw.y != (int32_t)v) { nq.y = qw.y; nm.y = umin64(m.y, mw.y); }
            }
            qd[v] = nq;
            md[v] = nm;
            const bool path_done = nq.x < 0 && nq.y < 0;
            const bool cyc_done = nq.x >= 0 && nq.y >= 0 && (nm.x == nm.y || nq.x == nq.y);
            notdone += (path_done || cyc_done) ? 0 : 1;
        }
        const int tot = block_reduce_add(notdone, sh);
        if (threadIdx.x == 0 && tot) atomicAdd(&a.ctl[kCtlCycle + step], tot);
        grid.sync();
        if (*(volatile int*)&a.ctl[kCtlCycle + step] == 0) { step++; break; }
    }
    // results are in the buffer written by the last step
    const int2* qf = (step & 1) ? a.q1 : a.q0;
    const ulonglong2* mf = (step & 1) ? a.m1 : a.m0;
    unsigned long long ncyc = 0;
    for (int64_t v = t0; v < a.N; v += stride) {
        int2 f = a.pi2[v];
        const int2 q = qf[v];
        if (q.x >= 0 && q.y >= 0) {  // on a cycle (L245): drop the weakest edge
            const ulonglong2 m = mf[v];
            const uint64_t kmin = umin64(m.x, m.y);
            const ulonglong2 ek = a.ekey[v];
            if (ek.x == kmin) {
                f.x = f.y;
                f.y = -1;
                if ((int32_t)v < a.pi2[v].x) ncyc++;
            } else if (ek.y == kmin) {
                if ((int32_t)v < f.y) ncyc++;
                f.y = -1;
            }
        }
        a.forest[v] = f;
    }
    if (a.n_cycles) {
#pragma unroll
        for (int o = 16; o; o >>= 1) ncyc += __shfl_xor_sync(0xffffffffu, ncyc, o);
        if ((threadIdx.x & 31) == 0 && ncyc) atomicAdd(a.n_cycles, ncyc);
    }
}

struct RankArgs {
    int64_t N;
    const int2* __restrict__ forest;
    int2* q0;
    int2* q1;
    int2* r0;
    int2* r1;
    int32_t* path_id;
    int32_t* pos;
    int32_t* len;
    int* ctl;
    int max_steps;
};

__global__ void __launch_bounds__(256) k_rank_scan(RankArgs a) {
    __shared__ int sh[32];
    cg::grid_group grid = cg::this_grid();
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    const int64_t t0 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    for (int64_t v = t0; v < a.N; v += stride) {  // Alg. 3 L1-L4
        const int2 f = a.forest[v];
        int2 q;
        q.x = f.x >= 0 ? f.x : -(int32_t)(v + 1);
        q.y = f.y >= 0 ? f.y : -(int32_t)(v + 1);
        const int2 one = make_int2(1, 1);
        a.q0[v] = q;
        a.r0[v] = one;
        a.q1[v] = q;
        a.r1[v] = one;
    }
    grid.sync();
    int step = 0;
    for (; step < a.max_steps; step++) {  // Alg. 3 L5-L26
        const int2* qs = (step & 1) ? a.q1 : a.q0;
        const int2* rs = (step & 1) ? a.r1 : a.r0;
        int2* qd = (step & 1) ? a.q0 : a.q1;
        int2* rd = (step & 1) ? a.r0 : a.r1;
        int notdone = 0;
        for (int64_t v = t0; v < a.N; v += stride) {
            const int2 q = qs[v];
            if (q.x < 0 && q.y < 0) {
                const int2 qo = qd[v];
                if (qo.x != q.x || qo.y != q.y) {
                    qd[v] = q;
                    rd[v] = rs[v];
                }
                continue;
            }
            const int2 r = rs[v];
            int2 nq = q, nr = r;
            if (q.x >= 0) {
                const int2 qw = qs[q.x];
                const int2 rw = rs[q.x];
                if (qw.x != (int32_t)v) { nq.x = qw.x; nr.x = r.x + rw.x; }       // L16-L18
                else if (qw.y != (int32_t)v) { nq.x = qw.y; nr.x = r.x + rw.y; }
            }
            if (q.y >= 0) {
                const int2 qw = qs[q.y];
                const int2 rw = rs[q.y];
                if (qw.x != (int32_t)v) { nq.y = qw.x; nr.y = r.y + rw.x; }
                else if (qw.y != (int32_t)v) { nq.y = qw.y; nr.y = r.y + rw.y; }
            }
            qd[v] = nq;
            rd[v] = nr;
            notdone += (nq.x < 0 && nq.y < 0) ? 0 : 1;
        }
        const int tot = block_reduce_add(notdone, sh);
        if (threadIdx.x == 0 && tot) atomicAdd(&a.ctl[kCtlRank + step], tot);
        grid.sync();
        if (*(volatile int*)&a.ctl[kCtlRank + step] == 0) { step++; break; }
    }
    const int2* qf = (step & 1) ? a.q1 : a.q0;
    const int2* rf = (step & 1) ? a.r1 : a.r0;
    for (int64_t v = t0; v < a.N; v += stride) {  // Alg. 3 L27-L33 with l = min end (L223)
        const int2 q = qf[v];
        const int2 r = rf[v];
        const int32_t e0 = -(q.x + 1), e1 = -(q.y + 1);
        int32_t l, p;
        if (e0 <= e1) { l = e0; p = r.x; } else { l = e1; p = r.y; }
        a.path_id[v] = l;
        a.pos[v] = p;
        a.len[v] = (l == (int32_t)v) ? (r.x + r.y - 1) : 0;
    }
}

// step (3): new(v) = off[l(v)] + p(v) - 1
__global__ void k_perm(int64_t N, const int32_t* __restrict__ path_id, const int32_t* __restrict__ pos,
                       const int32_t* __restrict__ off, int32_t* perm, int32_t* iperm) {
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < N;
         v += (int64_t)gridDim.x * blockDim.x) {
        const int32_t r = __ldg(off + __ldg(path_id + v)) + __ldg(pos + v) - 1;
        iperm[v] = r;
        perm[r] = (int32_t)v;
    }
}

static size_t scan_temp_bytes(int64_t N) {
    // CUB's decoupled look-back scan needs one tile descriptor per tile (~1-2k items) plus
    // padding.  The query below can fail (it reports a pending CUDA error of an unrelated
    // earlier call), so the workspace uses a bound that covers it: 16 B per 64 items.
    const size_t bound = 16 * ((size_t)(N > 0 ? N : 1) / 64 + 256) + 4096;
    size_t b = 0;
    cudaError_t e = cub::DeviceScan::ExclusiveSum(nullptr, b, (const int32_t*)nullptr, (int32_t*)nullptr,
                                                  (int)(N > 0 ? N : 1));
    if (e != cudaSuccess) return bound;
    return b > bound ? b : bound;
}

size_t forest_ws_carve(Carve& c, int64_t N, ForestWs* w) {
    ForestWs t;
    const size_t n = (size_t)(N > 0 ? N : 1);
    t.q[0] = c.take<int32_t>(2 * n);
    t.q[1] = c.take<int32_t>(2 * n);
    t.mk[0] = c.take<uint64_t>(2 * n);
    t.mk[1] = c.take<uint64_t>(2 * n);
    // the rank scan reuses the min-key buffers for r (8 bytes per vertex each)
    t.r[0] = (int32_t*)t.mk[0];
    t.r[1] = (int32_t*)t.mk[1];
    t.ekey = c.take<uint64_t>(2 * n);
    t.len = c.take<int32_t>(n);
    t.off = c.take<int32_t>(n);
    t.ctl = c.take<int>(256);
    t.scan_tmp_bytes = scan_temp_bytes(N);
    t.scan_tmp = c.take<char>(t.scan_tmp_bytes);
    if (w) *w = t;
    return c.off;
}

static int max_steps_for(int64_t N) {
    int s = 0;
    while (s < 40 && ((int64_t)1 << s) < N) s++;
    return s + 3;  // ceil(log2 N) + margin for cycle detection and the final copy
}

int forest_run(int64_t N, const int32_t* pi2, const float* pi2_w, int32_t* forest, int32_t* path_id,
               int32_t* pos, int32_t* perm, int32_t* iperm, int64_t* n_cycles, const ForestWs& w,
               cudaStream_t s) {
    if (N == 0) {
        if (n_cycles) LF_CUDA(cudaMemsetAsync(n_cycles, 0, sizeof(int64_t), s));
        return LF_OK;
    }
    LF_CUDA(cudaMemsetAsync(w.ctl, 0, sizeof(int) * 256, s));
    if (n_cycles) LF_CUDA(cudaMemsetAsync(n_cycles, 0, sizeof(int64_t), s));
    const int steps = max_steps_for(N) < kMaxSteps ? max_steps_for(N) : kMaxSteps;
    {
        CycleArgs a;
        a.N = N;
        a.pi2 = (const int2*)pi2;
        a.pi2_w = (const float2*)pi2_w;
        a.q0 = (int2*)w.q[0];
        a.q1 = (int2*)w.q[1];
        a.m0 = (ulonglong2*)w.mk[0];
        a.m1 = (ulonglong2*)w.mk[1];
        a.ekey = (ulonglong2*)w.ekey;
        a.forest = (int2*)forest;
        a.ctl = w.ctl;
        a.n_cycles = (unsigned long long*)n_cycles;
        a.max_steps = steps;
        const int grid = persistent_grid((const void*)k_cycle_scan, 256);
        void* args[] = {&a};
        LF_PROF("cycle_scan", -1, s);
        LF_CUDA(cudaLaunchCooperativeKernel((const void*)k_cycle_scan, grid, 256, args, 0, s));
    }
    {
        RankArgs a;
        a.N = N;
        a.forest = (const int2*)forest;
        a.q0 = (int2*)w.q[0];
        a.q1 = (int2*)w.q[1];
        a.r0 = (int2*)w.r[0];
        a.r1 = (int2*)w.r[1];
        a.path_id = path_id;
        a.pos = pos;
        a.len = w.len;
        a.ctl = w.ctl;
        a.max_steps = steps;
        const int grid = persistent_grid((const void*)k_rank_scan, 256);
        void* args[] = {&a};
        LF_PROF("rank_scan", -1, s);
        LF_CUDA(cudaLaunchCooperativeKernel((const void*)k_rank_scan, grid, 256, args, 0, s));
    }
    {
        LF_PROF("path_offsets", -1, s);
        size_t tb = w.scan_tmp_bytes;
        LF_CUDA(cub::DeviceScan::ExclusiveSum(w.scan_tmp, tb, w.len, w.off, (int)N, s));
    }
    {
        LF_PROF("perm", -1, s);
        k_perm<<<persistent_grid((const void*)k_perm, 256), 256, 0, s>>>(N, path_id, pos, w.off, perm, iperm);
        LF_CUDA(cudaGetLastError());
    }
    return LF_OK;
}

}  // namespace lf
