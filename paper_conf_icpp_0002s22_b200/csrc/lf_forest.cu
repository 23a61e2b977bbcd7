// lf_forest.cu -- linear forest from a [0,2]-factor (§3.3,
// Algorithm 3, §4.2, §4.3).
//
// The paper runs its bidirectional scan (stride-doubling pointer jumping over the
// unoriented doubly-linked list, end markers -(e+1), ping-pong buffers) as ceil(log2 N)
// global launches over all N vertices, twice (cycles, then positions).  Here every scan
// level carries the FULL window of a vertex per direction (pointer, edges covered, minimum
// edge key, DK = distance to that edge's near endpoint), so ONE pass breaks the cycles and
// ranks the paths, in one of two organisations:
//
//   tile path (graphs whose paths stay in 1024-id tiles: C1-C3) -- k_lf_full1 ranks each
//     tile in shared memory (run contraction + ruling set) and emits one record per
//     boundary vertex; k_red_full scans that reduced list (one cluster through DSMEM, or
//     the whole grid, cooperative launch); k_lf_full2 expands; k_tile_prefix + k_perm_tri
//     write the permutation and the tridiagonal copy;
//   global ruling set (paths that leave every tile: C4, C5) -- k_grs_pack +
//     k_grs_list (16-byte records, splitter list in id order), k_grs_walk + k_grs_meet
//     (splitter-to-splitter walks that claim every vertex with its walk and distance),
//     k_red_full on the splitter list, k_grs_len / k_grs_cyccand / k_grs_cycfind /
//     k_grs_lenscan (path offsets, splitter-free cycles), k_grs_desc (walk descriptors),
//     k_grs_emit (one coalesced pass over the vertices) and k_grs_split.
//
// The row-partitioned multi-GPU path (forest_part_run) still uses the older two-pass
// kernels k_lf_local1/2/3 + k_red_scan: its exit-record exchange is built on them.
#include <cooperative_groups.h>
#include <cuda_runtime.h>

#include <cub/device/device_scan.cuh>
#include <cstdint>
#include <climits>
#include <cstdlib>
#include <cstring>

#include "lf_common.cuh"
#include "lf_internal.h"

namespace cg = cooperative_groups;

namespace lf {

#ifdef LF_TIMELINE
__device__ unsigned long long g_tl_forest[32];
#endif

constexpr uint64_t KEY_INF = ~0ull;
// 1024-vertex tiles, 512 threads: two tile-pass CTAs per SM (92 KB of shared memory each)
// overlap one tile's barriers and loads with the other's work (measured on C2: 1024/512/2
// beats 2048/1024/1 by 6 us per step even though the boundary list grows by half)
#ifndef LF_LB
#define LF_LB 1024
#endif
#ifndef LF_LT
#define LF_LT 512
#endif
#ifndef LF_LMINB
#define LF_LMINB 3    // expand / local2 CTAs per SM (4: register spills)
#endif
#ifndef LF_F1MINB
#define LF_F1MINB 2   // resident tile-pass CTAs per SM (k_lf_full1)
#endif
constexpr int LB = LF_LB;         // vertices per block-local tile
constexpr int LT = LF_LT;         // threads per tile CTA
constexpr int VPT = LB / LT;      // vertices per thread
constexpr int kCtlRed1 = 0;       // ctl[0..63]   per-step not-done counts, reduced scan 1
constexpr int kCtlRed2 = 64;      // ctl[64..127] reduced scan 2
constexpr int kCtlCnt1 = 128;     // boundary list sizes
constexpr int kCtlCnt2 = 129;
constexpr int kCtlTicket3 = 130;  // finished-CTA ticket of k_path_offsets / k_lf_full2 (the last one scans tsum)
constexpr int kCtlNcyc = 131;     // broken cycles (single-pass forest)
constexpr int kCtlGridBar = 133;  // arrival counter of k_red_full's grid barrier
constexpr int kCtlBad = 135;      // the tile path met a malformed factor: later kernels leave
constexpr int kCtlBadGrs = 136;   // a ruling-set walk met one (bounded; records stay well formed)
constexpr int kCtlCycMax = 138;   // longest splitter-free cycle (lf_forest_stats)
#ifndef LF_WALK_CTRS
#define LF_WALK_CTRS 4
#endif
constexpr int kCycStripes = 32;   // counters of the splitter-free cycles (k_grs_cycfind),
constexpr int kCtlCycS = 256;     //   ctl[256 + 32 s]: one 128-byte line each (atomics on one
constexpr int kCtlCycStride = 32; //   line queue behind each other in its L2 slice)
constexpr int kWalkCtrs = LF_WALK_CTRS;  // schedule counters of k_grs_walk, one line each
constexpr int kCtlWalkC = 256 + kCycStripes * kCtlCycStride;
constexpr int kCtlInts = kCtlWalkC + 4 * kCtlCycStride;
constexpr int kCtlCand = 139;     // candidates of k_grs_cyccand (list2)
constexpr int kMaxSteps = 62;
constexpr int kCtlStat = 192;     // ctl[192..]: diagnostics (lf_forest_stats)
// ctl[192] splitter nodes (cycle pass), [193] unvisited vertices (fallback), [194] tiles
// that needed the fallback, [195] splitter nodes (rank pass), [196] max node-scan steps

__device__ __forceinline__ uint64_t umin64(uint64_t a, uint64_t b) { return a < b ? a : b; }

// optional per-phase cycle accounting of the tile kernels (build with -DLF_PHASE_TIMING;
// accumulated into ctl[208 + phase], read with lf_forest_stats' extended slots)
#ifdef LF_PHASE_TIMING
#define LF_PHASE(ctl, i)                                                              \
    do {                                                                              \
        __syncthreads();                                                              \
        if (threadIdx.x == 0) {                                                       \
            const long long t_ = clock64();                                           \
            atomicAdd((unsigned long long*)&(ctl)[208 + 2 * (i)], (unsigned long long)(t_ - ph_t)); \
            ph_t = t_;                                                                \
        }                                                                             \
    } while (0)
#define LF_PHASE_INIT long long ph_t = clock64()
#else
#define LF_PHASE(ctl, i) do { } while (0)
#define LF_PHASE_INIT do { } while (0)
#endif

// Global key of edge {v,w} for the weakest-edge search, minimised: (|w| bits, -rank), rank
// = 2*min + c orders edges by (min, max) lexicographically (c = 1 iff max is the larger of
// min's two higher neighbours).  Realises reading c9 (ties -> larger (min,max) is weaker).
__device__ __forceinline__ uint64_t edge_key(int32_t v, int32_t w, float wabs, int2 nb_min) {
    const int32_t u = v < w ? v : w;
    const int32_t x = v < w ? w : v;
    const int32_t y = (nb_min.x == x) ? nb_min.y : nb_min.x;  // min endpoint's other neighbour
    const uint32_t c = (y > u && y < x) ? 1u : 0u;
    const uint32_t rank = 2u * (uint32_t)u + c;
    return ((uint64_t)__float_as_uint(wabs) << 32) | (uint64_t)(0xFFFFFFFFu - rank);
}

// shared-memory state of one tile
struct TileSmem {
    int2 nb[LB];          // global neighbours (slot order), -1 = none; run slots virtual
    union {
        float2 w[LB];     // |w| per slot (cycle pass; read by slot_keys before tile_rank)
        struct {
            short2 run[LB];  // (first, last) local vertex of the run of u
            short2 vw[LB];   // edges behind each slot (a run jump spans the run)
        } r;
    };
    short2 P[LB];         // stride pointer per direction (vertex or splitter node), or marker
    short2 R[LB];         // edges covered per direction (rank pass)
    uint64_t K0[LB];      // min edge key, direction 0 (cycle pass)
    uint64_t K1[LB];      // min edge key, direction 1
    short sidx[LB];       // splitter node index of a vertex, -1 if not a splitter
    short spl[LB];        // local vertex of each splitter node
    short2 recS[LB];      // per face: (node << 1 | start slot) of the walk that visited it
    short2 recD[LB];      // per face: distance to that node
    int nspl;             // number of splitter nodes
    int32_t b0, tend;     // first vertex of the tile, one past its last (own range end)
    // cycle pass only (kernels of the rank pass allocate the struct without these)
    uint64_t EK0[LB];     // key of the (virtual) link behind slot 0 / slot 1
    uint64_t EK1[LB];
};
constexpr size_t kTileSmemNoKeys = offsetof(TileSmem, EK0);

// x lies in this tile (the tile never extends past the own range [lo, hi))
// the tile's range in registers (read once from shared memory)
struct Tile {
    int32_t b0, tend;
};
template <class S>
__device__ __forceinline__ Tile tile_of(const S& s) { return Tile{s.b0, s.tend}; }
__device__ __forceinline__ bool is_local(int32_t x, const Tile& t) {
    return (uint32_t)(x - t.b0) < (uint32_t)(t.tend - t.b0);
}

// Bidirectional scan inside the tile (Alg. 3, or its min variant when MINK, restricted
// to local links: a missing or non-local neighbour ends the walk like a path end).
// Each thread keeps its own vertices' state in registers and publishes it to shared
// memory for its neighbours; vertices whose both pointers are terminal markers are final
// and drop out (markers are absorbing, so their published state stays valid).  Cycle
// vertices keep stepping until the whole tile is done (their neighbours read them).
// On return P[k] holds, per direction, a terminal marker -(t+1) (t local) or, on a
// completed local cycle, non-negative pointers; R[k] the local distances (rank pass);
// K[k] the min edge keys (cycle pass).  ek: keys of the own vertices' slots.
template <bool MINK>
__device__ __noinline__ void tile_scan(TileSmem& s, int32_t b0, const ulonglong2 (&ek)[VPT], int2 (&P)[VPT],
                          int2 (&R)[VPT], ulonglong2 (&K)[VPT], const bool (&skip)[VPT]) {
    const int tid = threadIdx.x;
    const Tile T = tile_of(s);
    bool fin[VPT];
#pragma unroll
    for (int k = 0; k < VPT; k++) {
        const int u = tid + k * LT;
        if (skip[k]) { fin[k] = true; continue; }
        const int2 nb = s.nb[u];
        const bool l0 = nb.x >= 0 && is_local(nb.x, T);
        const bool l1 = nb.y >= 0 && is_local(nb.y, T);
        P[k] = make_int2(l0 ? nb.x - b0 : -(u + 1), l1 ? nb.y - b0 : -(u + 1));
        fin[k] = !l0 && !l1;
        s.P[u] = make_short2((short)P[k].x, (short)P[k].y);
        if (MINK) {
            K[k].x = l0 ? ek[k].x : KEY_INF;
            K[k].y = l1 ? ek[k].y : KEY_INF;
            s.K0[u] = K[k].x;
            s.K1[u] = K[k].y;
        } else {
            R[k] = make_int2(l0 ? 1 : 0, l1 ? 1 : 0);
            s.R[u] = make_short2((short)R[k].x, (short)R[k].y);
        }
    }
    int notdone = 0;
#pragma unroll
    for (int k = 0; k < VPT; k++) notdone |= !fin[k];
    if (!__syncthreads_or(notdone)) return;
    for (int step = 0; step < 16; step++) {
        int2 nP[VPT], nR[VPT];
        ulonglong2 nK[VPT];
#pragma unroll
        for (int k = 0; k < VPT; k++) {
            const int u = tid + k * LT;
            nP[k] = P[k];
            if (MINK) nK[k] = K[k]; else nR[k] = R[k];
            if (fin[k]) continue;
#pragma unroll
            for (int i = 0; i < 2; i++) {
                const int w = i ? P[k].y : P[k].x;
                if (w < 0) continue;
                const short2 pw = s.P[w];
                int j = -1;
                if (pw.x != u) j = 0;
                else if (pw.y != u) j = 1;
                if (j < 0) continue;  // stall (reading c13)
                const int tgt = j ? pw.y : pw.x;
                if (i) nP[k].y = tgt; else nP[k].x = tgt;
                if (MINK) {
                    const uint64_t kv = j ? s.K1[w] : s.K0[w];
                    if (i) nK[k].y = umin64(nK[k].y, kv); else nK[k].x = umin64(nK[k].x, kv);
                } else {
                    const short2 rw = s.R[w];
                    const int dv = j ? rw.y : rw.x;
                    if (i) nR[k].y += dv; else nR[k].x += dv;
                }
            }
        }
        __syncthreads();
        notdone = 0;
#pragma unroll
        for (int k = 0; k < VPT; k++) {
            if (fin[k]) continue;
            const int u = tid + k * LT;
            P[k] = nP[k];
            s.P[u] = make_short2((short)P[k].x, (short)P[k].y);
            if (MINK) {
                K[k] = nK[k];
                s.K0[u] = K[k].x;
                s.K1[u] = K[k].y;
            } else {
                R[k] = nR[k];
                s.R[u] = make_short2((short)R[k].x, (short)R[k].y);
            }
            fin[k] = P[k].x < 0 && P[k].y < 0;
            bool cyc_done = false;
            if (MINK) cyc_done = P[k].x >= 0 && P[k].y >= 0 && (K[k].x == K[k].y || P[k].x == P[k].y);
            notdone |= !(fin[k] || cyc_done);
        }
        if (!__syncthreads_or(notdone)) break;
    }
}

constexpr int kSplitShift = 29;  // splitter density 1/8 from the top 3 bits of a hash

__device__ __forceinline__ bool hashed_splitter(int32_t g) {
    return (((uint32_t)g * 0x9E3779B1u) >> kSplitShift) == 0u;
}

// block-wide inclusive scans over LB values, thread t owning u = VPT*t .. VPT*t+VPT-1
__device__ __forceinline__ int block_scan_max(int x, int* sh) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x = max(x, y);
    }
    if (lane == 31) sh[w] = x;
    __syncthreads();
    if (w == 0) {
        int t = lane < LT / 32 ? sh[lane] : INT_MIN;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int y = __shfl_up_sync(0xffffffffu, t, o);
            if (lane >= o) t = max(t, y);
        }
        if (lane < LT / 32) sh[lane] = t;
    }
    __syncthreads();
    const int pre = w > 0 ? sh[w - 1] : INT_MIN;
    __syncthreads();
    return max(x, pre);
}

// exclusive block max-scan (over threads 0..tid-1), INT_MIN for thread 0
__device__ __forceinline__ int block_scan_max_excl(int x, int* sh) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    int inc = x;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int y = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane >= o) inc = max(inc, y);
    }
    int exc = __shfl_up_sync(0xffffffffu, inc, 1);
    if (lane == 0) exc = INT_MIN;
    if (lane == 31) sh[w] = inc;
    __syncthreads();
    if (w == 0) {
        int t = lane < LT / 32 ? sh[lane] : INT_MIN;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int y = __shfl_up_sync(0xffffffffu, t, o);
            if (lane >= o) t = max(t, y);
        }
        if (lane < LT / 32) sh[lane] = t;
    }
    __syncthreads();
    return w > 0 ? max(exc, sh[w - 1]) : exc;
}

// exclusive block sum-scan with a single barrier: each warp reads the other warps' sums
// itself.  *total = the block's sum.  sh must not be reused before another barrier.
__device__ __forceinline__ int block_scan_sum_excl1(int x, int* sh, int* total) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int nw = (int)(blockDim.x >> 5);
    int inc = x;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int y = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane >= o) inc += y;
    }
    if (lane == 31) sh[w] = inc;
    __syncthreads();
    const int ws = lane < nw ? sh[lane] : 0;
    int before = lane < w ? ws : 0, all = ws;
#pragma unroll
    for (int o = 16; o; o >>= 1) {
        before += __shfl_xor_sync(0xffffffffu, before, o);
        all += __shfl_xor_sync(0xffffffffu, all, o);
    }
    *total = all;
    return inc - x + before;
}

// exclusive block sum-scan (over threads 0..tid-1); *total = the block's sum
__device__ __forceinline__ int block_scan_sum_excl(int x, int* sh, int* total) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    int inc = x;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int y = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane >= o) inc += y;
    }
    if (lane == 31) sh[w] = inc;
    __syncthreads();
    if (w == 0) {
        int t = lane < (int)(blockDim.x >> 5) ? sh[lane] : 0;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int y = __shfl_up_sync(0xffffffffu, t, o);
            if (lane >= o) t += y;
        }
        sh[lane] = t;
    }
    __syncthreads();
    const int res = inc - x + (w > 0 ? sh[w - 1] : 0);
    *total = sh[31];
    __syncthreads();
    return res;
}

// V independent exclusive block scans at once (sh: 32 * V ints)
template <int V>
__device__ __forceinline__ void block_scan_sum_excl_v(const int (&x)[V], int* sh, int (&ex)[V], int (&total)[V]) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int nw = (int)(blockDim.x >> 5);
    int inc[V];
#pragma unroll
    for (int v = 0; v < V; v++) inc[v] = x[v];
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
#pragma unroll
        for (int v = 0; v < V; v++) {
            const int y = __shfl_up_sync(0xffffffffu, inc[v], o);
            if (lane >= o) inc[v] += y;
        }
    }
    if (lane == 31) {
#pragma unroll
        for (int v = 0; v < V; v++) sh[v * 32 + w] = inc[v];
    }
    __syncthreads();
#pragma unroll
    for (int v = 0; v < V; v++) {
        const int ws = lane < nw ? sh[v * 32 + lane] : 0;
        int before = lane < w ? ws : 0, all = ws;
#pragma unroll
        for (int o = 16; o; o >>= 1) {
            before += __shfl_xor_sync(0xffffffffu, before, o);
            all += __shfl_xor_sync(0xffffffffu, all, o);
        }
        ex[v] = inc[v] - x[v] + before;
        total[v] = all;
    }
}

__device__ __forceinline__ int block_scan_min_rev(int x, int* sh) {
    // suffix minimum: scan from the last thread backwards
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int y = __shfl_down_sync(0xffffffffu, x, o);
        if (lane + o < 32) x = min(x, y);
    }
    if (lane == 0) sh[w] = x;
    __syncthreads();
    if (w == 0) {
        int t = lane < LT / 32 ? sh[lane] : INT_MAX;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int y = __shfl_down_sync(0xffffffffu, t, o);
            if (lane + o < 32) t = min(t, y);
        }
        if (lane < LT / 32) sh[lane] = t;
    }
    __syncthreads();
    const int suf = w + 1 < LT / 32 ? sh[w + 1] : INT_MAX;
    __syncthreads();
    return min(x, suf);
}

// Bidirectional scan over the splitter nodes 0..C-1 of a tile (node arrays in s.P and
// s.R / s.K0,K1).  WARP: warp 0 alone, NPN nodes per lane, warp barriers; else the whole
// block, NPN = VPT nodes per thread, block barriers.
constexpr int kWarpScanNodes = 4;  // one warp scans up to 128 nodes

template <bool MINK, int NPN, bool WARP>
__device__ __forceinline__ void node_scan(TileSmem& s, int C, int* stats) {
    const int tid = threadIdx.x;
    constexpr int STRIDE = WARP ? 32 : LT;
    for (int step = 0; step < 16; step++) {
        int notdone = 0;
        short2 nP[NPN], nR[NPN];
        uint64_t nk0[NPN], nk1[NPN];
#pragma unroll
        for (int k = 0; k < NPN; k++) {
            const int i = tid + k * STRIDE;
            if (i >= C) continue;
            const short2 p = s.P[i];
            short2 q = p, r = s.R[i];
            uint64_t k0 = 0, k1 = 0;
            if (MINK) { k0 = s.K0[i]; k1 = s.K1[i]; }
#pragma unroll
            for (int dd = 0; dd < 2; dd++) {
                const int w = dd ? p.y : p.x;
                if (w < 0) continue;
                const short2 pw = s.P[w];
                int j = -1;
                if (pw.x != i) j = 0;
                else if (pw.y != i) j = 1;
                if (j < 0) continue;  // stall (reading c13)
                const short tgt = j ? pw.y : pw.x;
                if (dd) q.y = tgt; else q.x = tgt;
                if (MINK) {
                    const uint64_t kv = j ? s.K1[w] : s.K0[w];
                    if (dd) k1 = umin64(k1, kv); else k0 = umin64(k0, kv);
                } else {
                    const short2 rw = s.R[w];
                    const short dv = j ? rw.y : rw.x;
                    if (dd) r.y = (short)(r.y + dv); else r.x = (short)(r.x + dv);
                }
            }
            nP[k] = q;
            nR[k] = r;
            nk0[k] = k0;
            nk1[k] = k1;
            const bool path_done = q.x < 0 && q.y < 0;
            bool cyc_done = false;
            if (MINK) cyc_done = q.x >= 0 && q.y >= 0 && (k0 == k1 || q.x == q.y);
            notdone |= !(path_done || cyc_done);
        }
        if (WARP) __syncwarp(); else __syncthreads();
#pragma unroll
        for (int k = 0; k < NPN; k++) {
            const int i = tid + k * STRIDE;
            if (i >= C) continue;
            s.P[i] = nP[k];
            if (MINK) { s.K0[i] = nk0[k]; s.K1[i] = nk1[k]; } else s.R[i] = nR[k];
        }
        const bool any = WARP ? (__syncwarp(), __any_sync(0xffffffffu, notdone)) : __syncthreads_or(notdone);
        if (!any) {
            if (tid == 0 && stats) atomicMax(&stats[4], step + 1);
            break;
        }
    }
}

// Block-local ranking.  Same outputs as tile_scan, O(1) work per vertex:
//  0. runs: maximal intervals of consecutive vertex ids linked in the factor (an x-line of
//     a natural-order grid) are found with block-wide scans and contracted -- each end's
//     slot into the run becomes a virtual link to the other end (weight = run length - 1,
//     key = the run's weakest edge key); a run closed by a direct link between its ends is
//     a cycle by itself.  Interior vertices drop out until step 5.
//  1. splitters: terminals plus hashed vertices (density 1/8) among the remaining ones;
//  2. each splitter walks sequentially through shared memory to the next splitter in both
//     directions, recording (node, distance) in every vertex it passes;
//  3. the bidirectional scan runs on the splitter nodes only;
//  4. every remaining vertex combines its record with its node's result (cycles without a
//     splitter fall back to tile_scan; cycle pass only -- a forest has none);
//  5. interior run vertices take their run ends' results plus their offset in the run.
template <bool MINK>
__device__ void tile_rank(TileSmem& s, int32_t b0, const ulonglong2 (&ek)[VPT], int2 (&P)[VPT],
                          int2 (&R)[VPT], ulonglong2 (&K)[VPT], int* stats) {
    __shared__ int sh[32];
    const int tid = threadIdx.x;
    LF_PHASE_INIT;
    const Tile T = tile_of(s);
    const int tlen = T.tend - T.b0;
    if (tid == 0) s.nspl = 0;
    // 0a. (cycle pass) slot keys and the temporary K0 = key of the run link (u-1,u); the
    //     barriers of the scan below order these writes before their readers
    const auto linked_prev = [&](int u) {  // u-1 and u linked in the factor (same tile)
        const int2 nb = s.nb[u];
        const int32_t g = b0 + u;
        return u > 0 && u < tlen && (nb.x == g - 1 || nb.y == g - 1);
    };
    if (MINK) {
#pragma unroll
        for (int k = 0; k < VPT; k++) {
            const int u = tid + k * LT;
            const int2 nb = s.nb[u];
            const int32_t g = b0 + u;
            const bool lp = u > 0 && u < tlen && (nb.x == g - 1 || nb.y == g - 1);
            s.EK0[u] = ek[k].x;
            s.EK1[u] = ek[k].y;
            s.K0[u] = lp ? (nb.x == g - 1 ? ek[k].x : ek[k].y) : KEY_INF;
        }
    }
    // 0b. run bounds (contiguous ownership: thread t owns VPT*t..VPT*t+VPT-1): the run
    //     start by an exclusive block max-scan; the run end by a scatter from the next
    //     run's start (a run ends one before the next run starts)
    {
        const int u0 = tid * VPT;
        int st[VPT];
        bool lk[VPT + 1];  // lk[j]: u0+j linked to u0+j-1
#pragma unroll
        for (int j = 0; j <= VPT; j++) lk[j] = u0 + j < LB && linked_prev(u0 + j);
        int run = INT_MIN;
#pragma unroll
        for (int j = 0; j < VPT; j++) {
            if (!lk[j]) run = u0 + j;  // u0+j starts a run
            st[j] = run;
        }
        const int prev_max = block_scan_max_excl(run, sh);
#pragma unroll
        for (int j = 0; j < VPT; j++) {
            const int u = u0 + j;
            if (st[j] == INT_MIN) st[j] = prev_max;
            s.r.run[u].x = (short)st[j];
            if (!lk[j + 1]) s.r.run[st[j]].y = (short)u;  // run end: the run start learns it
        }
        __syncthreads();
        short en[VPT];
#pragma unroll
        for (int j = 0; j < VPT; j++) en[j] = s.r.run[st[j]].y;
        __syncthreads();
#pragma unroll
        for (int j = 0; j < VPT; j++) s.r.run[u0 + j].y = en[j];
        if (MINK) {
            // weakest link of each run: segmented inclusive min-scan of the link keys
            // (segments = runs); the value at the run's last vertex is the run's minimum
            uint64_t x[VPT];
            bool hd[VPT];
            uint64_t agg = KEY_INF;
            bool anyh = false;
#pragma unroll
            for (int j = 0; j < VPT; j++) {
                hd[j] = !lk[j];
                const uint64_t kv = s.K0[u0 + j];
                agg = hd[j] ? kv : umin64(agg, kv);
                anyh |= hd[j];
                x[j] = agg;
            }
            // warp scan of (head, min) pairs: (f1,x1)+(f2,x2) = (f1|f2, f2 ? x2 : min(x1,x2))
            const int lane = tid & 31, wid = tid >> 5;
            bool f = anyh;
            uint64_t v = agg;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const uint64_t yv = __shfl_up_sync(0xffffffffu, v, o);
                const int yf = __shfl_up_sync(0xffffffffu, (int)f, o);
                if (lane >= o) { if (!f) v = umin64(v, yv); f = f || yf; }
            }
            __shared__ uint64_t wv[LT / 32];
            __shared__ int wf[LT / 32];
            if (lane == 31) { wv[wid] = v; wf[wid] = f; }
            __syncthreads();
            if (wid == 0) {
                uint64_t tv = lane < LT / 32 ? wv[lane] : KEY_INF;
                bool tf = lane < LT / 32 ? wf[lane] != 0 : false;
#pragma unroll
                for (int o = 1; o < 32; o <<= 1) {
                    const uint64_t yv = __shfl_up_sync(0xffffffffu, tv, o);
                    const int yf = __shfl_up_sync(0xffffffffu, (int)tf, o);
                    if (lane >= o) { if (!tf) tv = umin64(tv, yv); tf = tf || yf; }
                }
                if (lane < LT / 32) { wv[lane] = tv; wf[lane] = tf; }
            }
            __syncthreads();
            // carry into this thread: inclusive value of the previous thread
            uint64_t cv = __shfl_up_sync(0xffffffffu, v, 1);
            bool cf = __shfl_up_sync(0xffffffffu, (int)f, 1) != 0;
            if (lane == 0) { cv = KEY_INF; cf = true; }
            if (wid > 0 && !cf) cv = umin64(cv, wv[wid - 1]);
            if (wid > 0 && lane == 0) { cv = wv[wid - 1]; cf = false; }
            // apply the carry to the thread's prefix up to its first head
#pragma unroll
            for (int j = 0; j < VPT; j++) {
                if (hd[j]) break;
                x[j] = umin64(x[j], cv);
            }
#pragma unroll
            for (int j = 0; j < VPT; j++) s.K1[u0 + j] = x[j];
        }
    }
    __syncthreads();
    // 0c. contract: virtual links between run ends; run cycles; interior flags (sidx = -2)
#pragma unroll
    for (int k = 0; k < VPT; k++) {
        const int u = tid + k * LT;
        const short2 rr = s.r.run[u];
        const int32_t g = b0 + u;
        short2 vw = make_short2(1, 1);
        const int len = rr.y - rr.x + 1;
        if (len >= 2 && (u == rr.x || u == rr.y)) {
            const int other = (u == rr.x) ? rr.y : rr.x;
            const int32_t inside = (u == rr.x) ? g + 1 : g - 1;
            int2 nb = s.nb[u];
            const uint64_t rk = MINK ? s.K1[rr.y] : 0;  // run minimum at its last vertex
            if (nb.x == inside) { nb.x = b0 + other; vw.x = (short)(len - 1); if (MINK) s.EK0[u] = rk; }
            else { nb.y = b0 + other; vw.y = (short)(len - 1); if (MINK) s.EK1[u] = rk; }
            s.nb[u] = nb;
        }
        s.r.vw[u] = vw;
    }
    __syncthreads();
    // 1. splitters among run ends and single vertices; a run closed into a cycle by a
    //    direct link between its ends is resolved here (sidx = -3)
#pragma unroll
    for (int k = 0; k < VPT; k++) {
        const int u = tid + k * LT;
        const short2 rr = s.r.run[u];
        const int2 nb = s.nb[u];
        const bool interior = u > rr.x && u < rr.y;
        const bool run_cycle = rr.y - rr.x >= 2 && nb.x == nb.y;  // both slots reach the other end
        short id = -1;
        bool node = false;
        if (u >= tlen) {
            node = true;  // padding: isolated terminal
        } else if (interior || run_cycle) {
            id = run_cycle ? -3 : -2;
        } else {
            const bool l0 = nb.x >= 0 && is_local(nb.x, T);
            const bool l1 = nb.y >= 0 && is_local(nb.y, T);
            // run ends are always splitters: every cycle through a run has one
            const bool run_end = rr.y > rr.x;
            node = !l0 || !l1 || run_end || hashed_splitter(b0 + u);
        }
        {  // warp-aggregated node numbering
            const unsigned m = __ballot_sync(0xffffffffu, node);
            const int lane = tid & 31;
            int base = 0;
            if (lane == 0 && m) base = atomicAdd(&s.nspl, __popc(m));
            base = __shfl_sync(0xffffffffu, base, 0);
            if (node) id = (short)(base + __popc(m & ((1u << lane) - 1u)));
        }
        s.sidx[u] = id;
        if (id >= 0) s.spl[id] = (short)u;
        s.recS[u] = make_short2(-1, -1);
    }
    __syncthreads();
    if (MINK) LF_PHASE(stats - kCtlStat, 3);
    const int C = s.nspl;
    if (tid == 0 && stats) atomicAdd(&stats[MINK ? 0 : 3], C);
    // 2. walks: one per (node, slot), sequential through non-splitters (weighted links)
    for (int wk = tid; wk < 2 * C; wk += LT) {
        const int i = wk >> 1, f = wk & 1;
        const int su = s.spl[i];
        const int2 nbs = s.nb[su];
        const int32_t x = f ? nbs.y : nbs.x;
        short ptr = (short)(-(i + 1));
        int dist = 0;
        uint64_t km = KEY_INF;
        if (x >= 0 && is_local(x, T)) {
            const short2 vws = s.r.vw[su];
            int prev = su, cur = x - b0, d = f ? vws.y : vws.x;
            if (MINK) km = f ? s.EK1[su] : s.EK0[su];
            while (s.sidx[cur] < 0) {
                const int2 nbc = s.nb[cur];
                const int face = (nbc.x == b0 + prev) ? 0 : 1;
                if (face == 0) { s.recS[cur].x = (short)((i << 1) | f); s.recD[cur].x = (short)d; }
                else { s.recS[cur].y = (short)((i << 1) | f); s.recD[cur].y = (short)d; }
                const int nxt = (face ? nbc.x : nbc.y) - b0;  // local (else cur were a splitter)
                const short2 vwc = s.r.vw[cur];
                d += face ? vwc.x : vwc.y;
                if (MINK) km = umin64(km, face ? s.EK0[cur] : s.EK1[cur]);
                prev = cur;
                cur = nxt;
            }
            ptr = s.sidx[cur];
            dist = d;
        }
        if (f) { s.P[i].y = ptr; s.R[i].y = (short)dist; s.K1[i] = km; }
        else { s.P[i].x = ptr; s.R[i].x = (short)dist; s.K0[i] = km; }
    }
    __syncthreads();
    if (MINK) LF_PHASE(stats - kCtlStat, 4);
    // 3. bidirectional scan over the splitter nodes (node arrays in s.P/s.R/s.K*): by one
    //    warp with warp barriers when the nodes are few, else by the whole block
    if (C <= 32 * kWarpScanNodes) {
        if (tid < 32) node_scan<MINK, kWarpScanNodes, true>(s, C, stats);
        __syncthreads();
    } else {
        node_scan<MINK, VPT, false>(s, C, stats);
    }
    if (MINK) LF_PHASE(stats - kCtlStat, 5);
    // 4. expand run ends and single vertices from their node or walk records
    bool unvisited[VPT];
    int any_unvisited = 0;
#pragma unroll
    for (int k = 0; k < VPT; k++) {
        const int u = tid + k * LT;
        unvisited[k] = false;
        const int id = s.sidx[u];
        P[k] = make_int2(0, 0);
        R[k] = make_int2(0, 0);
        if (id == -2 || id == -3) continue;  // interior run vertex / run cycle: step 5
        if (id >= 0) {
            const short2 p = s.P[id];
            P[k].x = p.x;
            P[k].y = p.y;
            if (p.x < 0) P[k].x = -(s.spl[-(p.x + 1)] + 1);
            if (p.y < 0) P[k].y = -(s.spl[-(p.y + 1)] + 1);
            if (MINK) { K[k].x = s.K0[id]; K[k].y = s.K1[id]; }
            else { const short2 r = s.R[id]; R[k] = make_int2(r.x, r.y); }
            continue;
        }
        const short2 rs = s.recS[u];
        if (rs.x < 0 && rs.y < 0) { unvisited[k] = true; any_unvisited = 1; continue; }
        const short2 rd = s.recD[u];
#pragma unroll
        for (int f = 0; f < 2; f++) {
            const int rec = f ? rs.y : rs.x;
            const int i = rec >> 1, f0 = rec & 1;
            const short2 p = s.P[i];
            const int away = f0 ^ 1;  // node i's direction that leads away from u
            const int pa = away ? p.y : p.x;
            if (pa >= 0) {  // node on a cycle: the cycle's weakest key is min(K0,K1)
                if (f) P[k].y = 0; else P[k].x = 0;
                if (MINK) { K[k].x = s.K0[i]; K[k].y = s.K1[i]; }
                continue;
            }
            const int t = s.spl[-(pa + 1)];
            const int dd = (f ? rd.y : rd.x) + (MINK ? 0 : (away ? s.R[i].y : s.R[i].x));
            if (f) { P[k].y = -(t + 1); R[k].y = dd; } else { P[k].x = -(t + 1); R[k].x = dd; }
        }
        // a vertex on a cycle: make both pointers non-negative (cycle flag)
        if (P[k].x >= 0 || P[k].y >= 0) { P[k].x = 0; P[k].y = 0; }
    }
    if (MINK) LF_PHASE(stats - kCtlStat, 6);
    if (MINK) {
        if (stats) {
            int nu = 0;
#pragma unroll
            for (int k = 0; k < VPT; k++) nu += unvisited[k];
            if (nu) atomicAdd(&stats[1], nu);
        }
        if (__syncthreads_or(any_unvisited)) {
            if (tid == 0 && stats) atomicAdd(&stats[2], 1);
            // splitter-free cycles of the contracted graph: pointer jumping on them alone,
            // with the virtual link keys
            bool skip[VPT];
            ulonglong2 ekv[VPT];
#pragma unroll
            for (int k = 0; k < VPT; k++) {
                const int u = tid + k * LT;
                skip[k] = !unvisited[k];
                ekv[k] = make_ulonglong2(s.EK0[u], s.EK1[u]);
            }
            int2 P2[VPT], R2[VPT];
            ulonglong2 K2[VPT];
            tile_scan<true>(s, b0, ekv, P2, R2, K2, skip);
#pragma unroll
            for (int k = 0; k < VPT; k++)
                if (unvisited[k]) { P[k] = P2[k]; K[k] = K2[k]; }
        }
    }
    // 5. interior run vertices and run cycles from the run ends.  Publish the ends'
    //    results: recS = terminal markers (or (0,0) cycle), recD = distances, EK = keys.
    __syncthreads();
#pragma unroll
    for (int k = 0; k < VPT; k++) {
        const int u = tid + k * LT;
        const short2 rr = s.r.run[u];
        if (rr.y > rr.x && (u == rr.x || u == rr.y) && s.sidx[u] != -3) {
            s.recS[u] = make_short2((short)P[k].x, (short)P[k].y);
            s.recD[u] = make_short2((short)R[k].x, (short)R[k].y);
            if (MINK) { s.EK0[u] = K[k].x; s.EK1[u] = K[k].y; }
        }
    }
    __syncthreads();
#pragma unroll
    for (int k = 0; k < VPT; k++) {
        const int u = tid + k * LT;
        const int id = s.sidx[u];
        if (id != -2 && id != -3) continue;
        const short2 rr = s.r.run[u];
        if (s.sidx[rr.x] == -3) {  // the run closes into a cycle through its ends' direct link
            // weakest of the run links (virtual key) and the closing link (real key)
            P[k] = make_int2(0, 0);
            if (MINK) {
                const uint64_t km = umin64(s.EK0[rr.x], s.EK1[rr.x]);
                K[k] = make_ulonglong2(km, km);
            }
            continue;
        }
        const int32_t g = b0 + u;
        const int2 nb = s.nb[u];
        // interior: slot toward u-1 leads to the run start, the other to the run end
        const short2 pa = s.recS[rr.x], pb = s.recS[rr.y];
        const int2 nba = s.nb[rr.x], nbb = s.nb[rr.y];
        const int oa = (nba.x == b0 + rr.y) ? 1 : 0;  // the start's outer slot
        const int ob = (nbb.x == b0 + rr.x) ? 1 : 0;  // the end's outer slot
        const int ta = oa ? pa.y : pa.x, tb = ob ? pb.y : pb.x;
        const bool cyc = (pa.x >= 0 && pa.y >= 0);
        const short2 da = s.recD[rr.x], db = s.recD[rr.y];
        const int dA = (oa ? da.y : da.x) + (u - rr.x), dB = (ob ? db.y : db.x) + (rr.y - u);
        const int sa = (nb.x == g - 1) ? 0 : 1;  // u's slot toward the run start
        if (cyc) {
            P[k] = make_int2(0, 0);
            if (MINK) K[k] = make_ulonglong2(s.EK0[rr.x], s.EK1[rr.x]);
        } else if (sa == 0) {
            P[k] = make_int2(ta, tb);
            R[k] = make_int2(dA, dB);
        } else {
            P[k] = make_int2(tb, ta);
            R[k] = make_int2(dB, dA);
        }
    }
    __syncthreads();
    if (MINK) LF_PHASE(stats - kCtlStat, 7);
}

// the slot of local terminal t (t not the walk's start) that leaves its segment: the
// one that is not a local link (a remote neighbour or none)
__device__ __forceinline__ int outward_slot(int2 nbt, const Tile& T) {
    const bool l0 = nbt.x >= 0 && is_local(nbt.x, T);
    return l0 ? 1 : 0;
}

// warp-aggregated slot claim in two halves, so that nothing waits for the atomic's return
// until the slot is used: claim_issue (ballot + one atomic per warp, result in lane 0) and
// claim_pos (broadcast + rank; -1 if not taken)
struct Claim {
    unsigned m;
    int base;  // lane 0: the warp's first slot
};
__device__ __forceinline__ Claim claim_issue(int* count, bool take) {
    Claim c;
    c.m = __ballot_sync(0xffffffffu, take);
    c.base = 0;
    if ((threadIdx.x & 31) == 0 && c.m) c.base = atomicAdd(count, __popc(c.m));
    return c;
}
__device__ __forceinline__ int claim_pos(const Claim& c) {
    const int lane = threadIdx.x & 31;
    const int base = __shfl_sync(0xffffffffu, c.base, 0);
    return ((c.m >> lane) & 1u) ? base + __popc(c.m & ((1u << lane) - 1u)) : -1;
}

// warp-aggregated append; returns the list position of g (-1 if not taken)
__device__ __forceinline__ int list_append(int32_t* list, int* count, int32_t g, bool take) {
    const unsigned m = __ballot_sync(0xffffffffu, take);
    const int lane = threadIdx.x & 31;
    int base = 0;
    if (lane == 0 && m) base = atomicAdd(count, __popc(m));
    base = __shfl_sync(0xffffffffu, base, 0);
    const int idx = base + __popc(m & ((1u << lane) - 1u));
    if (take) list[idx] = g;
    return take ? idx : -1;
}

struct ForestArgs {
    int64_t N;             // global vertex count (markers: end -(e+1), exit -(N+1+e))
    int64_t lo, hi;        // own vertex range (a whole graph: 0, N); arrays are offset so
                           // that vertex g is element g
    // foreign neighbours' slots (partitioned runs): sorted ghost ids and their slots
    const int32_t* ghost_list;
    int64_t n_ghost, ghost_below;
    const int2* ghost_nb;  // [local id] slots (global ids) of ghost vertices
    // results of the reduced scans are stored at list positions (compact, coalesced);
    // bidx1 / bidx2 map a boundary vertex to its position in list1 / list2
    int32_t* bidx1;        // [v] list1 position of a boundary vertex of the cycle pass
    int32_t* bidx2;        // [v] list2 position of a boundary vertex of the rank pass
    ulonglong2* kraw;      // [list1 pos] final per-direction min keys of the cycle pass
    ulonglong2* ekb;       // [list1 pos] slot keys of boundary vertices
    const int2* __restrict__ pi2;
    const float2* __restrict__ pi2_w;
    int2* forest;
    // per-vertex local results (written by the local pass, read by the expand pass)
    short2* loc1;          // [N] local terminal markers of the cycle pass (>= 0: local cycle)
    uint64_t* kst;         // [N] weakest key of a local cycle (written on local cycles only)
    int2* loc2;            // [N] (terminal markers as shorts packed, local distances)
    // reduced graph, pass 1 (cycles)
    int2* rq1[2];
    ulonglong2* rk1[2];
    uint64_t* cyc_k;       // [list1 pos] weakest key of the global cycle through it
    int32_t* list1;
    // reduced graph, pass 2 (positions)
    int2* rq2[2];
    int2* rr2[2];
    int2* end2;            // [list2 pos] path ends per direction of a boundary vertex
    int2* dist2;           // [list2 pos] distances to them
    int32_t* list2;
    // compact records of the list being built / scanned (list position -> record)
    int2* cq;              // stride pointers (vertex ids or markers)
    ulonglong2* cq_k;      // MIN: min keys; ADD: distances in the low words
    int* ctl;
    int32_t* path_id;
    int32_t* pos;
    int32_t* len;
    uint8_t* pdir;         // [N] forest slot toward the path-ID end
    unsigned long long* n_cycles;
    int max_steps;
    // single-pass forest (FULL windows): reduced records and results at list positions
    int2* cq_r;            // [list pos] initial window lengths per direction
    int2* cq_dk;           // [list pos] initial DK per direction
    int2* dk2;             // [list pos] final DK per direction
    int2* rdk[2];          // grid-path ping-pong DK
    int32_t* off;          // [N] exclusive tile prefix of path lengths (at path-ID vertices)
    int32_t* tsum;         // [tiles] tile totals -> exclusive prefix (last expand CTA)
    // global ruling set (k_grs_*): packed records, visit bitmap, splitter-free cycles, and
    // the permutation / tridiagonal outputs its last walk writes directly
    int4* grs_rec;
    uint32_t* grs_bits;
    int4* grs_cyc;
    uint64_t* grs_cyck;
    int32_t* perm;
    int32_t* iperm;
    float *ta, *tb, *tc;
    const float2* pi2_val;
    const float* diag;
    int grs_shift;         // hashed splitter density 2^-(32 - grs_shift)
    int4* grs_meet;        // [2N] per (vertex, slot): the partial window of the walk that stopped
    uint64_t* grs_meetk;   //   there looking along that slot: (item, R, DK, 0) and K
    int4* grs_mstop;       // [2 cnt] (last, next | slot << 31, stop key) of a walk that met its partner; x = -1: final
    int4* grs_rout;        // [N] (perm, a, b, c) at the new index (the meet records' storage, free by then)
    int4* grs_desc;        // [2 (cnt + cycles)] walk descriptors (k_grs_desc); cnt + cycles <= N
};

__device__ __forceinline__ bool is_foreign(int64_t x, const ForestArgs& a) { return x < a.lo || x >= a.hi; }

// slots of a vertex of another rank (binary search in the sorted ghost list)
__device__ __forceinline__ int2 ghost_slots(const ForestArgs& a, int32_t x) {
    int64_t l = 0, h = a.n_ghost;
    while (l < h) {
        const int64_t m = (l + h) >> 1;
        if (a.ghost_list[m] < x) l = m + 1; else h = m;
    }
    const int64_t lid = l < a.ghost_below ? l : l + (a.hi - a.lo);
    return a.ghost_nb[lid];
}

// keys of the own vertices' slots (global; a remote min endpoint needs one gather)
template <class S, int TT = LT>
__device__ __forceinline__ void slot_keys(const ForestArgs& a, S& s, int32_t b0,
                                         ulonglong2 (&ek)[LB / TT]) {
    constexpr int VV = LB / TT;
    const Tile T = tile_of(s);
#pragma unroll
    for (int k = 0; k < VV; k++) {
        const int u = threadIdx.x + k * TT;
        const int32_t g = b0 + u;
        const int2 nb = s.nb[u];
        ek[k].x = KEY_INF;
        ek[k].y = KEY_INF;
        if (g >= a.hi) continue;
        const float2 w = s.w[u];
        if (nb.x >= 0) {
            const int32_t mn = g < nb.x ? g : nb.x;
            const int2 nbm = is_local(mn, T) ? s.nb[mn - b0] : (is_foreign(mn, a) ? ghost_slots(a, mn) : a.pi2[mn]);
            ek[k].x = edge_key(g, nb.x, w.x, nbm);
        }
        if (nb.y >= 0) {
            const int32_t mn = g < nb.y ? g : nb.y;
            const int2 nbm = is_local(mn, T) ? s.nb[mn - b0] : (is_foreign(mn, a) ? ghost_slots(a, mn) : a.pi2[mn]);
            ek[k].y = edge_key(g, nb.y, w.y, nbm);
        }
    }
}

// slots and weights of the tile in one round trip (cycle pass)
template <class S, int TT = LT>
__device__ __forceinline__ void load_tile_w(const int2* __restrict__ src, const float2* __restrict__ wsrc,
                                            S& s, int32_t b0, int64_t hi) {
    constexpr int VV = LB / TT;
    if (threadIdx.x == 0) {
        s.b0 = b0;
        s.tend = (int32_t)((int64_t)b0 + LB < hi ? (int64_t)b0 + LB : hi);
    }
#pragma unroll
    for (int k = 0; k < VV; k++) {
        const int u = threadIdx.x + k * TT;
        const int64_t g = (int64_t)b0 + u;
        const bool in = g < hi;
        const int2 nb = in ? src[g] : make_int2(-1, -1);
        const float2 w = in ? wsrc[g] : make_float2(0.f, 0.f);
        s.nb[u] = nb;
        s.w[u] = w;
    }
    __syncthreads();
}

template <class S>
__device__ __forceinline__ void load_tile(const int2* __restrict__ src, S& s, int32_t b0, int64_t hi) {
    if (threadIdx.x == 0) {
        s.b0 = b0;
        s.tend = (int32_t)((int64_t)b0 + LB < hi ? (int64_t)b0 + LB : hi);
    }
#pragma unroll
    for (int k = 0; k < VPT; k++) {
        const int u = threadIdx.x + k * LT;
        const int64_t g = (int64_t)b0 + u;
        s.nb[u] = g < hi ? src[g] : make_int2(-1, -1);
    }
    __syncthreads();
}

// reduced-graph direction of boundary vertex g through its slot i:
//   none -> end marker -(g+1) (distance 0); another rank -> exit marker -(N+1+g)
//   (distance 0; the exit list continues it); another tile -> the neighbour (distance 1);
//   local -> the segment's other terminal t: t if t continues (another tile or rank),
//   else an end marker at t (distance = local length).
__device__ __forceinline__ void reduced_dir(const ForestArgs& a, const TileSmem& s, int32_t b0, int32_t g,
                                            int2 nb, int i, int2 p, int2 r, int32_t& q, int32_t& d) {
    const Tile T = tile_of(s);
    const int32_t x = i ? nb.y : nb.x;
    if (x < 0) { q = -(g + 1); d = 0; return; }
    if (is_foreign(x, a)) { q = (int32_t)(-(a.N + 1 + g)); d = 0; return; }
    if (!is_local(x, T)) { q = x; d = 1; return; }
    const int t = -((i ? p.y : p.x) + 1);
    const int2 nbt = s.nb[t];
    const int so = outward_slot(nbt, T);
    const int32_t xo = so ? nbt.y : nbt.x;
    const int32_t tg = b0 + t;
    // t continues (in another tile or on another rank): t is itself a boundary vertex,
    // so point at it -- its own cross-rank slot carries the exit marker
    q = xo < 0 ? -(tg + 1) : tg;
    d = i ? r.y : r.x;
}

// Pass 1, local part: local min-scan; store the local results; emit the reduced-graph
// records of boundary vertices.
__global__ void __launch_bounds__(LT, 1) k_lf_local1(ForestArgs a) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    TileSmem& s = *reinterpret_cast<TileSmem*>(smem_raw);
    const int32_t b0 = (int32_t)(a.lo + (int64_t)blockIdx.x * LB);
    LF_PHASE_INIT;
    if (a.n_cycles && blockIdx.x == 0 && threadIdx.x == 0) *a.n_cycles = 0;  // summed by local2
    load_tile_w(a.pi2, a.pi2_w, s, b0, a.hi);
    const Tile T{b0, (int32_t)((int64_t)b0 + LB < a.hi ? (int64_t)b0 + LB : a.hi)};
    LF_PHASE(a.ctl, 0);
    ulonglong2 ek[VPT];
    slot_keys(a, s, b0, ek);
    LF_PHASE(a.ctl, 1);
    int2 P[VPT], R[VPT];
    ulonglong2 K[VPT];
    tile_rank<true>(s, b0, ek, P, R, K, a.ctl + kCtlStat);
#pragma unroll
    for (int k = 0; k < VPT; k++) {
        const int u = threadIdx.x + k * LT;
        const int32_t g = b0 + u;
        const int2 nb = s.nb[u];
        const bool r0 = nb.x >= 0 && !is_local(nb.x, T);
        const bool r1 = nb.y >= 0 && !is_local(nb.y, T);
        const bool boundary = g < a.hi && (r0 || r1);
        if (g < a.hi) {
            a.loc1[g] = make_short2((short)P[k].x, (short)P[k].y);
            if (P[k].x >= 0 && P[k].y >= 0) a.kst[g] = umin64(K[k].x, K[k].y);
        }
        const int idx = list_append(a.list1, &a.ctl[kCtlCnt1], g, boundary);
        if (boundary) {
            int32_t q0, q1, d0, d1;
            reduced_dir(a, s, b0, g, nb, 0, P[k], R[k], q0, d0);
            reduced_dir(a, s, b0, g, nb, 1, P[k], R[k], q1, d1);
            // key of each reduced link: the remote edge's key, or the segment's min key
            ulonglong2 rk;
            rk.x = (nb.x < 0 || is_foreign(nb.x, a)) ? KEY_INF : (r0 ? ek[k].x : K[k].x);
            rk.y = (nb.y < 0 || is_foreign(nb.y, a)) ? KEY_INF : (r1 ? ek[k].y : K[k].y);
            if (a.ekb) a.ekb[idx] = ek[k];
            a.bidx1[g] = idx;
            a.cq[idx] = make_int2(q0, q1);
            a.cq_k[idx] = rk;
        }
    }
    LF_PHASE(a.ctl, 2);  // outputs
}

// One step of the reduced bidirectional scan for the list entries t0, t0+stride, ...
// Nodes are processed in batches of RB so that each thread keeps several independent
// L2 gathers in flight.  Returns the number of entries not yet done.
constexpr int RB = 4;

template <bool MIN>
__device__ __forceinline__ int red_step(const ForestArgs& a, const int32_t* __restrict__ list, int cnt,
                                        int step, int t0, int stride) {
    const int2* __restrict__ qs = MIN ? a.rq1[step & 1] : a.rq2[step & 1];
    int2* __restrict__ qd = MIN ? a.rq1[(step & 1) ^ 1] : a.rq2[(step & 1) ^ 1];
    const ulonglong2* __restrict__ ks = a.rk1[step & 1];
    ulonglong2* __restrict__ kd = a.rk1[(step & 1) ^ 1];
    const int2* __restrict__ rs = a.rr2[step & 1];
    int2* __restrict__ rd = a.rr2[(step & 1) ^ 1];
    int notdone = 0;
    for (int base = t0; base < cnt; base += stride * RB) {
        int32_t v[RB];
        int2 q[RB];
#pragma unroll
        for (int b = 0; b < RB; b++) {
            const int idx = base + b * stride;
            v[b] = idx < cnt ? list[idx] : -1;
        }
#pragma unroll
        for (int b = 0; b < RB; b++) q[b] = v[b] >= 0 ? qs[v[b]] : make_int2(-1, -1);
        int2 qw[RB][2];
#pragma unroll
        for (int b = 0; b < RB; b++) {
            qw[b][0] = q[b].x >= 0 ? qs[q[b].x] : make_int2(0, 0);
            qw[b][1] = q[b].y >= 0 ? qs[q[b].y] : make_int2(0, 0);
        }
#pragma unroll
        for (int b = 0; b < RB; b++) {
            if (v[b] < 0) continue;
            if (q[b].x < 0 && q[b].y < 0) {  // final: keep both buffers equal
                const int2 qo = qd[v[b]];
                if (qo.x != q[b].x || qo.y != q[b].y) {
                    qd[v[b]] = q[b];
                    if (MIN) kd[v[b]] = ks[v[b]]; else rd[v[b]] = rs[v[b]];
                }
                continue;
            }
            int2 nq = q[b];
            ulonglong2 nk = make_ulonglong2(0, 0);
            int2 nr = make_int2(0, 0);
            if (MIN) nk = ks[v[b]]; else nr = rs[v[b]];
#pragma unroll
            for (int i = 0; i < 2; i++) {
                const int32_t w = i ? q[b].y : q[b].x;
                if (w < 0) continue;
                const int2 qww = qw[b][i];
                int j = -1;
                if (qww.x != v[b]) j = 0;
                else if (qww.y != v[b]) j = 1;
                if (j < 0) continue;  // stall (reading c13)
                const int32_t tgt = j ? qww.y : qww.x;
                if (i) nq.y = tgt; else nq.x = tgt;
                if (MIN) {
                    const ulonglong2 kw = ks[w];
                    const uint64_t kv = j ? kw.y : kw.x;
                    if (i) nk.y = umin64(nk.y, kv); else nk.x = umin64(nk.x, kv);
                } else {
                    const int2 rw = rs[w];
                    const int32_t dv = j ? rw.y : rw.x;
                    if (i) nr.y += dv; else nr.x += dv;
                }
            }
            qd[v[b]] = nq;
            if (MIN) kd[v[b]] = nk; else rd[v[b]] = nr;
            const bool path_done = nq.x < 0 && nq.y < 0;
            bool cyc_done = false;
            if (MIN) cyc_done = nq.x >= 0 && nq.y >= 0 && (nk.x == nk.y || nq.x == nq.y);
            notdone += (path_done || cyc_done) ? 0 : 1;
        }
    }
    return notdone;
}

template <bool MIN>
__device__ __forceinline__ void red_epilogue(const ForestArgs& a, const int32_t* list, int cnt, int fb,
                                             int t0, int stride) {
    for (int idx = t0; idx < cnt; idx += stride) {
        const int32_t v = list[idx];
        if (MIN) {
            const int2 q = a.rq1[fb][v];
            const ulonglong2 k = a.rk1[fb][v];
            a.cyc_k[idx] = (q.x >= 0 && q.y >= 0) ? umin64(k.x, k.y) : KEY_INF;
            a.end2[idx] = q;  // raw markers (exit list construction)
            if (a.kraw) a.kraw[idx] = k;
        } else {
            a.end2[idx] = a.rq2[fb][v];  // raw end markers -(e+1) (or exit markers)
            a.dist2[idx] = a.rr2[fb][v];
        }
    }
}

constexpr int RT = 1024;                    // reduced-scan block size
#ifndef LF_RED_SMALL
#define LF_RED_SMALL (4 * 1024)
#endif
constexpr int kRedSmall = LF_RED_SMALL;     // lists up to this size run in one CTA, in smem
constexpr int kRedHash = 2 * kRedSmall;     // open-addressing table vertex -> list position
static_assert((kRedHash & (kRedHash - 1)) == 0, "hash table size must be a power of two");

// smem image of a small reduced graph (pointers are list positions or end markers)
struct RedSmem {
    int2 q[kRedSmall];
    uint64_t k0[kRedSmall];   // MIN: min keys per direction; ADD: distances (low words)
    uint64_t k1[kRedSmall];
    int32_t v[kRedSmall];     // vertex id of each list position
    int2 ht[kRedHash];        // (vertex, list position), vertex -1 = empty
};

__device__ __forceinline__ uint32_t red_hash(int32_t v) {
    return ((uint32_t)v * 0x9E3779B1u) >> (32 - __builtin_ctz(kRedHash));
}

// list position of a listed vertex (every stride pointer of the reduced graph is one)
__device__ __forceinline__ int red_lookup(const RedSmem& S, int32_t v) {
    uint32_t h = red_hash(v);
    for (int n = 0; n < kRedHash; n++) {
        const int2 e = S.ht[h];
        if (e.x == v) return e.y;
        if (e.x < 0) break;
        h = (h + 1) & (kRedHash - 1);
    }
    return -(v + 1);  // unreachable for a well-formed list: an end marker at v
}

// The whole reduced scan inside one CTA: the list's compact records are loaded with
// coalesced reads, their vertex-id pointers are turned into list positions through a
// shared-memory hash table, the bidirectional scan runs in shared memory with block
// barriers, and the results are written per vertex.  Used when the boundary list is small.
#ifdef LF_PHASE_TIMING
__device__ __forceinline__ unsigned long long gtime() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}
#define RS_MARK(i) do { __syncthreads(); if (threadIdx.x == 0) atomicAdd((unsigned long long*)&a.ctl[224 + 2 * (i)], gtime() - t_start); } while (0)
#else
#define RS_MARK(i) do { } while (0)
#endif

template <int T, bool MIN>
__device__ void red_scan_small(const ForestArgs& a, const int32_t* list, int cnt, int* ctl, RedSmem& S) {
    constexpr int NPT = (kRedSmall + T - 1) / T;
    const int tid = threadIdx.x;
#ifdef LF_PHASE_TIMING
    const unsigned long long t_start = gtime();
#endif
    for (int i = tid; i < kRedHash; i += T) S.ht[i] = make_int2(-1, -1);
    __syncthreads();
    int32_t v[NPT];
    int2 q[NPT];
    ulonglong2 kk[NPT];
#pragma unroll
    for (int k = 0; k < NPT; k++) {
        const int idx = tid + k * T;
        v[k] = -1;
        if (idx >= cnt) continue;
        v[k] = list[idx];
        q[k] = a.cq[idx];
        kk[k] = a.cq_k[idx];
    }
#pragma unroll
    for (int k = 0; k < NPT; k++) {
        if (v[k] < 0) continue;
        const int idx = tid + k * T;
        S.v[idx] = v[k];
        uint32_t h = red_hash(v[k]);
        while (atomicCAS(&S.ht[h].x, -1, v[k]) != -1) h = (h + 1) & (kRedHash - 1);
        S.ht[h].y = idx;
    }
    __syncthreads();
    RS_MARK(0);
    bool fin[NPT];
#pragma unroll
    for (int k = 0; k < NPT; k++) {
        fin[k] = true;
        if (v[k] < 0) continue;
        if (q[k].x >= 0) q[k].x = red_lookup(S, q[k].x);
        if (q[k].y >= 0) q[k].y = red_lookup(S, q[k].y);
        fin[k] = q[k].x < 0 && q[k].y < 0;
        S.q[tid + k * T] = q[k];
        S.k0[tid + k * T] = kk[k].x;
        S.k1[tid + k * T] = kk[k].y;
    }
    RS_MARK(1);
    int step = 0;
    int notdone = 0;
#pragma unroll
    for (int k = 0; k < NPT; k++) notdone |= !fin[k];
    if (__syncthreads_or(notdone)) {
        for (; step < a.max_steps; step++) {
            int2 nq[NPT];
            ulonglong2 nk[NPT];
#pragma unroll
            for (int k = 0; k < NPT; k++) {
                if (fin[k]) continue;
                const int me = tid + k * T;
                nq[k] = q[k];
                nk[k] = kk[k];
#pragma unroll
                for (int i = 0; i < 2; i++) {
                    const int w = i ? q[k].y : q[k].x;
                    if (w < 0) continue;
                    const int2 qw = S.q[w];
                    int j = -1;
                    if (qw.x != me) j = 0;
                    else if (qw.y != me) j = 1;
                    if (j < 0) continue;  // stall (reading c13)
                    const int tgt = j ? qw.y : qw.x;
                    if (i) nq[k].y = tgt; else nq[k].x = tgt;
                    const uint64_t kv = j ? S.k1[w] : S.k0[w];
                    if (MIN) { if (i) nk[k].y = umin64(nk[k].y, kv); else nk[k].x = umin64(nk[k].x, kv); }
                    else { if (i) nk[k].y += kv; else nk[k].x += kv; }
                }
            }
            __syncthreads();
            notdone = 0;
#pragma unroll
            for (int k = 0; k < NPT; k++) {
                if (fin[k]) continue;
                const int me = tid + k * T;
                q[k] = nq[k];
                kk[k] = nk[k];
                S.q[me] = q[k];
                S.k0[me] = kk[k].x;
                S.k1[me] = kk[k].y;
                fin[k] = q[k].x < 0 && q[k].y < 0;
                bool cyc_done = false;
                if (MIN) cyc_done = q[k].x >= 0 && q[k].y >= 0 && (kk[k].x == kk[k].y || q[k].x == q[k].y);
                notdone |= !(fin[k] || cyc_done);
            }
            const int any = __syncthreads_or(notdone);
            if (tid == 0) ctl[step] = 1;  // diagnostics: steps taken
            if (!any) break;
        }
    }
    RS_MARK(2);
#pragma unroll
    for (int k = 0; k < NPT; k++) {
        if (v[k] < 0) continue;
        // pointers back to vertex ids (markers pass through unchanged)
        const int2 qg = make_int2(q[k].x >= 0 ? S.v[q[k].x] : q[k].x, q[k].y >= 0 ? S.v[q[k].y] : q[k].y);
        const int idx = tid + k * T;
        if (MIN) {
            a.cyc_k[idx] = (q[k].x >= 0 && q[k].y >= 0) ? umin64(kk[k].x, kk[k].y) : KEY_INF;
            a.end2[idx] = qg;
            if (a.kraw) a.kraw[idx] = kk[k];
        } else {
            a.end2[idx] = qg;
            a.dist2[idx] = make_int2((int)kk[k].x, (int)kk[k].y);
        }
    }
    RS_MARK(3);
}

// Reduced bidirectional scan over a boundary list (one cooperative kernel).
//   MIN: min-scan of edge keys; epilogue writes cyc_k (INF unless on a global cycle).
//   ADD: position scan with weighted hops; epilogue writes end2 / dist2.
// Small lists run in block 0 alone, in shared memory (a grid barrier costs more than the
// work); large ones use the whole grid with grid barriers on vertex-indexed ping-pong
// buffers initialised from the compact records.  Both leave as soon as every node is done.
template <bool MIN>
__global__ void __launch_bounds__(RT) k_red_scan(ForestArgs a) {
    __shared__ int sh[32];
    extern __shared__ __align__(16) unsigned char red_smem[];
    pdl_trigger();  // the next tile kernel may launch and wait meanwhile
    const int32_t* list = MIN ? a.list1 : a.list2;
    const int cnt = *(volatile int*)&a.ctl[MIN ? kCtlCnt1 : kCtlCnt2];
    int* ctl = a.ctl + (MIN ? kCtlRed1 : kCtlRed2);
    if (cnt <= kRedSmall) {
        if (blockIdx.x == 0) red_scan_small<RT, MIN>(a, list, cnt, ctl, *reinterpret_cast<RedSmem*>(red_smem));
        return;
    }
    cg::grid_group grid = cg::this_grid();
    const int stride = gridDim.x * blockDim.x;
    const int t0 = blockIdx.x * blockDim.x + threadIdx.x;
    for (int idx = t0; idx < cnt; idx += stride) {
        const int32_t v = list[idx];
        const int2 q = a.cq[idx];
        const ulonglong2 k = a.cq_k[idx];
        if (MIN) {
            a.rq1[0][v] = q; a.rq1[1][v] = q;
            a.rk1[0][v] = k; a.rk1[1][v] = k;
        } else {
            const int2 d = make_int2((int)k.x, (int)k.y);
            a.rq2[0][v] = q; a.rq2[1][v] = q;
            a.rr2[0][v] = d; a.rr2[1][v] = d;
        }
    }
    grid.sync();
    int step = 0;
    for (; step < a.max_steps; step++) {
        int notdone = red_step<MIN>(a, list, cnt, step, t0, stride);
        // block reduction of notdone, one atomic per block
#pragma unroll
        for (int o = 16; o; o >>= 1) notdone += __shfl_xor_sync(0xffffffffu, notdone, o);
        if ((threadIdx.x & 31) == 0) sh[threadIdx.x >> 5] = notdone;
        __syncthreads();
        if (threadIdx.x == 0) {
            int tot = 0;
            for (int w = 0; w < (int)(blockDim.x >> 5); w++) tot += sh[w];
            if (tot) atomicAdd(&ctl[step], tot);
        }
        grid.sync();
        if (*(volatile int*)&ctl[step] == 0) { step++; break; }
    }
    red_epilogue<MIN>(a, list, cnt, step & 1, t0, stride);
}

// Pass 1 expand (break cycles, write the forest) fused with pass 2's local part.
__global__ void __launch_bounds__(LT, LF_LMINB) k_lf_local2(ForestArgs a) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    TileSmem& s = *reinterpret_cast<TileSmem*>(smem_raw);
    const int32_t b0 = (int32_t)(a.lo + (int64_t)blockIdx.x * LB);
    load_tile_w(a.pi2, a.pi2_w, s, b0, a.hi);
    const Tile T{b0, (int32_t)((int64_t)b0 + LB < a.hi ? (int64_t)b0 + LB : a.hi)};
    ulonglong2 ek[VPT];
    slot_keys(a, s, b0, ek);
    pdl_wait();  // the factor slots above predate the chain; the cycle results below do not
    // weakest edge of the cycle through each own vertex (INF: not on a cycle)
    int2 f[VPT];
    unsigned long long ncyc = 0;
#pragma unroll
    for (int k = 0; k < VPT; k++) {
        const int u = threadIdx.x + k * LT;
        const int32_t g = b0 + u;
        const int2 nb = s.nb[u];
        f[k] = nb;
        if (g >= a.hi) continue;
        const short2 p = a.loc1[g];
        uint64_t kstar = KEY_INF;
        if (p.x >= 0 && p.y >= 0) {  // local cycle
            kstar = a.kst[g];
        } else {
            // a segment: its cycle status is that of a terminal that continues in another
            // block (a segment ending in a path end is on a path)
#pragma unroll
            for (int i = 0; i < 2; i++) {
                const int t = -((i ? p.y : p.x) + 1);
                const int2 nbt = s.nb[t];
                const int so = (t == u) ? i : outward_slot(nbt, T);
                const int32_t xo = so ? nbt.y : nbt.x;
                if (xo >= 0 && kstar == KEY_INF) kstar = a.cyc_k[a.bidx1[b0 + t]];
            }
        }
        if (kstar != KEY_INF) {
            if (ek[k].x == kstar) {
                if (g < nb.x) ncyc++;
                f[k].x = f[k].y;
                f[k].y = -1;
            } else if (ek[k].y == kstar) {
                if (g < nb.y) ncyc++;
                f[k].y = -1;
            }
        }
        a.forest[g] = f[k];
    }
    if (a.n_cycles) {
#pragma unroll
        for (int o = 16; o; o >>= 1) ncyc += __shfl_xor_sync(0xffffffffu, ncyc, o);
        if ((threadIdx.x & 31) == 0 && ncyc) atomicAdd(a.n_cycles, ncyc);
    }
    __syncthreads();
    // pass 2 local scan on the broken forest (still in shared memory)
#pragma unroll
    for (int k = 0; k < VPT; k++) s.nb[threadIdx.x + k * LT] = f[k];
    __syncthreads();
    int2 P[VPT], R[VPT];
    ulonglong2 K[VPT];
    tile_rank<false>(s, b0, ek, P, R, K, a.ctl + kCtlStat);
#pragma unroll
    for (int k = 0; k < VPT; k++) {
        const int u = threadIdx.x + k * LT;
        const int32_t g = b0 + u;
        const int2 nb = s.nb[u];
        const bool r0 = nb.x >= 0 && !is_local(nb.x, T);
        const bool r1 = nb.y >= 0 && !is_local(nb.y, T);
        const bool boundary = g < a.hi && (r0 || r1);
        if (g < a.hi) {
            // terminal markers (16 bits each) and local distances (16 bits each)
            const uint32_t pp = ((uint32_t)(uint16_t)(short)P[k].x) | ((uint32_t)(uint16_t)(short)P[k].y << 16);
            const uint32_t rr = ((uint32_t)(uint16_t)R[k].x) | ((uint32_t)(uint16_t)R[k].y << 16);
            a.loc2[g] = make_int2((int)pp, (int)rr);
        }
        const int idx = list_append(a.list2, &a.ctl[kCtlCnt2], g, boundary);
        if (boundary) {
            a.bidx2[g] = idx;
            int32_t q0, q1, d0, d1;
            reduced_dir(a, s, b0, g, nb, 0, P[k], R[k], q0, d0);
            reduced_dir(a, s, b0, g, nb, 1, P[k], R[k], q1, d1);
            a.cq[idx] = make_int2(q0, q1);
            a.cq_k[idx] = make_ulonglong2((uint32_t)d0, (uint32_t)d1);
        }
    }
}

// Pass 2 expand: path ID, position and (at the path-ID vertex) the path length.
__global__ void __launch_bounds__(LT) k_lf_local3(ForestArgs a) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    TileSmem& s = *reinterpret_cast<TileSmem*>(smem_raw);
    const int32_t b0 = (int32_t)(a.lo + (int64_t)blockIdx.x * LB);
    pdl_wait();
    load_tile(a.forest, s, b0, a.hi);
    const Tile T{b0, (int32_t)((int64_t)b0 + LB < a.hi ? (int64_t)b0 + LB : a.hi)};
#pragma unroll
    for (int k = 0; k < VPT; k++) {
        const int u = threadIdx.x + k * LT;
        const int32_t g = b0 + u;
        if (g >= a.hi) continue;
        const int2 lc = a.loc2[g];
        const int px = (short)(lc.x & 0xffff), py = (short)((uint32_t)lc.x >> 16);
        const int rx = lc.y & 0xffff, ry = (int)((uint32_t)lc.y >> 16);
        int32_t E[2], D[2];
#pragma unroll
        for (int i = 0; i < 2; i++) {
            const int t = -((i ? py : px) + 1);  // local terminal in direction i
            const int32_t d = i ? ry : rx;
            const int2 nbt = s.nb[t];
            // the outward slot of t: slot i itself when t == u (the walk never left u)
            const int so = (t == u) ? i : outward_slot(nbt, T);
            const int32_t xo = so ? nbt.y : nbt.x;
            if (xo >= 0) {  // continues in another block: reduced result of t (end marker)
                const int bi = a.bidx2[b0 + t];
                const int2 e = a.end2[bi];
                const int2 dd = a.dist2[bi];
                E[i] = -((so ? e.y : e.x) + 1);
                D[i] = d + (so ? dd.y : dd.x);
            } else {
                E[i] = b0 + t;
                D[i] = d;
            }
        }
        // the ID end l and the forest slot leading to it (the predecessor at p - 1)
        const int dir = E[0] <= E[1] ? 0 : 1;
        const int32_t l = E[dir];
        a.path_id[g] = l;
        a.pos[g] = D[dir] + 1;
        if (a.pdir) a.pdir[g] = (uint8_t)dir;
        a.len[g] = (l == g) ? (D[0] + D[1] + 1) : 0;
    }
}

// Path offsets, single pass: CTA c scans the path lengths of chunk c (kOffChunk vertices,
// in id order) into intra-chunk exclusive offsets and publishes the chunk total; the CTA
// that finishes last turns the totals into an exclusive prefix (tbase).  off[l] of a path
// ID l is then tbase[l / kOffChunk] + off[l].
constexpr int kOffT = 1024, kOffPT = 8, kOffChunk = kOffT * kOffPT;

__global__ void __launch_bounds__(kOffT) k_path_offsets(int64_t N, const int32_t* __restrict__ len,
                                                         int32_t* __restrict__ off, int32_t* tbase,
                                                         int* ticket) {
    __shared__ int sh[32];
    __shared__ int last;
    pdl_wait();
    pdl_trigger();  // one wave: the permutation kernel may launch and wait meanwhile
    const int64_t c0 = (int64_t)blockIdx.x * kOffChunk + (int64_t)threadIdx.x * kOffPT;
    int x[kOffPT];
    int sum = 0;
    if (c0 + kOffPT <= N) {
        const int4* p = reinterpret_cast<const int4*>(len + c0);
#pragma unroll
        for (int j = 0; j < kOffPT / 4; j++) {
            const int4 q = __ldg(p + j);
            x[4 * j] = q.x; x[4 * j + 1] = q.y; x[4 * j + 2] = q.z; x[4 * j + 3] = q.w;
        }
    } else {
#pragma unroll
        for (int j = 0; j < kOffPT; j++) x[j] = c0 + j < N ? __ldg(len + c0 + j) : 0;
    }
#pragma unroll
    for (int j = 0; j < kOffPT; j++) sum += x[j];
    int total = 0;
    int run = block_scan_sum_excl1(sum, sh, &total);
    if (c0 + kOffPT <= N) {
        int4* p = reinterpret_cast<int4*>(off + c0);
#pragma unroll
        for (int j = 0; j < kOffPT / 4; j++) {
            int4 q;
            q.x = run; run += x[4 * j];
            q.y = run; run += x[4 * j + 1];
            q.z = run; run += x[4 * j + 2];
            q.w = run; run += x[4 * j + 3];
            p[j] = q;
        }
    } else {
#pragma unroll
        for (int j = 0; j < kOffPT; j++) {
            if (c0 + j < N) off[c0 + j] = run;
            run += x[j];
        }
    }
    if (threadIdx.x == 0) {
        tbase[blockIdx.x] = total;
        __threadfence();
        last = atomicAdd(ticket, 1) == (int)gridDim.x - 1;
    }
    __syncthreads();
    if (!last) return;
    __threadfence();
    __syncthreads();  // sh is reused below
    int carry = 0;
    for (int base = 0; base < (int)gridDim.x; base += kOffT) {
        const int i = base + threadIdx.x;
        const int v = i < (int)gridDim.x ? __ldcg(tbase + i) : 0;
        int chunk = 0;
        const int ex = block_scan_sum_excl(v, sh, &chunk);
        if (i < (int)gridDim.x) tbase[i] = carry + ex;
        carry += chunk;
    }
}

// step (3) (+ step (4) when tri): r = new(v) = off[l(v)] + p(v) - 1 with off[l] = tile
// prefix + intra-tile prefix; the forest neighbour in slot pdir[v] is perm[r-1], the other
// one perm[r+1], so a[r] / c[r] are copied from the factor's signed slot values
#ifndef LF_PERMB
#define LF_PERMB 2
#endif
constexpr int kPermBatch = LF_PERMB;  // vertices per thread per iteration (loads in flight)
constexpr int kNoSlot = 2;     // pdir: no predecessor / successor slot (k_lf_full1/2)

__global__ void __launch_bounds__(256) k_perm_tri(int64_t N, const int32_t* __restrict__ path_id,
                                                  const int32_t* __restrict__ pos,
                                                  const int32_t* __restrict__ off,
                                                  const int32_t* __restrict__ tbase, int chunk,
                                                  const uint8_t* __restrict__ pdir,
                                                  const int2* __restrict__ forest, const int2* __restrict__ pi2,
                                                  const float2* __restrict__ pi2_val,
                                                  const float* __restrict__ diag, int32_t* __restrict__ perm,
                                                  int32_t* __restrict__ iperm, float* __restrict__ ta,
                                                  float* __restrict__ tb, float* __restrict__ tc,
                                                  const int* __restrict__ ctl) {
    LF_TL(g_tl_forest, 4);
    pdl_wait();
    if (ctl && __ldcg(ctl + kCtlBad)) return;  // a malformed factor: see k_lf_full1
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t v0 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v0 < N; v0 += stride * kPermBatch) {
        int32_t l[kPermBatch], p[kPermBatch], r[kPermBatch];
        float2 pv[kPermBatch];
        float dg[kPermBatch];
        int d[kPermBatch];
        // every per-vertex load first (the coefficients do not depend on the new index)
#pragma unroll
        for (int b = 0; b < kPermBatch; b++) {
            const int64_t v = v0 + b * stride;
            const bool in = v < N;
            l[b] = in ? __ldg(path_id + v) : 0;
            p[b] = in ? __ldg(pos + v) : 0;
            if (ta) {
                pv[b] = in ? __ldg(pi2_val + v) : make_float2(0.f, 0.f);
                d[b] = in ? __ldg(pdir + v) : 0;
                dg[b] = in ? __ldg(diag + v) : 0.f;
            }
        }
#pragma unroll
        for (int b = 0; b < kPermBatch; b++)
            r[b] = v0 + b * stride < N ? __ldg(tbase + l[b] / chunk) + __ldg(off + l[b]) + p[b] - 1 : 0;
#pragma unroll
        for (int b = 0; b < kPermBatch; b++) {
            const int64_t v = v0 + b * stride;
            if (v >= N) continue;
            iperm[v] = r[b];
            perm[r[b]] = (int32_t)v;
            if (ta) {
                const int ps = d[b] & 3, ss = (d[b] >> 2) & 3;
                ta[r[b]] = ps == kNoSlot ? 0.0f : (ps ? pv[b].y : pv[b].x);
                tc[r[b]] = ss == kNoSlot ? 0.0f : (ss ? pv[b].y : pv[b].x);
                tb[r[b]] = dg[b];
            }
        }
    }
}

// ===========================================================================
// Single-pass linear forest.  Every scan level carries the FULL window
// of a vertex in one direction instead of one quantity per pass:
//   pointer | R = edges covered | K = minimum edge key | DK = 2 * (distance to the near
//   endpoint of that minimum edge) + [the near endpoint is the edge's min-id endpoint].
// Appending window B (starting where A ends) to A:  R = R_A + R_B;  if K_B < K_A then
// K = K_B, DK = 2 R_A + DK_B.  The strict '<' keeps the first occurrence, so on a cycle
// DK is the true distance to the weakest edge (reading c9) in that direction, and with
// K (whose rank field names the min-id endpoint x, reading c11) it gives every cycle
// vertex its position on the broken cycle directly: pos = distance to x + 1 (reading c12).
// So cycles are broken AND all vertices ranked by one tile pass (k_lf_full1), one reduced
// scan (k_red_full) and one expand pass (k_lf_full2), instead of two of each.
// ===========================================================================

// the min-id endpoint of the edge behind a key (rank = 2 min + c, see edge_key)
__device__ __forceinline__ int32_t key_min_end(uint64_t k) {
    return (int32_t)((0xFFFFFFFFu - (uint32_t)k) >> 1);
}

struct TileSmemF {
    int2 nb[LB];          // slots (global ids); run slots virtual after contraction
    union {
        float2 w[LB];     // |w| per slot (read by slot_keys)
        struct {
            short2 run[LB];
            short2 vw[LB];
        } r;
    };
    uint64_t EK0[LB];     // key of the (virtual) link behind slot 0 / slot 1
    uint64_t EK1[LB];
    short sidx[LB];
    short spl[LB];
    short2 recS[LB];
    short2 recD[LB];
    // splitter-node arrays
    short2 P[LB];
    short2 R[LB];
    short2 DK[LB];
    uint64_t K0[LB];      // (also per-vertex temporaries of the run scan, before the walks)
    uint64_t K1[LB];
    uint64_t WK0[LB];     // minimum of each node's walk per slot (kept through the node scan)
    uint64_t WK1[LB];
    short2 WD[LB];        // DK of that minimum, from the node
    int nspl;
    int32_t b0, tend;
};
static_assert(sizeof(TileSmemF) <= 227 * 1024, "tile smem");

// DK of the (possibly virtual) link behind slot `slot` of local vertex u, from u
__device__ __forceinline__ int slot_dk(const TileSmemF& s, int u, int32_t g, int slot) {
    const int2 nb = s.nb[u];
    const int32_t z = slot ? nb.y : nb.x;
    const short2 vw = s.r.vw[u];
    if ((slot ? vw.y : vw.x) == 1) return g < z ? 1 : 0;  // a real link: near endpoint u
    const int32_t m = key_min_end(slot ? s.EK1[u] : s.EK0[u]);  // run minimum: link (m, m+1)
    return z > g ? 2 * (m - g) + 1 : 2 * (g - (m + 1));
}

// the virtual (run) slot of run end u whose other end is o
__device__ __forceinline__ int run_slot(const TileSmemF& s, int u, int32_t og) {
    const short2 vw = s.r.vw[u];
    if (vw.x > 1) return 0;
    if (vw.y > 1) return 1;
    return s.nb[u].x == og ? 0 : 1;
}

// Result of the tile pass for one own vertex
struct VRes {
    bool cyc;         // on a cycle that lies inside the tile
    int2 T;           // path type: local terminals per slot
    int2 R;           //   distances to them
    uint64_t Ks;      // cycle: its weakest edge key
    int2 C;           //   DK per slot (toward the weakest edge)
    ulonglong2 Kn;    // splitter node: window keys per slot (reduced records)
    int2 Dn;          //   window DK per slot
};

// named barrier 1 over the first nt threads (nt a multiple of 32), with an OR reduction
__device__ __forceinline__ void group_sync(int nt) {
    if (nt == LT) __syncthreads();
    else asm volatile("bar.sync 1, %0;" ::"r"(nt) : "memory");
}
__device__ __forceinline__ int group_or(int nt, int pred) {
    if (nt == LT) return __syncthreads_or(pred);
    int r;
    asm volatile("{\n\t.reg .pred p, q;\n\tsetp.ne.s32 p, %1, 0;\n\tbar.red.or.pred q, 1, %2, p;\n\tselp.s32 %0, 1, 0, q;\n\t}"
                 : "=r"(r) : "r"(pred), "r"(nt) : "memory");
    return r;
}

// the same scan for C <= 32 nodes by one warp, node i in lane i: the targets' windows
// come by shuffles, so a step needs no shared memory and no barrier (C2's contracted
// tiles have ~16 nodes)
__device__ __forceinline__ void node_scan_warp(TileSmemF& s, int C, int* stats) {
    const int i = threadIdx.x & 31;
    const bool on = i < C;
    int2 p = make_int2(-1, -1), r = make_int2(0, 0), dk = make_int2(0, 0);
    uint64_t k0 = KEY_INF, k1 = KEY_INF;
    if (on) {
        const short2 ps = s.P[i], rs = s.R[i], ds = s.DK[i];
        p = make_int2(ps.x, ps.y);
        r = make_int2(rs.x, rs.y);
        dk = make_int2(ds.x, ds.y);
        k0 = s.K0[i];
        k1 = s.K1[i];
    }
    for (int step = 0; step < 16; step++) {
        int2 q = p, nr = r, nd = dk;
        uint64_t n0 = k0, n1 = k1;
#pragma unroll
        for (int dd = 0; dd < 2; dd++) {
            const int w = dd ? p.y : p.x;
            const int src = (on && w >= 0) ? w : i;
            const int pwx = __shfl_sync(0xffffffffu, p.x, src), pwy = __shfl_sync(0xffffffffu, p.y, src);
            const int rwx = __shfl_sync(0xffffffffu, r.x, src), rwy = __shfl_sync(0xffffffffu, r.y, src);
            const int dwx = __shfl_sync(0xffffffffu, dk.x, src), dwy = __shfl_sync(0xffffffffu, dk.y, src);
            const uint64_t kw0 = __shfl_sync(0xffffffffu, k0, src), kw1 = __shfl_sync(0xffffffffu, k1, src);
            if (!on || w < 0) continue;
            const int Rd = dd ? r.y : r.x;
            uint64_t kc = dd ? k1 : k0;
            int dc = dd ? dk.y : dk.x;
            int j = -1;
            if (pwx != i) j = 0;
            else if (pwy != i) j = 1;
            if (j >= 0) {
                const uint64_t kw = j ? kw1 : kw0;
                if (kw < kc) { kc = kw; dc = 2 * Rd + (j ? dwy : dwx); }
                const int tgt = j ? pwy : pwx;
                const int rr = Rd + (j ? rwy : rwx);
                if (dd) { q.y = tgt; nr.y = rr; } else { q.x = tgt; nr.x = rr; }
            } else {  // stall (reading c13), as in node_scan_full
                if (kw0 < kc) { kc = kw0; dc = 2 * Rd + dwx; }
                if (kw1 < kc) { kc = kw1; dc = 2 * Rd + dwy; }
            }
            if (dd) { n1 = kc; nd.y = dc; } else { n0 = kc; nd.x = dc; }
        }
        p = q; r = nr; dk = nd; k0 = n0; k1 = n1;
        const bool path_done = q.x < 0 && q.y < 0;
        const bool cyc_done = q.x >= 0 && q.y >= 0 && n0 == n1;
        if (!__any_sync(0xffffffffu, on && !(path_done || cyc_done))) {
            if (i == 0 && stats) atomicMax(&stats[4], step + 1);
            break;
        }
    }
    if (on) {
        s.P[i] = make_short2((short)p.x, (short)p.y);
        s.R[i] = make_short2((short)r.x, (short)r.y);
        s.DK[i] = make_short2((short)dk.x, (short)dk.y);
        s.K0[i] = k0;
        s.K1[i] = k1;
    }
}

// bidirectional scan over the splitter nodes with full windows, by the first nt threads
// (NPN nodes each); the caller synchronises the block afterwards
template <int NPN>
__device__ __forceinline__ void node_scan_full(TileSmemF& s, int C, int nt, int* stats) {
    const int tid = threadIdx.x;
    for (int step = 0; step < 16; step++) {
        int notdone = 0;
        short2 nP[NPN], nR[NPN], nD[NPN];
        uint64_t nk0[NPN], nk1[NPN];
#pragma unroll
        for (int k = 0; k < NPN; k++) {
            const int i = tid + k * nt;
            if (i >= C) continue;
            const short2 p = s.P[i];
            short2 q = p, r = s.R[i], dk = s.DK[i];
            uint64_t k0 = s.K0[i], k1 = s.K1[i];
#pragma unroll
            for (int dd = 0; dd < 2; dd++) {
                const int w = dd ? p.y : p.x;
                if (w < 0) continue;
                const short2 pw = s.P[w];
                const int Rd = dd ? r.y : r.x;
                uint64_t kc = dd ? k1 : k0;
                int dc = dd ? dk.y : dk.x;
                int j = -1;
                if (pw.x != i) j = 0;
                else if (pw.y != i) j = 1;
                const short2 rw = s.R[w], dw = s.DK[w];
                const uint64_t kw0 = s.K0[w], kw1 = s.K1[w];
                if (j >= 0) {
                    const uint64_t kw = j ? kw1 : kw0;
                    if (kw < kc) { kc = kw; dc = 2 * Rd + (j ? dw.y : dw.x); }
                    const short tgt = j ? pw.y : pw.x;
                    const short nr = (short)(Rd + (j ? rw.y : rw.x));
                    if (dd) { q.y = tgt; r.y = nr; } else { q.x = tgt; r.x = nr; }
                } else {
                    // stall (reading c13): both windows of w return here; the one that
                    // continues covers the rest of the cycle, the other only repeats this
                    // window's edges and can never win the strict compare
                    if (kw0 < kc) { kc = kw0; dc = 2 * Rd + dw.x; }
                    if (kw1 < kc) { kc = kw1; dc = 2 * Rd + dw.y; }
                }
                if (dd) { k1 = kc; dk.y = (short)dc; } else { k0 = kc; dk.x = (short)dc; }
            }
            nP[k] = q; nR[k] = r; nD[k] = dk; nk0[k] = k0; nk1[k] = k1;
            const bool path_done = q.x < 0 && q.y < 0;
            const bool cyc_done = q.x >= 0 && q.y >= 0 && k0 == k1;
            notdone |= !(path_done || cyc_done);
        }
        group_sync(nt);
#pragma unroll
        for (int k = 0; k < NPN; k++) {
            const int i = tid + k * nt;
            if (i >= C) continue;
            s.P[i] = nP[k]; s.R[i] = nR[k]; s.DK[i] = nD[k]; s.K0[i] = nk0[k]; s.K1[i] = nk1[k];
        }
        if (!group_or(nt, notdone)) {
            if (tid == 0 && stats) atomicMax(&stats[4], step + 1);
            break;
        }
    }
}

// Block-local ranking with full windows (same phases as tile_rank).
// ek: real slot keys of the own vertices.  On return o[k] holds the vertex's result.
__device__ void tile_rank_full(TileSmemF& s, int32_t b0, const ulonglong2 (&ek)[VPT], VRes (&o)[VPT],
                               int* stats) {
    __shared__ int sh[32];
    const int tid = threadIdx.x;
    const Tile T = tile_of(s);
    const int tlen = T.tend - T.b0;
    int* ctlp = stats - kCtlStat;
    LF_PHASE_INIT;
    if (tid == 0) s.nspl = 0;
    const auto linked_prev = [&](int u) {
        const int2 nb = s.nb[u];
        const int32_t g = b0 + u;
        return u > 0 && u < tlen && (nb.x == g - 1 || nb.y == g - 1);
    };
    // 0a. slot keys; K0 = key of the run link (u-1, u)
#pragma unroll
    for (int k = 0; k < VPT; k++) {
        const int u = tid + k * LT;
        const int2 nb = s.nb[u];
        const int32_t g = b0 + u;
        const bool lp = u > 0 && u < tlen && (nb.x == g - 1 || nb.y == g - 1);
        s.EK0[u] = ek[k].x;
        s.EK1[u] = ek[k].y;
        s.K0[u] = lp ? (nb.x == g - 1 ? ek[k].x : ek[k].y) : KEY_INF;
    }
    // 0b. run bounds and each run's weakest link, with one block barrier: heads (no link
    //     to u-1) by warp ballots, the running minimum of K0 by a warp segmented scan,
    //     and the runs that cross warps from per-warp aggregates (last / first head, tail
    //     minimum) that every warp reduces for itself.  Position 0 is always a head.
    __syncthreads();  // K0 of 0a (other threads' vertices)
    {
        constexpr int NW = LT / 32;
        __shared__ int w_last[NW], w_first[NW], w_has[NW];
        __shared__ uint64_t w_min[NW];
        const int lane = tid & 31, wid = tid >> 5;
        const int u0 = tid * VPT;
        bool lk[VPT];
        uint64_t kv[VPT];
        int firstHead = INT_MAX, lastHead = -1;
        uint64_t tmin = KEY_INF;
#pragma unroll
        for (int j = 0; j < VPT; j++) {
            lk[j] = linked_prev(u0 + j);
            kv[j] = s.K0[u0 + j];
            if (!lk[j]) { if (firstHead == INT_MAX) firstHead = u0 + j; lastHead = u0 + j; }
            tmin = lk[j] ? umin64(tmin, kv[j]) : kv[j];
        }
        // warp segmented inclusive scan of the thread tails (reset at a thread with a head)
        uint64_t v = tmin;
        bool f = lastHead >= 0;
#pragma unroll
        for (int o2 = 1; o2 < 32; o2 <<= 1) {
            const uint64_t yv = __shfl_up_sync(0xffffffffu, v, o2);
            const int yf = __shfl_up_sync(0xffffffffu, (int)f, o2);
            if (lane >= o2) { if (!f) v = umin64(v, yv); f = f || yf; }
        }
        uint64_t cv = __shfl_up_sync(0xffffffffu, v, 1);
        bool cf = __shfl_up_sync(0xffffffffu, (int)f, 1) != 0;
        if (lane == 0) { cv = KEY_INF; cf = false; }
        const unsigned hm = __ballot_sync(0xffffffffu, lastHead >= 0);
        const int wl = __reduce_max_sync(0xffffffffu, lastHead);
        const unsigned wf = __reduce_min_sync(0xffffffffu, (unsigned)firstHead);
        if (lane == 31) { w_min[wid] = v; w_has[wid] = f; }
        if (lane == 0) { w_last[wid] = wl; w_first[wid] = (int)wf; }
        __syncthreads();
        // from the other warps: the last head before, the first head after, and the
        // minimum over the run that enters this warp from before
        const int pl = lane < wid ? w_last[lane] : -1;
        const int prevLast = __reduce_max_sync(0xffffffffu, pl);
        const unsigned nfv = (lane > wid && lane < NW) ? (unsigned)w_first[lane] : (unsigned)INT_MAX;
        const int nextFirst = (int)__reduce_min_sync(0xffffffffu, nfv);
        const int hw = __reduce_max_sync(0xffffffffu, (lane < wid && w_has[lane]) ? lane : 0);
        uint64_t cm = (lane >= hw && lane < wid) ? w_min[lane] : KEY_INF;
#pragma unroll
        for (int o2 = 16; o2; o2 >>= 1) cm = umin64(cm, __shfl_xor_sync(0xffffffffu, cm, o2));
        // this thread's incoming run start, running minimum and next head
        const unsigned before = hm & ((1u << lane) - 1u);
        const int srcb = before ? 31 - __clz(before) : lane;
        const int lastB = __shfl_sync(0xffffffffu, lastHead, srcb);
        int start = before ? lastB : prevLast;
        const unsigned after = lane == 31 ? 0u : (hm & ~((2u << lane) - 1u));
        const int srca = after ? __ffs(after) - 1 : lane;
        const int firstA = __shfl_sync(0xffffffffu, firstHead, srca);
        int nh = after ? firstA : nextFirst;
        uint64_t r = cf ? cv : umin64(cv, cm);
        short2 rr[VPT];
        uint64_t km[VPT];
#pragma unroll
        for (int j = 0; j < VPT; j++) {
            if (!lk[j]) { start = u0 + j; r = kv[j]; } else r = umin64(r, kv[j]);
            rr[j].x = (short)start;
            km[j] = r;
        }
#pragma unroll
        for (int j = VPT - 1; j >= 0; j--) {
            rr[j].y = (short)(nh == INT_MAX ? LB - 1 : nh - 1);
            if (!lk[j]) nh = u0 + j;
        }
#pragma unroll
        for (int j = 0; j < VPT; j++) { s.r.run[u0 + j] = rr[j]; s.K1[u0 + j] = km[j]; }
    }
    __syncthreads();
    // 0c. contract runs: virtual links between run ends (length, weakest key)
#pragma unroll
    for (int k = 0; k < VPT; k++) {
        const int u = tid + k * LT;
        const short2 rr = s.r.run[u];
        const int32_t g = b0 + u;
        short2 vw = make_short2(1, 1);
        const int len = rr.y - rr.x + 1;
        if (len >= 2 && (u == rr.x || u == rr.y)) {
            const int other = (u == rr.x) ? rr.y : rr.x;
            const int32_t inside = (u == rr.x) ? g + 1 : g - 1;
            int2 nb = s.nb[u];
            const uint64_t rk = s.K1[rr.y];
            if (nb.x == inside) { nb.x = b0 + other; vw.x = (short)(len - 1); s.EK0[u] = rk; }
            else { nb.y = b0 + other; vw.y = (short)(len - 1); s.EK1[u] = rk; }
            s.nb[u] = nb;
        }
        s.r.vw[u] = vw;
    }
    // no barrier: phase 1 reads only its own vertices' contracted slots and runs (this
    // thread wrote the slots; the runs are from before the last barrier)
    LF_PHASE(ctlp, 0);
    // 1. splitters (run ends, terminals, hashed vertices); run cycles -3, interiors -2
#pragma unroll
    for (int k = 0; k < VPT; k++) {
        const int u = tid + k * LT;
        const short2 rr = s.r.run[u];
        const int2 nb = s.nb[u];
        const bool interior = u > rr.x && u < rr.y;
        const bool run_cycle = rr.y - rr.x >= 2 && nb.x == nb.y;
        short id = -1;
        bool node = false;
        if (u >= tlen) {
            node = true;
        } else if (interior || run_cycle) {
            id = run_cycle ? -3 : -2;
        } else {
            const bool l0 = nb.x >= 0 && is_local(nb.x, T);
            const bool l1 = nb.y >= 0 && is_local(nb.y, T);
            node = !l0 || !l1 || rr.y > rr.x || hashed_splitter(b0 + u);
        }
        {
            const unsigned m = __ballot_sync(0xffffffffu, node);
            const int lane = tid & 31;
            int base = 0;
            if (lane == 0 && m) base = atomicAdd(&s.nspl, __popc(m));
            base = __shfl_sync(0xffffffffu, base, 0);
            if (node) id = (short)(base + __popc(m & ((1u << lane) - 1u)));
        }
        s.sidx[u] = id;
        if (id >= 0) s.spl[id] = (short)u;
        s.recS[u] = make_short2(-1, -1);
    }
    __syncthreads();
    LF_PHASE(ctlp, 1);
    const int C = s.nspl;
    if (tid == 0 && stats) atomicAdd(&stats[0], C);
    // 2. walks from every (node, slot) to the next node: length, weakest link and its DK
    for (int wk = tid; wk < 2 * C; wk += LT) {
        const int i = wk >> 1, f = wk & 1;
        const int su = s.spl[i];
        const int2 nbs = s.nb[su];
        const int32_t x = f ? nbs.y : nbs.x;
        short ptr = (short)(-(i + 1));
        int dist = 0, dk = 0;
        uint64_t km = KEY_INF;
        if (x >= 0 && is_local(x, T)) {
            const short2 vws = s.r.vw[su];
            int prev = su, cur = x - b0, d = f ? vws.y : vws.x;
            km = f ? s.EK1[su] : s.EK0[su];
            dk = slot_dk(s, su, b0 + su, f);
            for (int guard = 0; s.sidx[cur] < 0; guard++) {
                const int2 nbc = s.nb[cur];
                const int face = (nbc.x == b0 + prev) ? 0 : 1;
                if (face == 0) { s.recS[cur].x = (short)((i << 1) | f); s.recD[cur].x = (short)d; }
                else { s.recS[cur].y = (short)((i << 1) | f); s.recD[cur].y = (short)d; }
                const int nxt = (face ? nbc.x : nbc.y) - b0;
                if ((unsigned)nxt >= (unsigned)LB || guard >= LB) {  // a malformed factor (not symmetric)
                    if (stats) atomicOr(stats + (kCtlBad - kCtlStat), 1);
                    break;
                }
                const uint64_t kk = face ? s.EK0[cur] : s.EK1[cur];
                if (kk < km) {  // a walk passes real links only (run ends are nodes)
                    km = kk;
                    dk = 2 * d + ((b0 + cur) < (face ? nbc.x : nbc.y) ? 1 : 0);
                }
                d += 1;
                prev = cur;
                cur = nxt;
            }
            ptr = s.sidx[cur];
            dist = d;
        }
        if (f) { s.P[i].y = ptr; s.R[i].y = (short)dist; s.DK[i].y = (short)dk; s.K1[i] = km; s.WK1[i] = km; s.WD[i].y = (short)dk; }
        else { s.P[i].x = ptr; s.R[i].x = (short)dist; s.DK[i].x = (short)dk; s.K0[i] = km; s.WK0[i] = km; s.WD[i].x = (short)dk; }
    }
    __syncthreads();
    LF_PHASE(ctlp, 2);
    // 3. node scan: one warp (shuffles) or one node per thread of the smallest group
    if (C <= 32) {
        if (tid < 32) node_scan_warp(s, C, stats);
        __syncthreads();
    } else if (C <= 128 && LT > 128) {
        if (tid < 128) node_scan_full<1>(s, C, 128, stats);
        __syncthreads();
    } else if (C <= 512 && LT > 512) {
        if (tid < 512) node_scan_full<1>(s, C, 512, stats);
        __syncthreads();
    } else {
        node_scan_full<VPT>(s, C, LT, stats);
        __syncthreads();
    }
    LF_PHASE(ctlp, 3);
    // 4. nodes and walk-visited vertices
    bool unvisited[VPT];
    int any_unvisited = 0;
#pragma unroll
    for (int k = 0; k < VPT; k++) {
        const int u = tid + k * LT;
        unvisited[k] = false;
        VRes& r = o[k];
        r.cyc = false;
        r.T = make_int2(u, u);
        r.R = make_int2(0, 0);
        r.Ks = KEY_INF;
        r.C = make_int2(0, 0);
        r.Kn = make_ulonglong2(KEY_INF, KEY_INF);
        r.Dn = make_int2(0, 0);
        const int id = s.sidx[u];
        if (id == -2 || id == -3) continue;
        if (id >= 0) {
            const short2 p = s.P[id];
            const short2 dk = s.DK[id];
            r.Kn = make_ulonglong2(s.K0[id], s.K1[id]);
            r.Dn = make_int2(dk.x, dk.y);
            if (p.x >= 0 && p.y >= 0) {
                r.cyc = true;
                r.Ks = s.K0[id];
                r.C = make_int2(dk.x, dk.y);
            } else {
                const short2 rr = s.R[id];
                r.T = make_int2(s.spl[-(p.x + 1)], s.spl[-(p.y + 1)]);
                r.R = make_int2(rr.x, rr.y);
            }
            continue;
        }
        const short2 rs = s.recS[u];
        if (rs.x < 0 && rs.y < 0) { unvisited[k] = true; any_unvisited = 1; continue; }
        const short2 rd = s.recD[u];
#pragma unroll
        for (int f = 0; f < 2; f++) {
            const int rec = f ? rs.y : rs.x;
            const int i = rec >> 1, f0 = rec & 1, away = f0 ^ 1;
            const short2 p = s.P[i];
            const int pa = away ? p.y : p.x;
            const int d = f ? rd.y : rd.x;
            if (pa >= 0) {  // cycle: the weakest key is the node's (both windows agree)
                const uint64_t kc = s.K0[i];
                const uint64_t wk = f0 ? s.WK1[i] : s.WK0[i];
                const short2 wdp = s.WD[i];
                const int wd = f0 ? wdp.y : wdp.x;
                int cf;
                if (wk == kc && (wd >> 1) + 1 <= d) cf = 2 * (d - (wd >> 1) - 1) + ((wd & 1) ^ 1);
                else { const short2 dk = s.DK[i]; cf = 2 * d + (away ? dk.y : dk.x); }
                r.cyc = true;
                r.Ks = kc;
                if (f) r.C.y = cf; else r.C.x = cf;
            } else {
                const short2 rr = s.R[i];
                const int t = s.spl[-(pa + 1)];
                const int dd = d + (away ? rr.y : rr.x);
                if (f) { r.T.y = t; r.R.y = dd; } else { r.T.x = t; r.R.x = dd; }
            }
        }
    }
    // 4b. cycles of the contracted tile graph without a splitter (real links only): each
    //     of their vertices walks its cycle once
    if (__syncthreads_or(any_unvisited)) {
        if (tid == 0 && stats) atomicAdd(&stats[2], 1);
#pragma unroll
        for (int k = 0; k < VPT; k++) {
            if (!unvisited[k]) continue;
            const int u = tid + k * LT;
            if (stats) atomicAdd(&stats[1], 1);
            int prev = u, cur = s.nb[u].x - b0, d = 1;
            uint64_t km = s.EK0[u];
            int kd = (b0 + u) < s.nb[u].x ? 1 : 0;
            for (int guard = 0; cur != u; guard++) {
                if ((unsigned)cur >= (unsigned)LB || guard >= LB) {  // a malformed factor
                    if (stats) atomicOr(stats + (kCtlBad - kCtlStat), 1);
                    break;
                }
                const int2 nbc = s.nb[cur];
                const int face = (nbc.x == b0 + prev) ? 0 : 1;
                const uint64_t kk = face ? s.EK0[cur] : s.EK1[cur];
                const int32_t z = face ? nbc.x : nbc.y;
                if (kk < km) { km = kk; kd = 2 * d + ((b0 + cur) < z ? 1 : 0); }
                prev = cur;
                cur = z - b0;
                d++;
            }
            o[k].cyc = true;
            o[k].Ks = km;
            o[k].C = make_int2(kd, 2 * (d - (kd >> 1) - 1) + ((kd & 1) ^ 1));
        }
    }
    // 5. interior run vertices and run cycles, from the run ends' node windows (phase 4
    //    wrote registers only: no barrier needed since the one inside it)
    LF_PHASE(ctlp, 4);
#pragma unroll
    for (int k = 0; k < VPT; k++) {
        const int u = tid + k * LT;
        const int id = s.sidx[u];
        if (id != -2 && id != -3) continue;
        VRes& r = o[k];
        const short2 rr = s.r.run[u];
        const int a = rr.x, b = rr.y;
        const int32_t g = b0 + u;
        const int2 nb = s.nb[u];
        const int va = run_slot(s, a, b0 + b);
        const uint64_t RK = va ? s.EK1[a] : s.EK0[a];       // the run's weakest link
        const int ml = key_min_end(RK) - b0;                 // it is (ml, ml+1)
        // slots of u toward u-1 ("down") and u+1 ("up"); for the ends of a run cycle the
        // closing link continues the direction
        int sdown;
        if (u == a) sdown = va ^ 1;
        else if (u == b) sdown = run_slot(s, b, b0 + a);
        else sdown = (nb.x == g - 1) ? 0 : 1;
        int down, up;  // DK toward u-1 / u+1 (cycles)
        if (s.sidx[a] == -3) {  // the run closes into a cycle through the link (b, a)
            const uint64_t CK = va ? s.EK0[a] : s.EK1[a];
            const uint64_t ks = umin64(RK, CK);
            if (ks == CK) {
                up = 2 * (b - u);            // near endpoint b (not the min id)
                down = 2 * (u - a) + 1;      // near endpoint a = x
            } else {
                up = (u <= ml) ? 2 * (ml - u) + 1 : 2 * ((b - u) + 1 + (ml - a)) + 1;
                down = (u >= ml + 1) ? 2 * (u - ml - 1) : 2 * ((u - a) + 1 + (b - ml - 1));
            }
            r.cyc = true;
            r.Ks = ks;
        } else {
            const int ia = s.sidx[a], ib = s.sidx[b];
            const int oa = va ^ 1, ob = run_slot(s, b, b0 + a) ^ 1;   // outer slots of the ends
            const short2 pa = s.P[ia], pb = s.P[ib];
            const int qa = oa ? pa.y : pa.x, qb = ob ? pb.y : pb.x;
            if (qa >= 0) {  // on a cycle
                const uint64_t ks = s.K0[ia];
                const short2 da = s.DK[ia], db = s.DK[ib];
                down = (ks == RK && ml + 1 <= u) ? 2 * (u - ml - 1) : 2 * (u - a) + (oa ? da.y : da.x);
                up = (ks == RK && ml >= u) ? 2 * (ml - u) + 1 : 2 * (b - u) + (ob ? db.y : db.x);
                r.cyc = true;
                r.Ks = ks;
            } else {
                const short2 ra = s.R[ia], rb = s.R[ib];
                const int ta = s.spl[-(qa + 1)], tb = s.spl[-(qb + 1)];
                const int dA = (u - a) + (oa ? ra.y : ra.x), dB = (b - u) + (ob ? rb.y : rb.x);
                r.cyc = false;
                if (sdown == 0) { r.T = make_int2(ta, tb); r.R = make_int2(dA, dB); }
                else { r.T = make_int2(tb, ta); r.R = make_int2(dB, dA); }
                continue;
            }
        }
        r.C = sdown == 0 ? make_int2(down, up) : make_int2(up, down);
    }
    LF_PHASE(ctlp, 5);
}

// A vertex on a cycle (weakest key ks, DK per slot c): path id, position, forest slots,
// predecessor slot, path length at the path-ID vertex.  Reading c11/c12/c15/c9.
// predecessor / successor slots of a vertex in pi2-slot terms for the tridiagonal copy:
// bits 0-1 the slot toward the path-ID end (position p - 1), bits 2-3 the other one
// (p + 1); kNoSlot where that neighbour is missing or its edge was removed (slot rs)
__device__ __forceinline__ uint8_t nbr_slots(int2 nb, int dir, int rs) {
    const int32_t xp = dir ? nb.y : nb.x, xs = dir ? nb.x : nb.y;
    const int ps = (dir != rs && xp >= 0) ? dir : kNoSlot;
    const int ss = ((dir ^ 1) != rs && xs >= 0) ? (dir ^ 1) : kNoSlot;
    return (uint8_t)(ps | (ss << 2));
}

struct CycOut {
    int32_t l, pos, len;
    int2 f;
    uint8_t pdir;
    int ncyc;
};
__device__ __forceinline__ CycOut cycle_finish(int32_t g, int2 nb, ulonglong2 ek, uint64_t ks, int2 c) {
    CycOut o;
    o.l = key_min_end(ks);
    const int dir = (c.x & 1) ? 0 : 1;           // the slot whose near endpoint is x
    o.pos = ((dir ? c.y : c.x) >> 1) + 1;
    o.len = (g == o.l) ? (c.x >> 1) + (c.y >> 1) + 1 : 0;
    const int rs = (ek.x == ks) ? 0 : ((ek.y == ks) ? 1 : -1);
    o.f = nb;
    o.ncyc = 0;
    if (rs == 0) { o.f = make_int2(nb.y, -1); o.ncyc = g < nb.x; }
    else if (rs == 1) { o.f = make_int2(nb.x, -1); o.ncyc = g < nb.y; }
    o.pdir = nbr_slots(nb, dir, rs);
    return o;
}

// ---------------------------------------------------------------------------
// Reduced scan with full windows over the boundary list (pointers are list positions)
// ---------------------------------------------------------------------------
__device__ __forceinline__ void win_append(int32_t& R, uint64_t& K, int32_t& D, int32_t Rw, uint64_t Kw, int32_t Dw) {
    if (Kw < K) { K = Kw; D = 2 * R + Dw; }
    R += Rw;
}

// list position of the vertex a record points at (markers pass through)
__device__ __forceinline__ int2 to_pos(const ForestArgs& a, int2 q) {
    return make_int2(q.x >= 0 ? __ldcg(a.bidx1 + q.x) : q.x, q.y >= 0 ? __ldcg(a.bidx1 + q.y) : q.y);
}

// The reduced scan of lists up to kRedCl * kRedClNodes nodes on ONE thread-block cluster:
// node i lives in shared memory of CTA i / NPC (slot i % NPC) and every step reads the
// target's window through DSMEM.  One CTA's shared memory would hold C2's 5 k nodes,
// but then every step's random (bank-conflicted) window reads are served by a single SM;
// a cluster spreads them over kRedCl SMs (8 and 16 measure the same on C2; 4 is slower).
// Windows are ping-ponged between two
// buffers (a step reads buffer b everywhere and writes buffer b^1 of its own nodes), so
// one cluster barrier per step suffices; finished path nodes are copied forward.
#ifndef LF_REDCL
#define LF_REDCL 8
#endif
constexpr int kRedCl = LF_REDCL;     // CTAs of the cluster (portable size; 16 measured the same on C2)
constexpr int kRedClNodes = 2048;    // nodes per CTA
struct RedSmemC {
    int2 q[2][kRedClNodes];
    int r[2][2][kRedClNodes];        // [buffer][direction][slot]
    int d[2][2][kRedClNodes];
    uint64_t k[2][2][kRedClNodes];
    int nd[2];                       // this CTA's "some node not done" per step parity
};

__device__ void red_full_cluster(const ForestArgs& a, int cnt, int* ctl, RedSmemC& S) {
    constexpr int NPT = kRedClNodes / RT;
    cg::cluster_group cl = cg::this_cluster();
    const int rank = (int)cl.block_rank();
    const int tid = threadIdx.x;
    const int NPC = (cnt + kRedCl - 1) / kRedCl;
    const int base = rank * NPC;
    const int nmine = max(0, min(cnt - base, NPC));
    __shared__ RedSmemC* rem[kRedCl];
    if (tid < kRedCl) rem[tid] = cl.map_shared_rank(&S, tid);
    {
        int2 q[NPT], r[NPT], d[NPT];
        ulonglong2 kk[NPT];
#pragma unroll
        for (int k = 0; k < NPT; k++) {
            const int t = tid + k * RT;
            if (t >= nmine) continue;
            q[k] = __ldcg(a.cq + base + t);
            r[k] = __ldcg(a.cq_r + base + t);
            d[k] = __ldcg(a.cq_dk + base + t);
            kk[k] = __ldcg(a.cq_k + base + t);
        }
#pragma unroll
        for (int k = 0; k < NPT; k++) {
            const int t = tid + k * RT;
            if (t >= nmine) continue;
            q[k] = to_pos(a, q[k]);
            S.q[0][t] = q[k];
            S.r[0][0][t] = r[k].x; S.r[0][1][t] = r[k].y;
            S.d[0][0][t] = d[k].x; S.d[0][1][t] = d[k].y;
            S.k[0][0][t] = kk[k].x; S.k[0][1][t] = kk[k].y;
        }
    }
    cl.sync();
    int b = 0;
    for (int step = 0; step < a.max_steps; step++) {
        int notdone = 0;
#pragma unroll
        for (int k = 0; k < NPT; k++) {
            const int t = tid + k * RT;
            if (t >= nmine) continue;
            const int me = base + t;
            const int2 q = S.q[b][t];
            int2 nq = q;
            int32_t R[2] = {S.r[b][0][t], S.r[b][1][t]}, D[2] = {S.d[b][0][t], S.d[b][1][t]};
            uint64_t K[2] = {S.k[b][0][t], S.k[b][1][t]};
            if (!(q.x < 0 && q.y < 0)) {  // finished paths are only copied forward
#pragma unroll
                for (int i = 0; i < 2; i++) {
                    const int w = i ? q.y : q.x;
                    if (w < 0) continue;
                    const int rw = w / NPC, sw = w - rw * NPC;
                    const RedSmemC* P = rem[rw];
                    const int2 qw = P->q[b][sw];
                    int j = -1;
                    if (qw.x != me) j = 0;
                    else if (qw.y != me) j = 1;
                    if (j >= 0) {
                        win_append(R[i], K[i], D[i], P->r[b][j][sw], P->k[b][j][sw], P->d[b][j][sw]);
                        if (i) nq.y = j ? qw.y : qw.x; else nq.x = j ? qw.y : qw.x;
                    } else {  // stall (reading c13): see node_scan_full
                        const uint64_t kw0 = P->k[b][0][sw], kw1 = P->k[b][1][sw];
                        if (kw0 < K[i]) { K[i] = kw0; D[i] = 2 * R[i] + P->d[b][0][sw]; }
                        if (kw1 < K[i]) { K[i] = kw1; D[i] = 2 * R[i] + P->d[b][1][sw]; }
                    }
                }
                const bool path_done = nq.x < 0 && nq.y < 0;
                const bool cyc_done = nq.x >= 0 && nq.y >= 0 && K[0] == K[1];
                notdone |= !(path_done || cyc_done);
            }
            S.q[b ^ 1][t] = nq;
#pragma unroll
            for (int i = 0; i < 2; i++) { S.r[b ^ 1][i][t] = R[i]; S.d[b ^ 1][i][t] = D[i]; S.k[b ^ 1][i][t] = K[i]; }
        }
        const int any_local = __syncthreads_or(notdone);
        if (tid == 0) S.nd[step & 1] = any_local;
        cl.sync();  // buffer b^1 and the flags complete everywhere; nobody reads b any more
        b ^= 1;
        int f = tid < kRedCl ? rem[tid]->nd[step & 1] : 0;
        const int any = __syncthreads_or(f);
        if (rank == 0 && tid == 0) ctl[step] = 1;
        if (!any) break;
    }
#pragma unroll
    for (int k = 0; k < NPT; k++) {
        const int t = tid + k * RT;
        if (t >= nmine) continue;
        const int idx = base + t;
        a.end2[idx] = S.q[b][t];   // markers (paths); cycles keep list positions >= 0
        a.dist2[idx] = make_int2(S.r[b][0][t], S.r[b][1][t]);
        a.kraw[idx] = make_ulonglong2(S.k[b][0][t], S.k[b][1][t]);
        a.dk2[idx] = make_int2(S.d[b][0][t], S.d[b][1][t]);
    }
    cl.sync();  // the last step's flag reads are done before any CTA leaves
}

constexpr int32_t kLocDone = INT_MIN;

// the expand pass needs only the tile's slots and weights
struct TileSmemE {
    int2 nb[LB];
    float2 w[LB];
    int32_t b0, tend;
};  // loc marker: the tile pass wrote the final results

// Tile pass: full-window scan; local cycles finished here; per-vertex local results and
// the reduced records of boundary vertices.
__global__ void __launch_bounds__(LT, LF_F1MINB) k_lf_full1(ForestArgs a) {
    LF_TL(g_tl_forest, 0);
    pdl_wait();  // k_ctl_zero, and through it the factor
    extern __shared__ __align__(16) unsigned char smem_raw[];
    TileSmemF& s = *reinterpret_cast<TileSmemF*>(smem_raw);
    const int32_t b0 = (int32_t)(a.lo + (int64_t)blockIdx.x * LB);
    LF_PHASE_INIT;
    load_tile_w(a.pi2, a.pi2_w, s, b0, a.hi);
    const Tile T{b0, (int32_t)((int64_t)b0 + LB < a.hi ? (int64_t)b0 + LB : a.hi)};
    int2 orig[VPT];
    Claim cl_[VPT];  // boundary-list slots, claimed now: the atomic's round trip overlaps the ranking
#pragma unroll
    for (int k = 0; k < VPT; k++) {
        orig[k] = s.nb[threadIdx.x + k * LT];
        const int32_t g = b0 + (int)threadIdx.x + k * LT;
        const bool r0 = orig[k].x >= 0 && !is_local(orig[k].x, T);
        const bool r1 = orig[k].y >= 0 && !is_local(orig[k].y, T);
        cl_[k] = claim_issue(&a.ctl[kCtlCnt1], g < a.hi && (r0 || r1));  // positions in phase 7
    }
    ulonglong2 ek[VPT];
    slot_keys(a, s, b0, ek);
    {   // the input must be a symmetric [0,2]-factor in canonical form (include/lf.h): a tile
        // that is not stops here and flags it, and the later kernels leave (no walk can fault)
        bool bad = false;
#pragma unroll
        for (int k = 0; k < VPT; k++) {
            const int u = threadIdx.x + k * LT;
            const int32_t g = b0 + u;
            if (g >= a.hi) continue;
            const int2 nb = s.nb[u];
            bad |= nb.x < -1 || nb.y < -1 || (int64_t)nb.x >= a.N || (int64_t)nb.y >= a.N || nb.x == g ||
                   nb.y == g || (nb.x < 0 && nb.y >= 0) || (nb.x >= 0 && nb.x == nb.y);
            if (bad) continue;
#pragma unroll
            for (int i = 0; i < 2; i++) {
                const int32_t x = i ? nb.y : nb.x;
                if (x < 0) continue;
                const int2 px = is_local(x, T) ? s.nb[x - b0] : (is_foreign(x, a) ? ghost_slots(a, x) : a.pi2[x]);
                bad |= px.x != g && px.y != g;
            }
        }
        if (__syncthreads_or(bad)) {
            if (threadIdx.x == 0) atomicOr(&a.ctl[kCtlBad], 1);
            return;
        }
    }
    LF_PHASE(a.ctl, 6);
    VRes o[VPT];
    tile_rank_full(s, b0, ek, o, a.ctl + kCtlStat);
#ifdef LF_PHASE_TIMING
    ph_t = clock64();
#endif
    int ncyc = 0;
#pragma unroll
    for (int k = 0; k < VPT; k++) {
        const int u = threadIdx.x + k * LT;
        const int32_t g = b0 + u;
        const int2 nb = orig[k];
        const bool r0 = nb.x >= 0 && !is_local(nb.x, T);
        const bool r1 = nb.y >= 0 && !is_local(nb.y, T);
        const bool boundary = g < a.hi && (r0 || r1);
        const int idx = claim_pos(cl_[k]);  // warp-uniform (shuffle)
        if (g < a.hi) {
            if (o[k].cyc) {
                const CycOut c = cycle_finish(g, nb, ek[k], o[k].Ks, o[k].C);
                a.path_id[g] = c.l;
                a.pos[g] = c.pos;
                a.len[g] = c.len;
                a.forest[g] = c.f;
                a.pdir[g] = c.pdir;
                ncyc += c.ncyc;
                a.loc2[g] = make_int2(kLocDone, 0);
            } else {
                const uint32_t tt = (uint32_t)(uint16_t)o[k].T.x | ((uint32_t)(uint16_t)o[k].T.y << 16);
                const uint32_t rr = (uint32_t)(uint16_t)o[k].R.x | ((uint32_t)(uint16_t)o[k].R.y << 16);
                a.loc2[g] = make_int2((int)tt, (int)rr);
            }
        }
        if (boundary) {
            a.list1[idx] = g;
            int2 q, rl, dk;
            ulonglong2 kk;
#pragma unroll
            for (int i = 0; i < 2; i++) {
                const int32_t x = i ? nb.y : nb.x;
                int32_t qi, ri, di;
                uint64_t ki;
                if (x < 0) { qi = -(g + 1); ri = 0; ki = KEY_INF; di = 0; }
                else if (!is_local(x, T)) { qi = x; ri = 1; ki = i ? ek[k].y : ek[k].x; di = g < x ? 1 : 0; }
                else {
                    const int t = i ? o[k].T.y : o[k].T.x;
                    const int2 nbt = s.nb[t];
                    const int32_t xo = outward_slot(nbt, T) ? nbt.y : nbt.x;
                    const int32_t tg = b0 + t;
                    qi = xo < 0 ? -(tg + 1) : tg;
                    ri = i ? o[k].R.y : o[k].R.x;
                    ki = i ? o[k].Kn.y : o[k].Kn.x;
                    di = i ? o[k].Dn.y : o[k].Dn.x;
                }
                if (i) { q.y = qi; rl.y = ri; kk.y = ki; dk.y = di; }
                else { q.x = qi; rl.x = ri; kk.x = ki; dk.x = di; }
            }
            a.bidx1[g] = idx;
            a.cq[idx] = q;
            a.cq_r[idx] = rl;
            a.cq_k[idx] = kk;
            a.cq_dk[idx] = dk;
        }
    }
#pragma unroll
    for (int o2 = 16; o2; o2 >>= 1) ncyc += __shfl_xor_sync(0xffffffffu, ncyc, o2);
    if ((threadIdx.x & 31) == 0 && ncyc) atomicAdd(&a.ctl[kCtlNcyc], ncyc);
    LF_PHASE(a.ctl, 7);
}
constexpr size_t kFull1Smem = sizeof(TileSmemF);

// one synchronous step over list positions t0, t0+stride, ... (grid path)
__device__ __forceinline__ int red_full_step(const ForestArgs& a, int cnt, int step, int t0, int stride) {
    const int2* __restrict__ qs = a.rq1[step & 1];
    int2* __restrict__ qd = a.rq1[(step & 1) ^ 1];
    const ulonglong2* __restrict__ ks = a.rk1[step & 1];
    ulonglong2* __restrict__ kd = a.rk1[(step & 1) ^ 1];
    const int2* __restrict__ rs = a.rr2[step & 1];
    int2* __restrict__ rd = a.rr2[(step & 1) ^ 1];
    const int2* __restrict__ ds = a.rdk[step & 1];
    int2* __restrict__ dd = a.rdk[(step & 1) ^ 1];
    int notdone = 0;
    for (int me = t0; me < cnt; me += stride) {
        const int2 q = __ldcg(qs + me);
        int2 r = __ldcg(rs + me), d = __ldcg(ds + me);
        ulonglong2 k = __ldcg(ks + me);
        if (q.x < 0 && q.y < 0) {  // final: keep both buffers equal
            qd[me] = q; kd[me] = k; rd[me] = r; dd[me] = d;
            continue;
        }
        int2 nq = q;
#pragma unroll
        for (int i = 0; i < 2; i++) {
            const int w = i ? q.y : q.x;
            if (w < 0) continue;
            const int2 qw = __ldcg(qs + w), rw = __ldcg(rs + w), dw = __ldcg(ds + w);
            const ulonglong2 kw = __ldcg(ks + w);
            int32_t R = i ? r.y : r.x, D = i ? d.y : d.x;
            uint64_t K = i ? k.y : k.x;
            int j = -1;
            if (qw.x != me) j = 0;
            else if (qw.y != me) j = 1;
            int32_t tgt = w;
            if (j >= 0) {
                tgt = j ? qw.y : qw.x;
                win_append(R, K, D, j ? rw.y : rw.x, j ? kw.y : kw.x, j ? dw.y : dw.x);
            } else {
                if (kw.x < K) { K = kw.x; D = 2 * R + dw.x; }
                if (kw.y < K) { K = kw.y; D = 2 * R + dw.y; }
            }
            if (i) { nq.y = tgt; r.y = R; d.y = D; k.y = K; } else { nq.x = tgt; r.x = R; d.x = D; k.x = K; }
        }
        qd[me] = nq; kd[me] = k; rd[me] = r; dd[me] = d;
        const bool path_done = nq.x < 0 && nq.y < 0;
        const bool cyc_done = nq.x >= 0 && nq.y >= 0 && k.x == k.y;
        notdone += (path_done || cyc_done) ? 0 : 1;
    }
    return notdone;
}

// Grid barrier of k_red_full (monotone arrival counter; `gen` counts the barriers passed).
// k_red_full is a cooperative cluster launch (launch_red_full): the runtime guarantees
// that all its CTAs are co-resident, or fails the launch.
__device__ __forceinline__ void red_grid_sync(int* ctr, int& gen) {
    __syncthreads();
    gen++;
    if (threadIdx.x == 0) {
        __threadfence();
        atomicAdd(ctr, 1);
        const int target = gen * (int)gridDim.x;
        while (true) {
            int v;
            asm volatile("ld.acquire.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(ctr) : "memory");
            if (v >= target) break;
            __nanosleep(32);
        }
    }
    __syncthreads();
}

__global__ void __launch_bounds__(RT) k_red_full(ForestArgs a) {
    LF_TL(g_tl_forest, 1);
    __shared__ int sh[32];
    extern __shared__ __align__(16) unsigned char red_smem[];
    pdl_wait();  // the tile pass's records
    if (*(volatile int*)&a.ctl[kCtlBad]) return;  // a malformed factor (k_lf_full1): uniform
    const int cnt = *(volatile int*)&a.ctl[kCtlCnt1];
    int* ctl = a.ctl + kCtlRed1;
    if (cnt <= kRedCl * kRedClNodes) {
        pdl_trigger();  // the expand kernel's tile-only prologue overlaps this scan
        if (blockIdx.x < kRedCl) red_full_cluster(a, cnt, ctl, *reinterpret_cast<RedSmemC*>(red_smem));
        return;
    }
    int* bar = a.ctl + kCtlGridBar;
    int gen = 0;
    const int stride = gridDim.x * blockDim.x;
    const int t0 = blockIdx.x * blockDim.x + threadIdx.x;
    for (int me = t0; me < cnt; me += stride) {
        const int2 q = to_pos(a, a.cq[me]);
        a.rq1[0][me] = q;
        a.rk1[0][me] = a.cq_k[me];
        a.rr2[0][me] = a.cq_r[me];
        a.rdk[0][me] = a.cq_dk[me];
    }
    red_grid_sync(bar, gen);
    int step = 0;
    for (; step < a.max_steps; step++) {
        int notdone = red_full_step(a, cnt, step, t0, stride);
#pragma unroll
        for (int o = 16; o; o >>= 1) notdone += __shfl_xor_sync(0xffffffffu, notdone, o);
        if ((threadIdx.x & 31) == 0) sh[threadIdx.x >> 5] = notdone;
        __syncthreads();
        if (threadIdx.x == 0) {
            int tot = 0;
            for (int w = 0; w < (int)(blockDim.x >> 5); w++) tot += sh[w];
            if (tot) atomicAdd(&ctl[step], tot);
        }
        red_grid_sync(bar, gen);
        if (__ldcg(&ctl[step]) == 0) { step++; break; }
    }
    pdl_trigger();
    const int fb = step & 1;
    for (int me = t0; me < cnt; me += stride) {
        a.end2[me] = __ldcg(&a.rq1[fb][me]);
        a.dist2[me] = __ldcg(&a.rr2[fb][me]);
        a.kraw[me] = __ldcg(&a.rk1[fb][me]);
        a.dk2[me] = __ldcg(&a.rdk[fb][me]);
    }
}

// Expand pass: every vertex not finished by the tile pass combines its local result with
// the reduced results of its terminals; then the tile's path lengths are scanned into
// tile-local offsets and a tile total.  Everything that depends only on the tile pass
// (tile slots, slot keys, local results, terminal list positions, segment records -- all
// complete before the reduced scan even started) is done BEFORE pdl_wait, overlapping the
// reduced scan; vertices whose two terminals are path ends finish there too.

struct ExpState {       // a vertex waiting for reduced results
    int bi0, bi1;       // list positions of its terminals (-1: a path end)
    int so;             // bit i: outward slot of terminal i
    int R0, R1;
    uint64_t kseg;      // t0's inward segment window: weakest key, DK
    int dseg;
};

// threads and resident CTAs of the expand pass (measured on C2: 512 x 3 beats 256 x 4,
// 256 x 3 and 128 x 8 -- fewer threads per tile serialise each thread's vertices)
#ifndef LF_ET
#define LF_ET 512
#endif
#ifndef LF_EMINB
#define LF_EMINB 3
#endif
constexpr int ET = LF_ET;
constexpr int EV = LB / ET;

__global__ void __launch_bounds__(ET, LF_EMINB) k_lf_full2(ForestArgs a) {
    LF_TL(g_tl_forest, 2);
    extern __shared__ __align__(16) unsigned char smem_raw[];
    TileSmemE& s = *reinterpret_cast<TileSmemE*>(smem_raw);
    __shared__ int sh[32 * EV];  // the final vector scan (read once: no reuse barrier)
    // the tile pass completed before the reduced scan triggered this launch: its flag is final
    if (*(volatile int*)&a.ctl[kCtlBad]) return;
    const int32_t b0 = (int32_t)(a.lo + (int64_t)blockIdx.x * LB);
    int2 lcs[EV];  // the tile pass's local results, in flight with the tile's slots
#pragma unroll
    for (int k = 0; k < EV; k++) {
        const int64_t g = (int64_t)b0 + threadIdx.x + k * ET;
        lcs[k] = g < a.hi ? __ldg(a.loc2 + g) : make_int2(0, 0);
    }
    load_tile_w<TileSmemE, ET>(a.pi2, a.pi2_w, s, b0, a.hi);
    const Tile T{b0, (int32_t)((int64_t)b0 + LB < a.hi ? (int64_t)b0 + LB : a.hi)};
    ulonglong2 ek[EV];
    slot_keys<TileSmemE, ET>(a, s, b0, ek);
    int lens[EV];
    bool wait[EV];
    ExpState st[EV];
    int ncyc = 0;
#pragma unroll
    for (int k = 0; k < EV; k++) {
        const int u = threadIdx.x + k * ET;
        const int32_t g = b0 + u;
        lens[k] = 0;
        wait[k] = false;
        if (g >= a.hi) continue;
        const int2 lc = lcs[k];
        if (lc.x == kLocDone) { lens[k] = a.len[g]; continue; }
        const int Tl[2] = {(int)(lc.x & 0xffff), (int)((uint32_t)lc.x >> 16)};
        st[k].R0 = (int)(lc.y & 0xffff);
        st[k].R1 = (int)((uint32_t)lc.y >> 16);
        st[k].so = 0;
        int bi[2];
#pragma unroll
        for (int i = 0; i < 2; i++) {
            const int t = Tl[i];
            const int2 nbt = s.nb[t];
            const int so = (t == u) ? i : outward_slot(nbt, T);
            st[k].so |= so << i;
            bi[i] = (so ? nbt.y : nbt.x) < 0 ? -1 : a.bidx1[b0 + t];
        }
        st[k].bi0 = bi[0];
        st[k].bi1 = bi[1];
        if (bi[0] < 0 && bi[1] < 0) {  // a path inside the tile: both terminals are its ends
            const int2 nb = s.nb[u];
            const int32_t E0 = b0 + Tl[0], E1 = b0 + Tl[1];
            const int dir = E0 <= E1 ? 0 : 1;
            const int32_t l = dir ? E1 : E0;
            a.path_id[g] = l;
            a.pos[g] = (dir ? st[k].R1 : st[k].R0) + 1;
            a.pdir[g] = nbr_slots(nb, dir, -1);
            a.forest[g] = nb;
            lens[k] = (l == g) ? st[k].R0 + st[k].R1 + 1 : 0;
            continue;
        }
        wait[k] = true;
        st[k].kseg = KEY_INF;
        st[k].dseg = 0;
        if (bi[0] >= 0) {  // t0's inward window spans this vertex's segment
            const ulonglong2 ki = a.cq_k[bi[0]];
            const int2 di = a.cq_dk[bi[0]];
            st[k].kseg = (st[k].so & 1) ? ki.x : ki.y;
            st[k].dseg = (st[k].so & 1) ? di.x : di.y;
        }
    }
    pdl_wait();  // the reduced scan's results
#pragma unroll
    for (int k = 0; k < EV; k++) {
        if (!wait[k]) continue;
        const int u = threadIdx.x + k * ET;
        const int32_t g = b0 + u;
        const int2 nb = s.nb[u];
        const int Rl[2] = {st[k].R0, st[k].R1};
        const int bi[2] = {st[k].bi0, st[k].bi1};
        int32_t E[2], D[2];
        int dko[2] = {0, 0};
        uint64_t ks = KEY_INF;
        bool cyc = false;
#pragma unroll
        for (int i = 0; i < 2; i++) {
            const int so = (st[k].so >> i) & 1;
            if (bi[i] < 0) {  // a path end (the vertex reached it inside the tile)
                const int t = i ? (int)((uint32_t)lcs[k].x >> 16) : (int)(lcs[k].x & 0xffff);
                E[i] = b0 + t;
                D[i] = Rl[i];
                continue;
            }
            const int2 e = a.end2[bi[i]];
            const int32_t fq = so ? e.y : e.x;
            if (fq >= 0) {
                cyc = true;
                const int2 dk = a.dk2[bi[i]];
                dko[i] = so ? dk.y : dk.x;
                if (i == 0) { const ulonglong2 kf = a.kraw[bi[0]]; ks = so ? kf.y : kf.x; }
                continue;
            }
            const int2 dd = a.dist2[bi[i]];
            E[i] = -(fq + 1);
            D[i] = Rl[i] + (so ? dd.y : dd.x);
        }
        if (!cyc) {
            const int dir = E[0] <= E[1] ? 0 : 1;
            const int32_t l = E[dir];
            a.path_id[g] = l;
            a.pos[g] = D[dir] + 1;
            a.pdir[g] = nbr_slots(nb, dir, -1);
            a.forest[g] = nb;
            lens[k] = (l == g) ? D[0] + D[1] + 1 : 0;
            continue;
        }
        // on a cycle through other tiles (both terminals continue): is its weakest edge
        // inside this vertex's segment?  (reading c9)
        int2 c;
        if (st[k].kseg == ks) {
            const int delta = st[k].dseg >> 1, bt = st[k].dseg & 1;
            if (Rl[0] >= delta + 1) c = make_int2(2 * (Rl[0] - delta - 1) + (bt ^ 1), 2 * Rl[1] + dko[1]);
            else c = make_int2(2 * Rl[0] + dko[0], 2 * (delta - Rl[0]) + bt);
        } else {
            c = make_int2(2 * Rl[0] + dko[0], 2 * Rl[1] + dko[1]);
        }
        const CycOut co = cycle_finish(g, nb, ek[k], ks, c);
        a.path_id[g] = co.l;
        a.pos[g] = co.pos;
        a.pdir[g] = co.pdir;
        a.forest[g] = co.f;
        lens[k] = co.len;
        ncyc += co.ncyc;
    }
    // tile-local exclusive prefix of the path lengths in id order (thread t owns
    // u = t + k ET): the EV scans run together in one block scan (one set of barriers)
    {
        int e[EV], tot[EV];
        block_scan_sum_excl_v<EV>(lens, sh, e, tot);
        int carry = 0;
#pragma unroll
        for (int k = 0; k < EV; k++) {
            const int32_t gk = b0 + (int)threadIdx.x + k * ET;
            if (gk < a.hi && lens[k]) a.off[gk] = carry + e[k];
            carry += tot[k];
        }
        if (threadIdx.x == 0) a.tsum[blockIdx.x] = carry;
    }
#pragma unroll
    for (int o2 = 16; o2; o2 >>= 1) ncyc += __shfl_xor_sync(0xffffffffu, ncyc, o2);
    if ((threadIdx.x & 31) == 0 && ncyc) atomicAdd(&a.ctl[kCtlNcyc], ncyc);
}

// Exclusive prefix of the tile totals (one CTA; the permutation kernel then finds the
// new index r = tsum[tile of l] + off[l] + p - 1, reading c14), and the cycle count.
constexpr int kPrefT = 1024, kPrefPT = 8;

__global__ void __launch_bounds__(kPrefT) k_tile_prefix(int32_t* tsum, int tiles, const int* ctl,
                                                        unsigned long long* n_cycles, int grs_mode) {
    LF_TL(g_tl_forest, 3);
    __shared__ int sh[32];
    pdl_wait();
    pdl_trigger();
    if (n_cycles && threadIdx.x == 0) *n_cycles = (unsigned long long)__ldcg(ctl + kCtlNcyc);
    if (__ldcg(ctl + kCtlBad) && !grs_mode) return;  // a malformed factor: see k_lf_full1
    int carry = 0;
    for (int base = 0; base < tiles; base += kPrefT * kPrefPT) {
        int x[kPrefPT], sum = 0;
#pragma unroll
        for (int j = 0; j < kPrefPT; j++) {
            const int i = base + threadIdx.x * kPrefPT + j;
            x[j] = i < tiles ? __ldcg(tsum + i) : 0;
            sum += x[j];
        }
        int total = 0;
        int run = carry + block_scan_sum_excl(sum, sh, &total);
#pragma unroll
        for (int j = 0; j < kPrefPT; j++) {
            const int i = base + threadIdx.x * kPrefPT + j;
            if (i < tiles) tsum[i] = run;
            run += x[j];
        }
        carry += total;
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

size_t forest_ws_carve(Carve& c, int64_t N, ForestWs* w, bool with_grs) {
    ForestWs t;
    const size_t n = (size_t)(N > 0 ? N : 1);
    for (int i = 0; i < 2; i++) {
        t.rq1[i] = c.take<int2>(n);
        t.rk1[i] = c.take<ulonglong2>(n);
        t.rq2[i] = c.take<int2>(n);
        t.rr2[i] = c.take<int2>(n);
    }
    t.cyc_k = c.take<uint64_t>(n);
    t.loc1 = c.take<short2>(n);
    t.kst = c.take<uint64_t>(n);
    t.loc2 = c.take<int2>(n);
    t.end2 = c.take<int2>(n);
    t.dist2 = c.take<int2>(n);
    t.list1 = c.take<int32_t>(n);
    t.list2 = c.take<int32_t>(n);
    t.len = c.take<int32_t>(n);
    t.off = c.take<int32_t>(n);
    t.ctl = c.take<int>(kCtlInts);
    t.kraw = c.take<ulonglong2>(n);
    t.ekb = c.take<ulonglong2>(n);
    t.cq = c.take<int2>(n);
    t.bidx1 = c.take<int32_t>(n);
    t.bidx2 = c.take<int32_t>(n);
    t.pdir = c.take<uint8_t>(n);
    t.tsum = c.take<int32_t>(n / 256 + 2);  // per offset chunk (8192) or tile (>= 256)
    t.cq_k = c.take<ulonglong2>(n);
    t.cq_r = c.take<int2>(n);
    t.cq_dk = c.take<int2>(n);
    t.dk2 = c.take<int2>(n);
    t.rdk[0] = c.take<int2>(n);
    t.rdk[1] = c.take<int2>(n);
    const size_t ng = with_grs ? n : 1;  // the partitioned path runs the tile scans only
    t.grs_rec = c.take<int4>(ng);  // one 16-byte record per vertex
    t.grs_meet = c.take<int4>(2 * ng);
    t.grs_meetk = c.take<uint64_t>(2 * ng);
    t.grs_mstop = c.take<int4>(2 * ng);
    t.grs_bits = c.take<uint32_t>(ng / 32 + 1);
    t.grs_cyc = c.take<int4>(ng / 3 + 1 + kCycStripes);  // kCycStripes * grs_cyc_cap(N)
    t.grs_cyck = c.take<uint64_t>(ng / 3 + 1 + kCycStripes);
    t.grs_desc = c.take<int4>(2 * (ng + ng / 3 + 1 + kCycStripes));  // splitters + the cycle index space
    t.scan_tmp_bytes = scan_temp_bytes(N);
    t.scan_tmp = c.take<char>(t.scan_tmp_bytes);
    if (w) *w = t;
    return c.off;
}

static int max_steps_for(int64_t N) {
    int s = 0;
    while (s < 40 && ((int64_t)1 << s) < N) s++;
    return s + 3;  // ceil(log2 N) + margin for cycle detection
}

template <class K>
static int coop_launch(K kernel, int block, ForestArgs& a, cudaStream_t s, size_t smem = 0) {
    const int grid = persistent_grid((const void*)kernel, block, smem);
    void* args[] = {&a};
    LF_CUDA(cudaLaunchCooperativeKernel((const void*)kernel, grid, block, args, smem, s));
    return LF_OK;
}

// zero the 256-int control block once the stream predecessor has completed (its CTAs
// may still be running when this one is scheduled: nothing is written before pdl_wait,
// since the caller may hand the same workspace to consecutive calls)
__global__ void k_ctl_zero(int* ctl) {
    pdl_trigger();
    pdl_wait();
    for (int i = threadIdx.x; i < kCtlInts; i += blockDim.x) ctl[i] = 0;
}

static int forest_prepare() {
    static bool attr_done = false;
    if (attr_done) return LF_OK;
    const int smem = (int)sizeof(TileSmem);
    LF_CUDA(cudaFuncSetAttribute((const void*)k_lf_local1, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
    LF_CUDA(cudaFuncSetAttribute((const void*)k_lf_local2, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 (int)kTileSmemNoKeys));
    LF_CUDA(cudaFuncSetAttribute((const void*)k_lf_local3, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 (int)kTileSmemNoKeys));
    LF_CUDA(cudaFuncSetAttribute((const void*)k_red_scan<true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 (int)sizeof(RedSmem)));
    LF_CUDA(cudaFuncSetAttribute((const void*)k_red_scan<false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 (int)sizeof(RedSmem)));
    LF_CUDA(cudaFuncSetAttribute((const void*)k_lf_full1, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 (int)kFull1Smem));
    LF_CUDA(cudaFuncSetAttribute((const void*)k_red_full, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 (int)sizeof(RedSmemC)));
    LF_CUDA(cudaFuncSetAttribute((const void*)k_lf_full2, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 (int)sizeof(TileSmemE)));
    attr_done = true;
    return LF_OK;
}

// k_red_full: clusters of kRedCl CTAs (the small path runs on the first cluster), as
// many clusters as can be resident at once (the grid path's barrier needs them all)
static cudaError_t launch_red_full(const ForestArgs& a, cudaStream_t s) {
    static int nclusters = 0;
    cudaLaunchConfig_t cfg = {};
    cfg.blockDim = dim3(RT);
    cfg.dynamicSmemBytes = sizeof(RedSmemC);
    cfg.stream = s;
    cudaLaunchAttribute at[3];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = kRedCl;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    if (nclusters == 0) {
        cudaError_t e = cudaFuncSetAttribute((const void*)k_red_full, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
        if (e != cudaSuccess) return e;
        cfg.gridDim = dim3(kRedCl);
        cfg.numAttrs = 1;
        int n = 0;
        e = cudaOccupancyMaxActiveClusters(&n, (const void*)k_red_full, &cfg);
        if (e != cudaSuccess) return e;
        if (n < 1) return cudaErrorLaunchOutOfResources;
        nclusters = n < sm_count() / kRedCl ? n : sm_count() / kRedCl;
        if (nclusters < 1) nclusters = 1;
    }
    cfg.gridDim = dim3(kRedCl * nclusters);
    // the grid path's barrier needs every CTA resident: a cooperative launch makes the
    // runtime guarantee it (or fail the launch) instead of a scheduling argument
    at[1].id = cudaLaunchAttributeCooperative;
    at[1].val.cooperative = 1;
    at[2].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[2].val.programmaticStreamSerializationAllowed = 1;
    cfg.numAttrs = pdl_enabled() ? 3 : 2;
    return cudaLaunchKernelEx(&cfg, k_red_full, a);
}

// ===========================================================================
// Global ruling set (GRS) -- the single-pass window scan without the tile level, for
// graphs whose paths leave every tile (C5's 27-point snakes: 96% of the vertices are tile
// boundary vertices, so the reduced graph is nearly the whole graph and pointer jumping
// over it costs ~20 full passes).  DESIGN.md §5.5:
//   1. k_grs_pack / k_grs_list: a 16-byte record per vertex (slots, |w|), splitters = path
//      ends and a hashed 1/256 of the rest, the visit bitmap, the splitter list in id order.
//   2. k_grs_walk / k_grs_meet: the two walks of every segment fold its full window and
//      meet in the middle; each claims the vertices it visits with (walk, distance, slot).
//   3. k_red_full on the splitter list (the reduced scan of the tile path, unchanged).
//   4. k_grs_len, k_grs_cyccand / k_grs_cycfind (cycles without a splitter), k_grs_lenscan
//      + k_tile_prefix: path lengths at the path-ID vertices and their exclusive prefix.
//   5. k_grs_desc: one descriptor per walk; k_grs_emit: every output of a vertex from its
//      claim and its walk's descriptor in one coalesced pass; k_grs_split.
// Every output equals the tile path's (and the oracle's) bit for bit: the windows fold the
// same edge keys in the same walk order, and the readings c9/c11/c12/c14/c15 are applied by
// the same cycle_finish / path rules as k_lf_full2 / k_perm_tri.
// ===========================================================================
#ifndef LF_GRS_SHIFT
#define LF_GRS_SHIFT 24  // hashed splitter density 2^-(32 - 24) = 1/256 (C5: 1/16..1/256 measured, sparse wins)
#endif
constexpr int kGrsShift = LF_GRS_SHIFT;
// splitter-free cycles recorded by k_grs_cycfind: kCycStripes counters (a single one was
// the contended atomic that dominated the kernel, ~840 k cycles on C5), cycle c = stripe *
// grs_cyc_cap(N) + its rank in the stripe
__host__ __device__ __forceinline__ int64_t grs_cyc_cap(int64_t N) { return (N / 3 + 1) / kCycStripes + 1; }
__device__ __forceinline__ bool grs_cyc_valid(const ForestArgs& a, int64_t c) {
    const int64_t cap = grs_cyc_cap(a.N), s = c / cap;
    return c >= 0 && s < kCycStripes && c - s * cap < (int64_t)__ldcg(&a.ctl[kCtlCycS + kCtlCycStride * s]);
}

__device__ __forceinline__ bool grs_hashed(const ForestArgs& a, int32_t v) {
    return (((uint32_t)v * 0x9E3779B1u) >> a.grs_shift) == 0u;
}
__device__ __forceinline__ bool grs_splitter(const ForestArgs& a, int32_t v, int2 nb) {
    return nb.x < 0 || nb.y < 0 || grs_hashed(a, v);
}
// The 16-byte record of vertex v: (slot 0, slot 1, |w| slot 0, |w| slot 1) -- one random
// visit per walk step.  The walk that claims a non-splitter v (the visit bitmap) overwrites
// the |w| half it has just read with (walk t, 2d + fslot): v lies at distance d from the
// walk's splitter, fslot its slot pointing away from it.  k_grs_emit then derives every
// output of v in ONE coalesced pass over the vertices; the splitter-free
// cycles of k_grs_cycfind claim theirs as walks t = 2 cnt + c.  Splitters keep their record.
__device__ __forceinline__ void grs_load(const ForestArgs& a, int32_t v, int2& nb, float2& w) {
    const int4 r = __ldcg(a.grs_rec + (int64_t)v);
    nb = make_int2(r.x, r.y);
    w = make_float2(__int_as_float(r.z), __int_as_float(r.w));
}
__device__ __forceinline__ void grs_claim(const ForestArgs& a, int32_t v, int t, int32_t d, int fs) {
    reinterpret_cast<int2*>(a.grs_rec + (int64_t)v)[1] = make_int2(t, (int32_t)(((uint32_t)d << 1) | (uint32_t)fs));
}

// 8 vertices per thread per iteration: one list atomic per 2048 vertices (the splitter
// counter is a single address; a warp-level atomic per 32 vertices serialised ~4 M times on C5)
constexpr int kPackV = 8;
__global__ void __launch_bounds__(256) k_grs_pack(ForestArgs a) {
    LF_TL(g_tl_forest, 5);
    __shared__ int wsum[8];
    pdl_wait();
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    const int64_t chunk = (int64_t)blockDim.x * kPackV;  // 2048 (k_grs_list's chunk)
    for (int64_t c0 = (int64_t)blockIdx.x * chunk; c0 < a.N; c0 += (int64_t)gridDim.x * chunk) {
        unsigned m[kPackV];
        int mine = 0;
#pragma unroll
        for (int k = 0; k < kPackV; k++) {
            const int64_t v = c0 + threadIdx.x + (int64_t)k * blockDim.x;  // warp-uniform in/out
            const bool in = v < a.N;
            int2 nb = make_int2(0, 0);
            float2 w = make_float2(0.f, 0.f);
            if (in) {
                nb = __ldg(a.pi2 + v);
                w = __ldg(a.pi2_w + v);
            }
            const bool spl = in && grs_splitter(a, (int32_t)v, nb);
            m[k] = __ballot_sync(0xffffffffu, spl);
            mine += __popc(m[k]);
            if (in) {
                a.len[v] = 0;
                a.grs_rec[v] = make_int4(nb.x, nb.y, __float_as_int(w.x), __float_as_int(w.y));
                if (lane == 0) a.grs_bits[v >> 5] = m[k];  // v - lane is a multiple of 32
            }
        }
        if (lane == 0) wsum[wid] = mine;
        __syncthreads();
        if (threadIdx.x == 0) {  // the chunk's splitter count; k_tile_prefix + k_grs_list list them
            int t = 0;
            for (int q = 0; q < (int)(blockDim.x >> 5); q++) t += wsum[q];
            a.tsum[c0 / chunk] = t;
        }
        __syncthreads();  // wsum reused
    }
}

// The splitter list in id order: warp per 2048-vertex chunk (its 64 bitmap words as the pack
// left them: splitters only), at the chunk's exclusive prefix.  In id order, the walks that
// k_grs_walk hands out one after the other start at neighbouring splitters: the band of the
// id space they cover is what L2 holds (an atomic list order jittered over ~9 planes).
__global__ void __launch_bounds__(256) k_grs_list(ForestArgs a) {
    LF_TL(g_tl_forest, 14);
    pdl_wait();
    const int lane = threadIdx.x & 31;
    const int64_t chunks = (a.N + 2047) / 2048, words = (a.N + 31) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t c = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; c < chunks; c += nw) {
        const int base = __ldcg(a.tsum + c);
        const int64_t w0 = c * 64 + 2 * lane;
        uint32_t m0 = w0 < words ? __ldcg(a.grs_bits + w0) : 0u;
        uint32_t m1 = w0 + 1 < words ? __ldcg(a.grs_bits + w0 + 1) : 0u;
        const int cnt = __popc(m0) + __popc(m1);
        int incl = cnt;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int y = __shfl_up_sync(0xffffffffu, incl, o);
            if (lane >= o) incl += y;
        }
        int pos = base + incl - cnt;
        while (m0) {
            const int32_t v = (int32_t)(w0 * 32 + __ffs(m0) - 1);
            m0 &= m0 - 1u;
            a.list1[pos] = v;
            a.bidx1[v] = pos++;
        }
        while (m1) {
            const int32_t v = (int32_t)((w0 + 1) * 32 + __ffs(m1) - 1);
            m1 &= m1 - 1u;
            a.list1[pos] = v;
            a.bidx1[v] = pos++;
        }
        if (c == chunks - 1 && lane == 31) a.ctl[kCtlCnt1] = base + incl;
    }
}

// One (splitter, direction) per walk: the segment's full window and the next splitter.
// The two walks of a segment start at its two ends and meet in the middle: each claims
// every vertex it steps on in the visit bitmap (atomicOr) and stops at the first one its
// partner claimed, so every interior vertex is read by ONE walk (a random 32-byte visit
// costs ~128 bytes of DRAM traffic: this halves the kernel's).  A walk that stops at a
// splitter is final; every walk also leaves its partial window (without the stop edge) at
// (last vertex, slot toward the stop), where k_grs_meet finds it: a walk that met its
// partner becomes  own window ⊕ stop edge ⊕ reverse(partner's window).
__device__ __forceinline__ void walk_leave(const ForestArgs& a, int t, int32_t last, int slot, int32_t R,
                                           uint64_t K, int32_t DK) {
    a.grs_meet[2 * (int64_t)last + slot] = make_int4(t, R, DK, 0);
    a.grs_meetk[2 * (int64_t)last + slot] = K;
}

#ifndef LF_WALK_PAIR
#define LF_WALK_PAIR 2
#endif
__global__ void __launch_bounds__(256) k_grs_walk(ForestArgs a) {
    LF_TL(g_tl_forest, 6);
    pdl_wait();
    const int cnt = __ldcg(&a.ctl[kCtlCnt1]);
    const int lane = threadIdx.x & 31;
    // dynamic schedule: a warp takes the next 32 walks when its last one has ended, so the
    // walks in flight start at consecutive splitters -- a band of the id space -- instead of
    // drifting apart with the walk lengths under a static grid stride (C5: 9.6 -> 8.4 ms).
    // Lanes leave a walk at different times and, under independent thread scheduling, the
    // ones that are done take their next walks together (__activemask) without waiting for
    // the rest of the warp.  (A full-warp grab of 32 walks after all lanes are done measured
    // 11.5 ms, 4 x 32 at a time 7.7 ms, this one 6.0 ms.)
    // LF_WALK_PAIR: a lane takes both walks of a splitter (t, t + 1) per grab -- half the
    // atomics on the schedule counter, whose single address bounded the walk (C5: 1 walk
    // per grab 6.0 ms, 2 walks 5.4 ms, 4 walks 5.6 ms)
    // kWalkCtrs counters (one 128-byte line each) hand out interleaved chunks of 2048 walks:
    // counter c's n-th walk is walk (n / 2048 * kWalkCtrs + c) * 2048 + n % 2048, so the
    // counters advance together and the walks in flight stay one band
    int* ctr = a.ctl + kCtlWalkC + kCtlCycStride * (int)(blockIdx.x % kWalkCtrs);
    const int cidx = (int)(blockIdx.x % kWalkCtrs);
    auto walk_of = [&](int u) -> int {
        const int64_t w = ((int64_t)(u >> 11) * kWalkCtrs + cidx) * 2048 + (u & 2047);
        return w < 2 * (int64_t)cnt ? (int)w : INT_MAX;
    };
    int b = 0;
    if (lane == 0) b = atomicAdd(ctr, 32 * LF_WALK_PAIR);
    int u = __shfl_sync(0xffffffffu, b, 0) + LF_WALK_PAIR * lane;
    int spare = LF_WALK_PAIR - 1;
    for (int t = walk_of(u); t < 2 * cnt;) {
        const int i = t >> 1, f = t & 1;
        const int32_t sv = __ldcg(a.list1 + i);
        int2 nbs;
        float2 ws;
        grs_load(a, sv, nbs, ws);
        const int32_t x = f ? nbs.y : nbs.x;
        int32_t tgt, R = 0, DK = 0;
        uint64_t K = KEY_INF;
        int4 stop = make_int4(-1, -1, 0, 0);
        if (x < 0) {
            tgt = -(sv + 1);  // a path end: marker
        } else {
            int32_t prev = sv, cur = x;
            int2 nbp = nbs;                  // slots of prev
            int sp = f;                      // prev's slot toward cur
            float wpc = f ? ws.y : ws.x;     // |w| of edge prev-cur
            while (true) {
                // the claim (visit bitmap) and the record load are independent: both are in
                // flight at once, and whether cur is a splitter follows from its id (hashed)
                // and its record (a path end) -- one memory round trip per step
                const bool hs = grs_hashed(a, cur);
                uint32_t old = ~0u;
                if (!hs) old = atomicOr(a.grs_bits + (cur >> 5), 1u << (cur & 31));
                int2 nbc;
                float2 wc;
                grs_load(a, cur, nbc, wc);
                const bool spl = hs || nbc.x < 0 || nbc.y < 0;  // a path end's bit was set by the pack
                if (!spl && ((old >> (cur & 31)) & 1u)) {  // the partner's: met (only its slots are used)
                    walk_leave(a, t, prev, sp, R, K, DK);
                    // the stop edge's key and cur's slot toward prev, for k_grs_meet (cur's
                    // slots are intact: a claim overwrites the |w| half only)
                    const uint64_t ks = edge_key(prev, cur, wpc, prev < cur ? nbp : nbc);
                    const uint32_t sn = nbc.x == prev ? 0u : 1u;
                    stop = make_int4(prev, (int32_t)((uint32_t)cur | (sn << 31)), (int32_t)(uint32_t)ks,
                                     (int32_t)(uint32_t)(ks >> 32));
                    tgt = cur;
                    break;
                }
                if (spl) walk_leave(a, t, prev, sp, R, K, DK);  // for the walk from that splitter
                const uint64_t k = edge_key(prev, cur, wpc, prev < cur ? nbp : nbc);
                if (k < K) { K = k; DK = 2 * R + (prev < cur ? 1 : 0); }
                R++;
                if (spl) { tgt = cur; break; }
                const int fs = nbc.x == prev ? 1 : 0;  // the slot away from prev
                grs_claim(a, cur, t, R, fs);           // cur's |w| half was read above
                const int32_t nxt = fs ? nbc.y : nbc.x;
                if (R > a.N || (uint32_t)nxt >= (uint32_t)a.N) {  // a malformed factor: end the segment
                    atomicOr(&a.ctl[kCtlBadGrs], 1);                // as if at a path end
                    tgt = -(sv + 1);
                    break;
                }
                wpc = fs ? wc.y : wc.x;
                nbp = nbc;
                sp = fs;
                prev = cur;
                cur = nxt;
            }
        }
        a.grs_mstop[t] = stop;
        int32_t* q = reinterpret_cast<int32_t*>(a.cq + i);
        int32_t* r = reinterpret_cast<int32_t*>(a.cq_r + i);
        int32_t* d = reinterpret_cast<int32_t*>(a.cq_dk + i);
        uint64_t* k = reinterpret_cast<uint64_t*>(a.cq_k + i);
        q[f] = tgt;
        r[f] = R;
        d[f] = DK;
        k[f] = K;
        if (spare > 0) {  // the other walk of the same grab
            spare--;
            t = walk_of(++u);
            continue;
        }
        const unsigned act = __activemask();
        const int ld = __ffs(act) - 1;
        int nb = 0;
        if (lane == ld) nb = atomicAdd(ctr, LF_WALK_PAIR * __popc(act));
        u = __shfl_sync(act, nb, ld) + LF_WALK_PAIR * __popc(act & ((1u << lane) - 1u));
        t = walk_of(u);
        spare = LF_WALK_PAIR - 1;
    }
}

// Walks that met their partner: own window ⊕ stop edge ⊕ reverse(partner's window); the
// segment's far splitter is the partner's start.
__global__ void __launch_bounds__(256) k_grs_meet(ForestArgs a) {
    LF_TL(g_tl_forest, 12);
    pdl_wait();
    const int cnt = __ldcg(&a.ctl[kCtlCnt1]);
    for (int t = blockIdx.x * blockDim.x + threadIdx.x; t < 2 * cnt; t += gridDim.x * blockDim.x) {
        const int4 st = __ldcg(a.grs_mstop + t);
        if (st.x < 0) continue;
        const int i = t >> 1, f = t & 1;
        // the walk left (last, nxt, nxt's slot toward last, the stop edge's key)
        const int32_t last = st.x, nxt = (int32_t)((uint32_t)st.y & 0x7FFFFFFFu);
        const int sn = (int)((uint32_t)st.y >> 31);
        const uint64_t kstop = (uint64_t)(uint32_t)st.z | ((uint64_t)(uint32_t)st.w << 32);
        const int4 pm = __ldcg(a.grs_meet + 2 * (int64_t)nxt + sn);
        const uint64_t pk = __ldcg(a.grs_meetk + 2 * (int64_t)nxt + sn);
        int32_t* q = reinterpret_cast<int32_t*>(a.cq + i);
        int32_t* r = reinterpret_cast<int32_t*>(a.cq_r + i);
        int32_t* d = reinterpret_cast<int32_t*>(a.cq_dk + i);
        uint64_t* kk = reinterpret_cast<uint64_t*>(a.cq_k + i);
        int32_t R = r[f], DK = d[f];
        uint64_t K = kk[f];
        if (pm.x < 0 || pm.x >= 2 * cnt) {  // no partner record: a malformed factor
            atomicOr(&a.ctl[kCtlBadGrs], 1);
            q[f] = -(__ldcg(a.list1 + i) + 1);
            continue;
        }
        win_append(R, K, DK, 1, kstop, last < nxt ? 1 : 0);
        win_append(R, K, DK, pm.y, pk, pk == KEY_INF ? 0 : 2 * pm.y - 1 - pm.z);
        q[f] = __ldcg(a.list1 + (pm.x >> 1));
        r[f] = R;
        d[f] = DK;
        kk[f] = K;
    }
}

// a splitter's final windows oriented along its direction f (forward) and 1 - f (backward)
struct GrsWin {
    bool cyc;
    int32_t Ef, Eb;   // path: end vertices ahead / behind
    int32_t Rf, Rb;   // path: distances from s to them
    uint64_t ks;      // cycle: weakest key
    int32_t pf, pb;   // cycle: distance from s to the weakest edge's near endpoint, ahead / behind
    int32_t bf, bb;   //        and whether that endpoint is the edge's min-id end
};

__device__ __forceinline__ GrsWin grs_window(const ForestArgs& a, int i, int f) {
    const int2 e2 = __ldcg(a.end2 + i), d2 = __ldcg(a.dist2 + i), dk = __ldcg(a.dk2 + i);
    GrsWin W;
    W.cyc = !(e2.x < 0 && e2.y < 0);
    const int32_t ef = f ? e2.y : e2.x, eb = f ? e2.x : e2.y;
    W.Ef = -(ef + 1);
    W.Eb = -(eb + 1);
    W.Rf = f ? d2.y : d2.x;
    W.Rb = f ? d2.x : d2.y;
    W.ks = __ldcg(&a.kraw[i].x);
    const int32_t dkf = f ? dk.y : dk.x, dkb = f ? dk.x : dk.y;
    W.pf = dkf >> 1;
    W.bf = dkf & 1;
    W.pb = dkb >> 1;
    W.bb = dkb & 1;
    return W;
}

// path id of the walk of a splitter (constant along it) and its length
__device__ __forceinline__ int32_t grs_path_id(const GrsWin& W, int32_t& L) {
    if (W.cyc) {
        L = W.pf + W.pb + 1;
        return key_min_end(W.ks);
    }
    L = W.Rf + W.Rb + 1;
    return W.Eb < W.Ef ? W.Eb : W.Ef;
}

// results of a vertex at forward distance d from the splitter (d = 0: the splitter)
struct GrsOut {
    int32_t l, p;
    int2 f;
    int dir, rs;      // slot toward the path-id end; removed slot (-1: none)
    int ncyc;
};

__device__ __forceinline__ GrsOut grs_vertex(int32_t x, int2 nb, int fslot, int32_t d, const GrsWin& W) {
    const int bslot = fslot ^ 1;
    GrsOut o;
    o.ncyc = 0;
    o.rs = -1;
    o.f = nb;
    if (!W.cyc) {
        const int32_t Df = W.Rf - d, Db = W.Rb + d;
        // the smaller end is the path id (reading c11); equal ends: a single vertex (slot 0)
        if (W.Eb < W.Ef || (W.Eb == W.Ef && bslot == 0)) { o.dir = bslot; o.l = W.Eb; o.p = Db + 1; }
        else { o.dir = fslot; o.l = W.Ef; o.p = Df + 1; }
        return o;
    }
    const int32_t L = W.pf + W.pb + 1;
    int32_t dkf, dkb;
    if (d <= W.pf) { dkf = 2 * (W.pf - d) + W.bf; dkb = 2 * (d + W.pb) + W.bb; }
    else { dkf = 2 * (L - d + W.pf) + W.bf; dkb = 2 * (d - W.pf - 1) + W.bb; }
    // the weakest edge is the forward one (x its near endpoint) or the backward one
    // (x its far endpoint; for d = 0 the edge closing the cycle behind s)
    const bool remf = d == W.pf, remb = d == W.pf + 1 || (d == 0 && W.pb == 0);
    int2 c;
    ulonglong2 ek;
    if (fslot == 0) { c = make_int2(dkf, dkb); ek = make_ulonglong2(remf ? W.ks : 0ull, remb ? W.ks : 0ull); }
    else { c = make_int2(dkb, dkf); ek = make_ulonglong2(remb ? W.ks : 0ull, remf ? W.ks : 0ull); }
    const CycOut co = cycle_finish(x, nb, ek, W.ks, c);
    o.l = co.l;
    o.p = co.pos;
    o.f = co.f;
    o.dir = (c.x & 1) ? 0 : 1;
    o.rs = (ek.x == W.ks) ? 0 : ((ek.y == W.ks) ? 1 : -1);
    o.ncyc = co.ncyc;
    return o;
}

// path lengths at path-ID vertices, from the splitters' final windows
__global__ void __launch_bounds__(256) k_grs_len(ForestArgs a) {
    LF_TL(g_tl_forest, 7);
    pdl_wait();
    const int cnt = __ldcg(&a.ctl[kCtlCnt1]);
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < cnt; i += gridDim.x * blockDim.x) {
        const GrsWin W = grs_window(a, i, 0);
        int32_t L;
        const int32_t l = grs_path_id(W, L);
        // paths: the path-id end writes; cycles: every splitter on it (the same value)
        if (l < 0 || (int64_t)l >= a.N) { atomicOr(&a.ctl[kCtlBadGrs], 1); continue; }  // malformed
        if (W.cyc || l == __ldcg(a.list1 + i)) a.len[l] = L;
    }
}

// walk priority on splitter-free cycles: a hash, so that the walks that stop at the first
// lower-priority vertex are short whatever the id order along the cycle
__device__ __forceinline__ uint64_t grs_prio(int32_t v) {
    return ((uint64_t)((uint32_t)v * 0x85EBCA6Bu ^ 0xC2B2AE35u) << 32) | (uint32_t)v;
}

// vertices no walk visited lie on cycles without a splitter: the lowest-priority vertex of
// each walks it (slot 0 ahead), records the weakest edge (first occurrence, reading c9)
// and writes the path length at the path-ID vertex
// Vertices no walk claimed lie on cycles without a splitter (C5: ~840 k cycles, 3.7% of the
// vertices, the longest ~200).  Only a vertex whose priority is below both neighbours' can
// be its cycle's lowest: k_grs_cyccand lists those (one pass over the visit bitmap, one
// atomic per warp), k_grs_cycfind walks from each of them, dynamically scheduled.
__global__ void __launch_bounds__(256) k_grs_cyccand(ForestArgs a) {
    LF_TL(g_tl_forest, 15);
    pdl_wait();
    __shared__ int s_w[8];
    __shared__ int s_base;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    const int64_t words = (a.N + 31) >> 5;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    // block-uniform loop: one list atomic per CTA and pass (a per-warp atomic put ~10^5 on one
    // control line, the hot spot of §5.5)
    for (int64_t b0 = (int64_t)blockIdx.x * blockDim.x; b0 < words; b0 += stride) {
        const int64_t wi = b0 + threadIdx.x;
        uint32_t m = 0;
        if (wi < words) {
            m = ~__ldcg(a.grs_bits + wi);
            if ((wi + 1) * 32 > a.N) m &= (1u << (a.N - wi * 32)) - 1u;
        }
        uint32_t cm = 0;  // candidates among the unclaimed bits
        for (uint32_t q = m; q;) {
            const int bit = __ffs(q) - 1;
            q &= q - 1u;
            const int32_t v = (int32_t)(wi * 32 + bit);
            const int4 r = __ldcg(a.grs_rec + (int64_t)v);
            const bool ok = (uint32_t)r.x < (uint32_t)a.N && (uint32_t)r.y < (uint32_t)a.N;
            const uint64_t pv = grs_prio(v);
            if (!ok || (pv < grs_prio(r.x) && pv < grs_prio(r.y))) cm |= 1u << bit;  // malformed: let the walk flag it
        }
        const int n = __popc(cm);
        int incl = n;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int y = __shfl_up_sync(0xffffffffu, incl, o);
            if (lane >= o) incl += y;
        }
        if (lane == 31) s_w[wid] = incl;
        __syncthreads();
        if (threadIdx.x == 0) {
            int tsum = 0;
            for (int q = 0; q < (int)(blockDim.x >> 5); q++) { const int x = s_w[q]; s_w[q] = tsum; tsum += x; }
            s_base = tsum ? atomicAdd(&a.ctl[kCtlCand], tsum) : 0;
        }
        __syncthreads();
        int pos = s_base + s_w[wid] + incl - n;
        __syncthreads();  // s_w / s_base are reused by the next pass
        while (cm) {
            const int bit = __ffs(cm) - 1;
            cm &= cm - 1u;
            a.list2[pos++] = (int32_t)(wi * 32 + bit);
        }
    }
}

__device__ __forceinline__ void grs_cyc_walk(const ForestArgs& a, int32_t v, int cnt) {
    int2 nbv;
    float2 wv;
    grs_load(a, v, nbv, wv);
    const uint64_t pv = grs_prio(v);
    // one walk around the cycle from v (slot 0 ahead) folds the window and gives up at
    // the first lower-priority vertex: only the lowest one completes it (the critical
    // path of a long splitter-free cycle is this walk plus the claim walk below)
    uint64_t K = KEY_INF;
    int32_t DK = 0, R = 0;
    int32_t prev = v, cur = v;
    int2 nbc = nbv;
    float2 wc = wv;
    int fs = 0;
    bool lowest = true;
    do {
        const int32_t nxt = fs ? nbc.y : nbc.x;
        const float wn = fs ? wc.y : wc.x;
        if ((uint32_t)nxt >= (uint32_t)a.N || R > a.N) { atomicOr(&a.ctl[kCtlBadGrs], 1); lowest = false; break; }
        if (grs_prio(nxt) < pv) { lowest = false; break; }
        int2 nbn;
        float2 wnx;
        grs_load(a, nxt, nbn, wnx);
        const uint64_t k = edge_key(cur, nxt, wn, cur < nxt ? nbc : nbn);
        if (k < K) { K = k; DK = 2 * R + (cur < nxt ? 1 : 0); }
        R++;
        prev = cur;
        cur = nxt;
        nbc = nbn;
        wc = wnx;
        fs = nbc.x == prev ? 1 : 0;
    } while (cur != v);
    if (!lowest) return;
    if (cur != v) return;  // the walk was stopped (a malformed factor)
    const int stripe = (int)((v >> 5) & (kCycStripes - 1));
    const int64_t cap = grs_cyc_cap(a.N);
    const int local = atomicAdd(&a.ctl[kCtlCycS + kCtlCycStride * stripe], 1);
    if (local >= cap) { atomicOr(&a.ctl[kCtlBadGrs], 1); return; }  // overlapping "cycles"
    const int c = (int)(stripe * cap + local);
    a.grs_cyc[c] = make_int4(v, DK, R, 0);
    a.grs_cyck[c] = K;
    const int32_t lk = key_min_end(K);
    if (K == KEY_INF || lk < 0 || (int64_t)lk >= a.N) { atomicOr(&a.ctl[kCtlBadGrs], 1); return; }
    a.len[lk] = R;
    // claim the cycle's records as walk 2 cnt + c from v (slot 0 ahead) for k_grs_emit
    const int tc = 2 * cnt + c;
    prev = v;
    cur = v;
    nbc = nbv;
    fs = 0;
    int32_t d = 0;
    do {
        grs_claim(a, cur, tc, d, fs);
        atomicOr(a.grs_bits + (cur >> 5), 1u << (cur & 31));
        const int32_t nxt = fs ? nbc.y : nbc.x;
        const int4 rn = __ldcg(a.grs_rec + (int64_t)nxt);
        prev = cur;
        cur = nxt;
        nbc = make_int2(rn.x, rn.y);
        fs = nbc.x == prev ? 1 : 0;
        d++;
    } while (cur != v);
}

__global__ void __launch_bounds__(256) k_grs_cycfind(ForestArgs a) {
    LF_TL(g_tl_forest, 8);
    pdl_wait();
    const int ncand = __ldcg(&a.ctl[kCtlCand]);
    const int cnt = __ldcg(&a.ctl[kCtlCnt1]);
    // a static stride (a dynamic schedule's counter was one more hot line: 1.8 vs 1.4 ms)
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < ncand; i += gridDim.x * blockDim.x)
        grs_cyc_walk(a, __ldcg(a.list2 + i), cnt);
}

// tile-local exclusive prefix of the path lengths (the tail of k_lf_full2)
// LB / 8 threads per tile, 8 consecutive lengths each (two 16-byte loads): a serial local
// scan, one warp scan and one scan of the warp totals (a per-element block scan spent ~60
// instructions per vertex: the C5 len group 1.41 -> 1.24 ms)
constexpr int kLsT = LB / 8;
__global__ void __launch_bounds__(kLsT) k_grs_lenscan(ForestArgs a) {
    LF_TL(g_tl_forest, 9);
    __shared__ int wsum[kLsT / 32];
    pdl_wait();
    const int64_t b0 = a.lo + (int64_t)blockIdx.x * LB;
    const int64_t g0 = b0 + 8 * (int64_t)threadIdx.x;
    int x[8];
    if (g0 + 8 <= a.hi && ((((uintptr_t)(a.len + g0)) & 15) == 0)) {
        const int4 u = __ldcs(reinterpret_cast<const int4*>(a.len + g0));
        const int4 w = __ldcs(reinterpret_cast<const int4*>(a.len + g0) + 1);
        x[0] = u.x; x[1] = u.y; x[2] = u.z; x[3] = u.w; x[4] = w.x; x[5] = w.y; x[6] = w.z; x[7] = w.w;
    } else {
#pragma unroll
        for (int k = 0; k < 8; k++) x[k] = g0 + k < a.hi ? __ldcg(a.len + g0 + k) : 0;
    }
    int t = 0;
#pragma unroll
    for (int k = 0; k < 8; k++) t += x[k];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    int inc = t;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int y = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane >= o) inc += y;
    }
    if (lane == 31) wsum[w] = inc;
    __syncthreads();
    int before = 0, total = 0;
#pragma unroll
    for (int q = 0; q < kLsT / 32; q++) {
        const int ws = wsum[q];
        before += q < w ? ws : 0;
        total += ws;
    }
    int run = before + inc - t;  // exclusive prefix of this thread's first value in the tile
#pragma unroll
    for (int k = 0; k < 8; k++) {
        if (x[k] && g0 + k < a.hi) a.off[g0 + k] = run;
        run += x[k];
    }
    if (threadIdx.x == 0) a.tsum[blockIdx.x] = total;
}

// Walk descriptors: one 32-byte record per splitter j < cnt (its walks t = 2j + f) and per
// splitter-free cycle (j = cnt + c, walk t = 2 cnt + c), so that the emit reads ONE sector
// per vertex instead of the window arrays and the path offset.
//   path:  {kind 0, base, l, p_s | sgn, 0, 0, 0}: the splitter sits at position p_s; a vertex
//          at distance d along direction f has p = p_s + sgn_f d, sgn_f = f ? -sgn : sgn
//   cycle: {kind 1 | bf << 1 | bb << 2, base, pf, pb | ks}: the window of direction 0
//   kind & 8: a malformed factor (path id out of range)
// base = prefix(l), the exclusive prefix of the path lengths at the path id l.
constexpr int kDescBad = 8;
__global__ void __launch_bounds__(256) k_grs_desc(ForestArgs a) {
    LF_TL(g_tl_forest, 13);
    pdl_wait();
    const int cnt = __ldcg(&a.ctl[kCtlCnt1]);
    // descriptors fit [N]: splitters and splitter-free cycles (>= 3 vertices each) are
    // disjoint on a valid factor; a malformed one is cut off (its vertices flag it in the emit)
    auto put = [&](int64_t j, const GrsWin& W) {
        int32_t L;
        const int32_t l = grs_path_id(W, L);
        int4 h0, h1 = make_int4(0, 0, 0, 0);
        if (l < 0 || (int64_t)l >= a.N) {
            h0 = make_int4(kDescBad, 0, 0, 0);
        } else {
            const int32_t base = __ldcg(a.tsum + l / LB) + __ldcg(a.off + l);
            if (W.cyc) {
                h0 = make_int4(1 | (W.bf << 1) | (W.bb << 2), base, W.pf, W.pb);
                h1 = make_int4((int32_t)(uint32_t)W.ks, (int32_t)(uint32_t)(W.ks >> 32), 0, 0);
            } else {  // grs_vertex's path rule at d = 0, fslot 0: the back end is the path id iff Eb < Ef
                const bool back = W.Eb < W.Ef;
                h0 = make_int4(0, base, l, back ? W.Rb + 1 : W.Rf + 1);
                h1 = make_int4(back ? 1 : -1, 0, 0, 0);
            }
        }
        a.grs_desc[2 * j] = h0;
        a.grs_desc[2 * j + 1] = h1;
    };
    const int64_t stride = (int64_t)gridDim.x * blockDim.x, t0 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    for (int64_t j = t0; j < cnt; j += stride) put(j, grs_window(a, (int)j, 0));
    // the splitter-free cycles: the filled part of every stripe of the cycle index space
    const int64_t cap = grs_cyc_cap(a.N);
    int lmax = 0;
    for (int sidx = 0; sidx < kCycStripes; sidx++) {
        const int64_t ns = min((int64_t)__ldcg(&a.ctl[kCtlCycS + kCtlCycStride * sidx]), cap);
        for (int64_t q = t0; q < ns; q += stride) {
            const int64_t c = sidx * cap + q;
            const int4 cr = __ldcg(a.grs_cyc + c);
            lmax = max(lmax, cr.z);
            GrsWin W;
            W.cyc = true;
            W.ks = __ldcg(a.grs_cyck + c);
            W.pf = cr.y >> 1;
            W.bf = cr.y & 1;
            W.pb = cr.z - W.pf - 1;
            W.bb = W.bf ^ 1;  // the far endpoint of the weakest edge
            put(cnt + c, W);
        }
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) lmax = max(lmax, __shfl_xor_sync(0xffffffffu, lmax, o));
    if ((threadIdx.x & 31) == 0 && lmax) atomicMax(&a.ctl[kCtlCycMax], lmax);  // lf_forest_stats
}

// Every vertex's outputs in one coalesced pass over the vertices: its claim (walk t, d,
// fslot) selects the descriptor of walk t, from which d gives path id, position, forest
// slots and r = prefix(l) + p - 1 (grs_vertex's rules; cycles through grs_vertex itself).
// path_id, pos, iperm, forest are written in vertex order; (perm, a, b, c) go to r as one
// 16-byte record: the 32-byte sector of r-space is complete once the path neighbour
// (r xor 1) has been swept -- one or two planes later on C5 -- while four separate 4-byte
// stores per vertex left most sectors partial in L2 and paid a DRAM read-modify-write each
// (14.3 vs 6.6 ms).  k_grs_split copies the records out to the four arrays.
// one vertex of the emit: its claim (walk j's descriptor h0/h1, direction f, distance d,
// forward slot fs) -> outputs; pv / dg: its signed slot values and diagonal
__device__ __forceinline__ void grs_emit_one(const ForestArgs& a, int64_t v, int2 nb, int f, int32_t d, int fs,
                                             int4 h0, int4 h1, float2 pv, float dg, int& ncyc, bool& bad) {
    GrsOut o;
    if (!(h0.x & kDescBad)) {
        if (!(h0.x & 1)) {  // a path
            const int32_t sg = f ? -h1.x : h1.x;
            o.l = h0.z;
            o.p = h0.w + sg * d;
            o.dir = sg > 0 ? fs ^ 1 : fs;
            o.f = nb;
            o.rs = -1;
            o.ncyc = 0;
        } else {
            GrsWin W;
            W.cyc = true;
            W.ks = (uint64_t)(uint32_t)h1.x | ((uint64_t)(uint32_t)h1.y << 32);
            const int bf = (h0.x >> 1) & 1, bb = (h0.x >> 2) & 1;
            W.pf = f ? h0.w : h0.z;
            W.pb = f ? h0.z : h0.w;
            W.bf = f ? bb : bf;
            W.bb = f ? bf : bb;
            o = grs_vertex((int32_t)v, nb, fs, d, W);
        }
    }
    const int32_t r = h0.y + o.p - 1;
    if ((h0.x & kDescBad) || r < 0 || (int64_t)r >= a.N || o.l < 0 || (int64_t)o.l >= a.N) {
        bad = true;
        __stcs(a.path_id + v, -1);
        __stcs(a.pos + v, -1);
        __stcs(a.iperm + v, -1);
        __stcs(a.forest + v, make_int2(-1, -1));
        return;
    }
    __stcs(a.path_id + v, o.l);
    __stcs(a.pos + v, o.p);
    __stcs(a.iperm + v, r);
    __stcs(a.forest + v, o.f);
    ncyc += o.ncyc;
    int4 q4 = make_int4((int32_t)v, 0, 0, 0);
    if (a.ta) {  // the forest neighbour toward the path-id end is perm[r-1] (reading c15)
        const int ps = (o.dir != o.rs && (o.dir ? nb.y : nb.x) >= 0) ? o.dir : -1;
        const int ss = ((o.dir ^ 1) != o.rs && (o.dir ? nb.x : nb.y) >= 0) ? (o.dir ^ 1) : -1;
        q4.y = ps < 0 ? 0 : __float_as_int(ps ? pv.y : pv.x);
        q4.z = __float_as_int(dg);
        q4.w = ss < 0 ? 0 : __float_as_int(ss ? pv.y : pv.x);
    }
    a.grs_rout[r] = q4;
}

// Every vertex's outputs in one coalesced pass over the vertices: its claim (walk t, d,
// fslot) selects the descriptor of walk t, from which d gives path id, position, forest
// slots and r = prefix(l) + p - 1 (grs_vertex's rules; cycles through grs_vertex itself).
// path_id, pos, iperm, forest are written in vertex order; (perm, a, b, c) go to r as one
// 16-byte record: the 32-byte sector of r-space is complete once the path neighbour
// (r xor 1) has been swept -- one or two planes later on C5 -- while four separate 4-byte
// stores per vertex left most sectors partial in L2 and paid a DRAM read-modify-write each
// (14.3 vs 6.6 ms).  k_grs_split copies the records out to the four arrays.  A thread may
// take kEmitB vertices (a grid stride apart) per pass with all their loads issued first:
// measured on C5, 1 -> 3.17 ms, 2 -> 3.88, 4 -> 3.27 (the wider sweep costs the r-records'
// L2 locality what the extra loads in flight gain).
#ifndef LF_EMIT_B
#define LF_EMIT_B 1
#endif
constexpr int kEmitB = LF_EMIT_B;
__global__ void __launch_bounds__(256) k_grs_emit(ForestArgs a) {
    LF_TL(g_tl_forest, 10);
    pdl_wait();
    const int cnt = __ldcg(&a.ctl[kCtlCnt1]);
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    int ncyc = 0;
    bool bad = false;
    for (int64_t v0 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v0 < a.N; v0 += kEmitB * stride) {
        int4 rc[kEmitB], h0[kEmitB], h1[kEmitB];
        int j[kEmitB], f[kEmitB], fs[kEmitB];
        int32_t d[kEmitB];
        float2 pv[kEmitB];
        float dg[kEmitB];
#pragma unroll
        for (int u = 0; u < kEmitB; u++) {
            const int64_t v = v0 + u * stride;
            rc[u] = v < a.N ? __ldcs(a.grs_rec + v) : make_int4(-1, -1, 0, 0);
            pv[u] = (a.ta && v < a.N) ? __ldcs(a.pi2_val + v) : make_float2(0.f, 0.f);
            dg[u] = (a.ta && v < a.N) ? __ldcs(a.diag + v) : 0.f;
        }
#pragma unroll
        for (int u = 0; u < kEmitB; u++) {
            const int64_t v = v0 + u * stride;
            j[u] = -1;
            f[u] = 0;
            d[u] = 0;
            fs[u] = 0;
            if (v >= a.N) continue;
            const int2 nb = make_int2(rc[u].x, rc[u].y);
            if (grs_splitter(a, (int32_t)v, nb)) {  // a splitter: d = 0 on its slot-0 window
                j[u] = __ldcg(a.bidx1 + v);
            } else if (__ldcg(a.grs_bits + (v >> 5)) & (1u << (v & 31))) {  // claimed by walk t
                const int t = rc[u].z;
                d[u] = (int32_t)((uint32_t)rc[u].w >> 1);
                fs[u] = rc[u].w & 1;
                if (t >= 0 && t < 2 * cnt) { j[u] = t >> 1; f[u] = t & 1; }
                else if (t >= 2 * cnt && grs_cyc_valid(a, t - 2 * cnt)) j[u] = cnt + (t - 2 * cnt);
            }  // else no walk claimed it: a malformed factor
        }
#pragma unroll
        for (int u = 0; u < kEmitB; u++) {
            h0[u] = make_int4(kDescBad, 0, 0, 0);
            h1[u] = make_int4(0, 0, 0, 0);
            if (j[u] >= 0) {
                h0[u] = __ldcg(a.grs_desc + 2 * (int64_t)j[u]);
                h1[u] = __ldcg(a.grs_desc + 2 * (int64_t)j[u] + 1);
            }
        }
#pragma unroll
        for (int u = 0; u < kEmitB; u++) {
            const int64_t v = v0 + u * stride;
            if (v < a.N)
                grs_emit_one(a, v, make_int2(rc[u].x, rc[u].y), f[u], d[u], fs[u], h0[u], h1[u], pv[u], dg[u],
                             ncyc, bad);
        }
    }
    if (bad) atomicOr(&a.ctl[kCtlBadGrs], 1);
#pragma unroll
    for (int o = 16; o; o >>= 1) ncyc += __shfl_xor_sync(0xffffffffu, ncyc, o);
    if ((threadIdx.x & 31) == 0 && ncyc && a.n_cycles) atomicAdd(a.n_cycles, (unsigned long long)ncyc);
}

// perm, a, b, c from the emit's interleaved records at r: one coalesced pass
__global__ void __launch_bounds__(256) k_grs_split(ForestArgs a) {
    LF_TL(g_tl_forest, 11);
    pdl_wait();
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < a.N; r += stride) {
        const int4 q = __ldcs(a.grs_rout + r);
        __stcs(a.perm + r, q.x);
        if (a.ta) {
            __stcs(reinterpret_cast<int32_t*>(a.ta) + r, q.y);
            __stcs(reinterpret_cast<int32_t*>(a.tb) + r, q.z);
            __stcs(reinterpret_cast<int32_t*>(a.tc) + r, q.w);
        }
    }
}

// which linear-forest algorithm: the tile path for graphs whose paths stay in 1024-id
// tiles (C1-C3), the global ruling set for large graphs (LF_FOREST=tile|grs overrides)
static bool use_grs(int64_t N) {
    const char* e = getenv("LF_FOREST");
    if (e && !strcmp(e, "grs")) return true;
    if (e && !strcmp(e, "tile")) return false;
    return N >= ((int64_t)1 << 22);
}

int forest_run(int64_t N, const int32_t* pi2, const float* pi2_w, int32_t* forest, int32_t* path_id,
               int32_t* pos, int32_t* perm, int32_t* iperm, int64_t* n_cycles, const ForestWs& w,
               cudaStream_t s, const TriOut* tri) {
    if (N == 0) {
        if (n_cycles) LF_CUDA(cudaMemsetAsync(n_cycles, 0, sizeof(int64_t), s));
        return LF_OK;
    }
    int rcp = forest_prepare();
    if (rcp) return rcp;
    // zero the control block in a PDL kernel: it runs while the factor's last kernel is
    // still finishing, and k_lf_full1's CTAs become resident meanwhile (a memset node
    // would serialise: ~5 us between the factor and the tile pass)
    LF_CUDA(launch_pdl(k_ctl_zero, 1, 256, 0, s, w.ctl));
    ForestArgs a;
    memset(&a, 0, sizeof(a));
    a.N = N;
    a.lo = 0;
    a.hi = N;
    a.pi2 = (const int2*)pi2;
    a.pi2_w = (const float2*)pi2_w;
    a.forest = (int2*)forest;
    for (int i = 0; i < 2; i++) {
        a.rq1[i] = w.rq1[i];
        a.rk1[i] = w.rk1[i];
        a.rr2[i] = w.rr2[i];
        a.rdk[i] = w.rdk[i];
    }
    a.bidx1 = w.bidx1;
    a.loc2 = w.loc2;
    a.list1 = w.list1;
    a.end2 = w.end2;
    a.dist2 = w.dist2;
    a.kraw = w.kraw;
    a.dk2 = w.dk2;
    a.cq = w.cq;
    a.cq_k = w.cq_k;
    a.cq_r = w.cq_r;
    a.cq_dk = w.cq_dk;
    a.ctl = w.ctl;
    a.path_id = path_id;
    a.pos = pos;
    a.len = w.len;
    a.off = w.off;
    a.tsum = w.tsum;
    a.pdir = w.pdir;
    a.n_cycles = (unsigned long long*)n_cycles;
    a.max_steps = max_steps_for(N) < kMaxSteps ? max_steps_for(N) : kMaxSteps;
    const int tiles = (int)((N + LB - 1) / LB);
    if (use_grs(N)) {
        a.list1 = w.list1;
        a.grs_rec = w.grs_rec;
        a.list2 = w.list2;  // k_grs_cyccand's candidates
        a.grs_shift = getenv("LF_GRS_SHIFT") ? atoi(getenv("LF_GRS_SHIFT")) : kGrsShift;
        if (a.grs_shift < 20 || a.grs_shift > 31) a.grs_shift = kGrsShift;
        a.grs_bits = w.grs_bits;
        a.grs_cyc = w.grs_cyc;
        a.grs_cyck = w.grs_cyck;
        a.grs_meet = w.grs_meet;
        a.grs_meetk = w.grs_meetk;
        a.grs_mstop = w.grs_mstop;
        a.perm = perm;
        a.iperm = iperm;
        a.pi2_val = tri ? (const float2*)tri->pi2_val : nullptr;
        a.diag = tri ? tri->diag : nullptr;
        a.ta = tri ? tri->a : nullptr;
        a.tb = tri ? tri->b : nullptr;
        a.tc = tri ? tri->c : nullptr;
        {
            LF_PROF("grs_pack", -1, s);
            LF_CUDA(launch_pdl(k_grs_pack, persistent_grid((const void*)k_grs_pack, 256), 256, 0, s, a));
            const int chunks = (int)((N + 2047) / 2048);
            LF_CUDA(launch_pdl(k_tile_prefix, 1, kPrefT, 0, s, w.tsum, chunks, (const int*)w.ctl,
                               (unsigned long long*)nullptr, 1));
            LF_CUDA(launch_pdl(k_grs_list, persistent_grid((const void*)k_grs_list, 256), 256, 0, s, a));
        }
        {
            LF_PROF("grs_walk", -1, s);
            // large graphs: 2 CTAs (16 warps) per SM -- fewer walks in flight keep their band of
            // records in L2 (C5, dynamic schedule: 8 CTAs/SM 8.4 ms, 4: 7.3, 3: 6.9, 2: 6.6,
            // 1: 8.5); graphs whose records fit L2 anyway want the latency hiding (C4: 8 CTAs/SM)
            const int bpsm_def = N >= ((int64_t)1 << 25) ? 2 : 8;
            const int bpsm = getenv("LF_WALK_BPSM") ? atoi(getenv("LF_WALK_BPSM")) : bpsm_def;
            LF_CUDA(launch_pdl(k_grs_walk, sm_count() * (bpsm > 0 ? bpsm : 2), 256, 0, s, a));
            LF_CUDA(launch_pdl(k_grs_meet, persistent_grid((const void*)k_grs_meet, 256), 256, 0, s, a));
        }
        {
            LF_PROF("red_scan", -1, s);
            LF_CUDA(launch_red_full(a, s));
        }
        {
            LF_PROF("grs_len", -1, s);
            LF_CUDA(launch_pdl(k_grs_len, persistent_grid((const void*)k_grs_len, 256), 256, 0, s, a));
            LF_CUDA(launch_pdl(k_grs_cyccand, persistent_grid((const void*)k_grs_cyccand, 256), 256, 0, s, a));
            LF_CUDA(launch_pdl(k_grs_cycfind, persistent_grid((const void*)k_grs_cycfind, 256), 256, 0, s, a));
            LF_CUDA(launch_pdl(k_grs_lenscan, tiles, kLsT, 0, s, a));
            LF_CUDA(launch_pdl(k_tile_prefix, 1, kPrefT, 0, s, w.tsum, tiles, (const int*)w.ctl,
                               (unsigned long long*)n_cycles, 1));
        }
        a.grs_rout = w.grs_meet;  // [2N] int4, unused after k_grs_meet
        a.grs_desc = w.grs_desc;
        {
            LF_PROF("grs_desc", -1, s);
            LF_CUDA(launch_pdl(k_grs_desc, persistent_grid((const void*)k_grs_desc, 256), 256, 0, s, a));
        }
        {
            LF_PROF(tri ? "grs_emit_tri" : "grs_emit", -1, s);
            LF_CUDA(launch_pdl(k_grs_emit, persistent_grid((const void*)k_grs_emit, 256), 256, 0, s, a));
        }
        {
            LF_PROF(tri ? "grs_split_tri" : "grs_split", -1, s);
            LF_CUDA(launch_pdl(k_grs_split, persistent_grid((const void*)k_grs_split, 256), 256, 0, s, a));
        }
        return LF_OK;
    } else {
        {
            LF_PROF("lf_tile", -1, s);
            LF_CUDA(launch_pdl(k_lf_full1, tiles, LT, kFull1Smem, s, a));
            LF_CUDA(cudaGetLastError());
        }
        {
            LF_PROF("red_scan", -1, s);
#ifndef LF_NO_GRID_RED  // diagnostics only: measures the launch cost (wrong results)
            // cooperative cluster launch (the grid path's barrier): see launch_red_full
            LF_CUDA(launch_red_full(a, s));
#endif
        }
        {
            LF_PROF("lf_expand", -1, s);
            LF_CUDA(launch_pdl(k_lf_full2, tiles, ET, sizeof(TileSmemE), s, a));
        }
    }
    {
        LF_PROF(tri ? "perm_tridiag" : "perm", -1, s);
        LF_CUDA(launch_pdl(k_tile_prefix, 1, kPrefT, 0, s, w.tsum, tiles, (const int*)w.ctl,
                           (unsigned long long*)n_cycles, 0));
        LF_CUDA(launch_pdl(k_perm_tri, persistent_grid((const void*)k_perm_tri, 256), 256, 0, s, N,
                           (const int32_t*)path_id, (const int32_t*)pos, (const int32_t*)w.off,
                           (const int32_t*)w.tsum, (int)LB, (const uint8_t*)w.pdir, (const int2*)forest,
                           (const int2*)pi2, tri ? (const float2*)tri->pi2_val : nullptr,
                           tri ? tri->diag : nullptr, perm, iperm, tri ? tri->a : nullptr,
                           tri ? tri->b : nullptr, tri ? tri->c : nullptr, (const int*)w.ctl));
    }
    return LF_OK;
}

int forest_stats(const ForestWs& w, int32_t* out, int cap) {
    int h[kCtlInts];
    LF_CUDA(cudaMemcpy(h, w.ctl, sizeof(h), cudaMemcpyDeviceToHost));
    // [0] boundary vertices cycle pass, [1] rank pass, [2] reduced steps cycle, [3] rank,
    // [4] splitter nodes cycle pass, [5] unvisited, [6] fallback tiles, [7] nodes rank pass,
    // [8] max node-scan steps
    int steps1 = 0, steps2 = 0;
    for (int i = 0; i < 64; i++) {
        if (h[kCtlRed1 + i]) steps1 = i + 2;
        if (h[kCtlRed2 + i]) steps2 = i + 2;
    }
    // [10] splitter-free cycles of the ruling-set path, [11] the longest of them
    int v[12] = {h[kCtlCnt1], h[kCtlCnt2], steps1, steps2, h[kCtlStat], h[kCtlStat + 1], h[kCtlStat + 2],
                 h[kCtlStat + 3], h[kCtlStat + 4], h[kCtlBad] | h[kCtlBadGrs], 0, h[kCtlCycMax]};
    for (int q = 0; q < kCycStripes; q++) v[10] += h[kCtlCycS + kCtlCycStride * q];
    for (int i = 0; i < cap && i < 12; i++) out[i] = v[i];
    // [16..31]: per-phase cycle sums (units of 1024 cycles; LF_PHASE_TIMING builds only)
    const unsigned long long* ph = reinterpret_cast<const unsigned long long*>(h + 208);
    for (int i = 0; i < 8 && 16 + i < cap; i++) out[16 + i] = (int)(ph[i] >> 10);
    // [24..27]: reduced-scan small-path timestamps (ns, summed over runs; timing builds)
    const unsigned long long* rt = reinterpret_cast<const unsigned long long*>(h + 224);
    for (int i = 0; i < 4 && 24 + i < cap; i++) out[24 + i] = (int)(rt[i] >> 10);
    return LF_OK;
}


// ---------------------------------------------------------------------------
// partitioned runs: exit records, global exit-graph scan, fold-back, offsets
// ---------------------------------------------------------------------------
struct ExitRec {
    int32_t g, q0, q1, d0, d1, pad;
    uint64_t k0, k1;
};

size_t exit_record_bytes() { return sizeof(ExitRec); }

__device__ __forceinline__ bool is_exit_marker(int32_t m, int64_t N) { return (int64_t)m <= -(N + 1); }
__device__ __forceinline__ int32_t exit_vertex(int32_t m, int64_t N) { return (int32_t)(-(int64_t)m - N - 1); }

// one record per own boundary vertex with a cross-rank link: per slot, the cross-rank
// neighbour (distance 1, edge key), or the rank-local result of the reduced scan (an end
// marker, or the next exit vertex of this rank with the distance and min key to it)
template <bool MIN>
__global__ void k_exit_records(ForestArgs a, const int32_t* list, const int* count, ExitRec* rec, int* rcount) {
    const int cnt = *count;
    const int stride = gridDim.x * blockDim.x;
    for (int base = blockIdx.x * blockDim.x + (threadIdx.x & ~31); base < cnt; base += stride) {
        const int idx = base + (threadIdx.x & 31);
        bool take = false;
        ExitRec r;
        if (idx < cnt) {
            const int32_t v = list[idx];
            const int2 nb = MIN ? a.pi2[v] : a.forest[v];
            const bool f0 = nb.x >= 0 && is_foreign(nb.x, a), f1 = nb.y >= 0 && is_foreign(nb.y, a);
            take = f0 || f1;
            if (take) {
                r.g = v;
                r.pad = 0;
                const int2 raw = a.end2[idx];
                int32_t q[2], d[2];
                uint64_t k[2];
#pragma unroll
                for (int i = 0; i < 2; i++) {
                    const int32_t x = i ? nb.y : nb.x;
                    const bool fx = i ? f1 : f0;
                    d[i] = 0;
                    k[i] = KEY_INF;
                    if (x < 0) q[i] = -(v + 1);
                    else if (fx) {
                        q[i] = x;
                        d[i] = 1;
                        if (MIN) k[i] = i ? a.ekb[idx].y : a.ekb[idx].x;
                    } else {
                        const int32_t m = i ? raw.y : raw.x;
                        q[i] = is_exit_marker(m, a.N) ? exit_vertex(m, a.N) : m;
                        if (MIN) k[i] = i ? a.kraw[idx].y : a.kraw[idx].x;
                        else d[i] = i ? a.dist2[idx].y : a.dist2[idx].x;
                    }
                }
                r.q0 = q[0]; r.q1 = q[1];
                r.d0 = d[0]; r.d1 = d[1];
                r.k0 = k[0]; r.k1 = k[1];
            }
        }
        const unsigned m = __ballot_sync(0xffffffffu, take);
        const int lane = threadIdx.x & 31;
        int pos = 0;
        if (lane == 0 && m) pos = atomicAdd(rcount, __popc(m));
        pos = __shfl_sync(0xffffffffu, pos, 0);
        if (take) rec[pos + __popc(m & ((1u << lane) - 1u))] = r;
    }
}

// the exit graph from the gathered records of all ranks (padding has g = -1)
template <bool MIN>
__global__ void k_exit_build(const ExitRec* rec, int64_t total, int32_t* glist, int2* gcq, ulonglong2* gcq_k,
                             int32_t* gbidx, int* gcount) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
        const ExitRec r = rec[i];
        if (r.g < 0) continue;
        const int pos = atomicAdd(gcount, 1);
        glist[pos] = r.g;
        gbidx[r.g] = pos;
        gcq[pos] = make_int2(r.q0, r.q1);
        gcq_k[pos] = MIN ? make_ulonglong2(r.k0, r.k1) : make_ulonglong2((uint32_t)r.d0, (uint32_t)r.d1);
    }
}

// exit marker at t -> the global result of t through its cross-rank slot
template <bool MIN>
__global__ void k_exit_fold(ForestArgs a, const int32_t* list, const int* count, const uint64_t* gcyc,
                            const int2* gend, const int2* gdist, const int32_t* gbidx) {
    const int cnt = *count;
    for (int idx = blockIdx.x * blockDim.x + threadIdx.x; idx < cnt; idx += gridDim.x * blockDim.x) {
        const int32_t b = list[idx];
        int2 raw = a.end2[idx];
        int2 dd = MIN ? make_int2(0, 0) : a.dist2[idx];
#pragma unroll
        for (int i = 0; i < 2; i++) {
            const int32_t m = i ? raw.y : raw.x;
            if (!is_exit_marker(m, a.N)) continue;
            const int32_t t = exit_vertex(m, a.N);
            const int gi = gbidx[t];
            if (MIN) {
                if (gcyc[gi] != KEY_INF) a.cyc_k[idx] = gcyc[gi];
            } else {
                const int2 nt = a.forest[t];
                const int so = (t == b) ? i : ((nt.x >= 0 && is_foreign(nt.x, a)) ? 0 : 1);
                const int32_t e = so ? gend[gi].y : gend[gi].x;
                const int32_t dg = so ? gdist[gi].y : gdist[gi].x;
                if (i) { raw.y = e; dd.y += dg; } else { raw.x = e; dd.x += dg; }
            }
        }
        if (!MIN) {
            a.end2[idx] = raw;
            a.dist2[idx] = dd;
        }
    }
}

// rank totals -> this rank's base offset; tot[G] = base, tot[G+1] = own total
__global__ void k_rank_base(int64_t* tot, int G, int rank) {
    if (threadIdx.x == 0) {
        int64_t b = 0;
        for (int q = 0; q < rank; q++) b += tot[q];
        tot[G] = b;
    }
}

__global__ void k_own_total(const int32_t* len, const int32_t* off, int64_t n_own, int64_t* out) {
    if (threadIdx.x == 0) *out = n_own > 0 ? (int64_t)off[n_own - 1] + len[n_own - 1] : 0;
}

// global offsets of the cross-rank paths whose ID vertex this rank owns
__global__ void k_publish(const int32_t* glist, const int* gcount, const int2* gend, int64_t lo, int64_t hi,
                          const int32_t* off_own /* indexed by global id */, const int64_t* tot, int G,
                          int2* pub, int* pcount) {
    const int cnt = *gcount;
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < cnt; i += gridDim.x * blockDim.x) {
        const int32_t g = glist[i];
        if (g < lo || g >= hi) continue;  // each path with an own ID has an own exit vertex
        const int2 e = gend[i];
        const int32_t e0 = -(e.x + 1), e1 = -(e.y + 1);
        const int32_t l = e0 < e1 ? e0 : e1;
        if (l >= lo && l < hi) pub[atomicAdd(pcount, 1)] = make_int2(l, (int32_t)(tot[G] + off_own[l]));
    }
}

__global__ void k_pub_apply(const int2* pub, int64_t total, int32_t* offG) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
        const int2 p = pub[i];
        if (p.x >= 0) offG[p.x] = p.y;
    }
}

__global__ void k_perm_part(int64_t lo, int64_t hi, const int32_t* path_id, const int32_t* pos, const int32_t* off,
                            const int32_t* offG, const int64_t* tot, int G, int32_t* iperm) {
    const int64_t base = tot[G];
    for (int64_t v = lo + (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < hi; v += (int64_t)gridDim.x * blockDim.x) {
        const int32_t l = path_id[v];
        const int64_t o = (l >= lo && l < hi) ? base + off[l] : (int64_t)offG[l];
        iperm[v] = (int32_t)(o + pos[v] - 1);
    }
}

// the global exit-graph scan (same kernel as the reduced scan, on global-id buffers)
template <bool MIN>
static int exit_pass(const ForestArgs& a, const int32_t* list, const int* count, const ForestPartCtx& pc,
                     int64_t N, cudaStream_t s) {
    ExitRec* send = (ExitRec*)pc.rec_send;
    ExitRec* all = (ExitRec*)pc.rec_all;
    LF_CUDA(cudaMemsetAsync(send, 0xff, sizeof(ExitRec) * pc.exit_cap, s));
    LF_CUDA(cudaMemsetAsync(pc.gctl, 0, sizeof(int) * 256, s));
    {
        LF_PROF(MIN ? "exit_records_cycles" : "exit_records_ranks", -1, s);
        k_exit_records<MIN><<<persistent_grid((const void*)k_exit_records<MIN>, 256), 256, 0, s>>>(
            a, list, count, send, pc.gctl + 250);
        LF_CUDA(cudaGetLastError());
    }
    int rc = pc.allgather(pc.ctx, send, all, sizeof(ExitRec) * pc.exit_cap, s);
    if (rc) return rc;
    const int64_t total = (int64_t)pc.G * pc.exit_cap;
    const int kBuildCnt = MIN ? kCtlCnt1 : kCtlCnt2;
    k_exit_build<MIN><<<persistent_grid((const void*)k_exit_build<MIN>, 256), 256, 0, s>>>(
        all, total, pc.glist, pc.gcq, pc.gcq_k, pc.gbidx, pc.gctl + kBuildCnt);
    LF_CUDA(cudaGetLastError());
    ForestArgs g;
    memset(&g, 0, sizeof(g));
    g.N = N;
    g.lo = 0;
    g.hi = N;
    for (int i = 0; i < 2; i++) {
        g.rq1[i] = pc.gq[i];
        g.rk1[i] = pc.gk[i];
        g.rq2[i] = pc.gq[i];
        g.rr2[i] = pc.gr[i];
    }
    g.list1 = pc.glist;
    g.list2 = pc.glist;
    g.cq = pc.gcq;
    g.cq_k = pc.gcq_k;
    g.ctl = pc.gctl;
    g.cyc_k = pc.gcyc;
    g.end2 = pc.gend;
    g.dist2 = pc.gdist;
    g.max_steps = a.max_steps;
    {
        LF_PROF(MIN ? "exit_scan_cycles" : "exit_scan_ranks", -1, s);
        rc = coop_launch(k_red_scan<MIN>, RT, g, s, sizeof(RedSmem));
        if (rc) return rc;
    }
    {
        LF_PROF(MIN ? "exit_fold_cycles" : "exit_fold_ranks", -1, s);
        k_exit_fold<MIN><<<persistent_grid((const void*)k_exit_fold<MIN>, 256), 256, 0, s>>>(
            a, list, count, pc.gcyc, pc.gend, pc.gdist, pc.gbidx);
        LF_CUDA(cudaGetLastError());
    }
    return LF_OK;
}

int forest_part_run(int64_t N, const int32_t* pi2, const float* pi2_w, int32_t* forest, int32_t* path_id,
                    int32_t* pos, int32_t* iperm, int64_t* n_cycles, const ForestWs& w,
                    const ForestPartCtx& pc, cudaStream_t s) {
    const int64_t lo = pc.lo, hi = pc.hi, n_own = hi - lo;
    int rc = forest_prepare();
    if (rc) return rc;
    LF_CUDA(cudaMemsetAsync(w.ctl, 0, sizeof(int) * kCtlInts, s));
    LF_CUDA(cudaMemsetAsync(pc.tot, 0, sizeof(int64_t) * (pc.G + 2), s));
    ForestArgs a;
    memset(&a, 0, sizeof(a));
    a.N = N;
    a.lo = lo;
    a.hi = hi;
    // own-slice buffers, offset so that vertex g is element g
    a.pi2 = (const int2*)pi2 - lo;
    a.pi2_w = (const float2*)pi2_w - lo;
    a.forest = (int2*)forest - lo;
    for (int i = 0; i < 2; i++) {
        a.rq1[i] = w.rq1[i] - lo;
        a.rk1[i] = w.rk1[i] - lo;
        a.rq2[i] = w.rq2[i] - lo;
        a.rr2[i] = w.rr2[i] - lo;
    }
    a.cyc_k = w.cyc_k;
    a.bidx1 = w.bidx1 - lo;
    a.bidx2 = w.bidx2 - lo;
    a.loc1 = w.loc1 - lo;
    a.kst = w.kst - lo;
    a.loc2 = w.loc2 - lo;
    a.end2 = w.end2;
    a.dist2 = w.dist2;
    a.kraw = w.kraw;
    a.ekb = w.ekb;
    a.list1 = w.list1;
    a.list2 = w.list2;
    a.cq = w.cq;
    a.cq_k = w.cq_k;
    a.ctl = w.ctl;
    a.path_id = path_id - lo;
    a.pos = pos - lo;
    a.len = w.len - lo;
    a.pdir = w.pdir - lo;
    a.n_cycles = (unsigned long long*)&pc.tot[pc.G + 1];
    a.ghost_list = pc.ghost_list;
    a.n_ghost = pc.n_ghost;
    a.ghost_below = pc.ghost_below;
    a.ghost_nb = pc.ghost_nb;
    a.max_steps = max_steps_for(N) < kMaxSteps ? max_steps_for(N) : kMaxSteps;
    const int tiles = (int)((n_own + LB - 1) / LB);
    const int smem = (int)sizeof(TileSmem);
    if (tiles > 0) {
        LF_PROF("lf_local1", -1, s);
        k_lf_local1<<<tiles, LT, smem, s>>>(a);
        LF_CUDA(cudaGetLastError());
    }
    {
        LF_PROF("red_scan_cycles", -1, s);
        rc = coop_launch(k_red_scan<true>, RT, a, s, sizeof(RedSmem));
        if (rc) return rc;
    }
    rc = exit_pass<true>(a, w.list1, w.ctl + kCtlCnt1, pc, N, s);
    if (rc) return rc;
    if (tiles > 0) {
        LF_PROF("lf_local2", -1, s);
        k_lf_local2<<<tiles, LT, kTileSmemNoKeys, s>>>(a);
        LF_CUDA(cudaGetLastError());
    }
    {
        LF_PROF("red_scan_ranks", -1, s);
        rc = coop_launch(k_red_scan<false>, RT, a, s, sizeof(RedSmem));
        if (rc) return rc;
    }
    rc = exit_pass<false>(a, w.list2, w.ctl + kCtlCnt2, pc, N, s);
    if (rc) return rc;
    if (tiles > 0) {
        LF_PROF("lf_local3", -1, s);
        k_lf_local3<<<tiles, LT, kTileSmemNoKeys, s>>>(a);
        LF_CUDA(cudaGetLastError());
    }
    // path offsets: own exclusive scan, rank bases, published offsets of cross-rank paths
    {
        LF_PROF("path_offsets", -1, s);
        if (n_own > 0) {
            size_t tb = w.scan_tmp_bytes;
            LF_CUDA(cub::DeviceScan::ExclusiveSum(w.scan_tmp, tb, w.len, w.off, (int)n_own, s));
        }
        k_own_total<<<1, 32, 0, s>>>(w.len, w.off, n_own, &pc.tot[pc.rank]);
        rc = pc.allreduce_i64(pc.ctx, pc.tot, pc.G, s);  // every rank's slot is filled by its owner
        if (rc) return rc;
        k_rank_base<<<1, 32, 0, s>>>(pc.tot, pc.G, pc.rank);
        LF_CUDA(cudaMemsetAsync(pc.pub_send, 0xff, sizeof(int2) * pc.exit_cap, s));
        k_publish<<<persistent_grid((const void*)k_publish, 256), 256, 0, s>>>(
            pc.glist, pc.gctl + kCtlCnt2, pc.gend, lo, hi, w.off - lo, pc.tot, pc.G, pc.pub_send, pc.gctl + 251);
        LF_CUDA(cudaGetLastError());
        rc = pc.allgather(pc.ctx, pc.pub_send, pc.pub_all, sizeof(int2) * pc.exit_cap, s);
        if (rc) return rc;
        k_pub_apply<<<persistent_grid((const void*)k_pub_apply, 256), 256, 0, s>>>(pc.pub_all, (int64_t)pc.G * pc.exit_cap,
                                                                               pc.offG);
        LF_CUDA(cudaGetLastError());
    }
    {
        LF_PROF("perm", -1, s);
        k_perm_part<<<persistent_grid((const void*)k_perm_part, 256), 256, 0, s>>>(lo, hi, path_id - lo, pos - lo,
                                                                               w.off - lo, pc.offG, pc.tot, pc.G,
                                                                               iperm - lo);
        LF_CUDA(cudaGetLastError());
    }
    if (n_cycles) {
        rc = pc.allreduce_i64(pc.ctx, &pc.tot[pc.G + 1], 1, s);
        if (rc) return rc;
        LF_CUDA(cudaMemcpyAsync(n_cycles, &pc.tot[pc.G + 1], sizeof(int64_t), cudaMemcpyDeviceToDevice, s));
    }
    return LF_OK;
}

#ifdef LF_TIMELINE
int timeline_forest(unsigned long long* out, int reset) {
    if (reset) {
        unsigned long long h[32];
        for (int i = 0; i < 32; i += 2) { h[i] = ~0ull; h[i + 1] = 0; }
        return cudaMemcpyToSymbol(g_tl_forest, h, sizeof(h)) == cudaSuccess ? 0 : -1;
    }
    return cudaMemcpyFromSymbol(out, g_tl_forest, sizeof(g_tl_forest)) == cudaSuccess ? 0 : -1;
}
#else
int timeline_forest(unsigned long long*, int) { return -1; }
#endif
}  // namespace lf
