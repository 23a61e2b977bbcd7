// lf_factor.cu -- weighted [0,n]-factor, Algorithm 2 of PAPER.md (L93-L128, §3.2, §4.1).
//
// B200 design:
//  * one `propose` kernel per round (Alg. 2 L14-L22, the generalized SpMV of §4.1): G
//    lanes per CSR row stream col/val with read-only loads, each lane keeps a sorted
//    register top-n of 64-bit keys, a shuffle butterfly merges the G lists.  The key
//    order is total, so the reduction order never changes the result (bit parity).
//  * one `mutual` kernel per round (Alg. 2 L26-L28): confirms mutual proposals, keeps
//    pi canonical, writes the next round's state byte (degree + charge, L8-L12) and
//    appends still-live rows to the next worklist.  Rows whose charge-free candidate
//    set became empty are retired: they provably never propose or receive a proposal
//    again, so later rounds only touch live rows.
//  * no host synchronisation: round count, worklist sizes and the maximality flags
//    (L23-L25) stay on the device; the launch chain is fixed and graph-capturable.
#include <cooperative_groups.h>
#include <cuda_runtime.h>

#include <climits>
#include <cstdint>

#include "lf_common.cuh"
#include "lf_internal.h"

#include <cstdio>
#include <cstdlib>
#include <cstring>

namespace cg = cooperative_groups;

namespace lf {

#ifdef LF_TIMELINE
__device__ unsigned long long g_tl_factor[16];
#endif

struct ProposeArgs {
    int64_t N;                           // CSR rows (this partition's own rows)
    int64_t row_base;                    // vertex id of CSR row r is row_base + r
    const int64_t* __restrict__ rowptr;
    const int32_t* __restrict__ col;
    const float* __restrict__ val;
    const uint8_t* __restrict__ state;   // NULL in a fresh round 0 (all degrees 0, no charge)
    const int32_t* __restrict__ pi;      // NULL in a fresh round 0
    const int32_t* __restrict__ wl;      // worklist; NULL = all rows
    const int32_t* __restrict__ wl_count;
    int32_t* __restrict__ prop_j;        // [N*n] new proposals of worklist rows
    float* __restrict__ prop_v;          // [N*n] their signed values
    float* __restrict__ diag;            // [N] written when non-NULL (round 0)
    int charging;
    unsigned long long* live_rows;       // NULL or 64 partial-sum slots of round k
    unsigned long long* live_nnz;        // NULL or 64 partial-sum slots of round k
    int* proposed;                       // &flags[k]: set to 1 if anything was proposed
    int64_t defer_len;                   // rows with more entries go to the long-row list
    int32_t* defer_list;                 // long rows of this round (processed warp-per-row)
    int32_t* defer_count;
};

// append the rows flagged by lanes of this warp to the long-row list
__device__ __forceinline__ void defer_append(const ProposeArgs& a, bool take, int32_t v) {
    const unsigned m = __ballot_sync(0xffffffffu, take);
    if (!m) return;
    const int lane = threadIdx.x & 31;
    int base = 0;
    if (lane == 0) base = atomicAdd(a.defer_count, __popc(m));
    base = __shfl_sync(0xffffffffu, base, 0);
    if (take) a.defer_list[base + __popc(m & ((1u << lane) - 1u))] = v;
}

// G lanes per row (G = 1..32), NN = n.  Persistent grid-stride over the worklist.
template <int NN, int G>
__device__ __forceinline__ void propose_phase(const ProposeArgs& a) {
    constexpr int RPW = 32 / G;  // rows per warp per iteration
    const int lane = threadIdx.x & 31;
    const int li = lane & (G - 1);
    const int64_t warp_global = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t n_warps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const int64_t count = a.wl_count ? (int64_t)*a.wl_count : a.N;

    unsigned long long my_live = 0, my_nnz = 0;
    int my_prop = 0;

    for (int64_t base = warp_global * RPW; base < count; base += n_warps * RPW) {
        const int64_t idx = base + lane / G;
        const bool valid = idx < count;
        int32_t v = -1;
        if (valid) v = a.wl ? __ldg(a.wl + idx) : (int32_t)(a.row_base + idx);
        const int64_t row = (int64_t)v - a.row_base;
        int deg = 0;
        uint32_t cv = 0;
        int32_t p[NN];
#pragma unroll
        for (int s = 0; s < NN; s++) p[s] = -1;
        int64_t rs = 0, re = 0;
        if (valid) {
            if (a.state) {
                uint8_t st = a.state[v];
                deg = st & ST_DEG;
                cv = (st & ST_CHARGE) ? 1u : 0u;
            }
            if (a.pi && deg > 0) {
#pragma unroll
                for (int s = 0; s < NN; s++) p[s] = a.pi[(int64_t)v * NN + s];
            }
            rs = __ldg(a.rowptr + row);
            re = __ldg(a.rowptr + row + 1);
        }
        const bool deferred = valid && (re - rs) > a.defer_len;
        defer_append(a, deferred && li == 0, v);
        if (deferred) re = rs;
        uint64_t top[NN];
#pragma unroll
        for (int s = 0; s < NN; s++) top[s] = 0;
        uint32_t theta0 = 0;
        uint32_t dbits = 0;
        for (int64_t e = rs + li; e < re; e += G) {
            const int32_t j = __ldg(a.col + e);
            const float x = __ldg(a.val + e);
            if (j == v) {  // diagonal: not an edge (A' = |A| - diag|A|, L231)
                dbits = __float_as_uint(x);
                continue;
            }
            if ((__float_as_uint(x) & 0x7FFFFFFFu) == 0u) continue;  // zero: not an edge (L31)
            uint32_t sj = 0;
            if (a.state) sj = a.state[j];
            if ((int)(sj & ST_DEG) == NN) continue;  // j saturated (L15)
            bool in_pi = false;
#pragma unroll
            for (int s = 0; s < NN; s++) in_pi |= (p[s] == j);
            if (in_pi) continue;  // already confirmed (L19: W \ pi(v))
            theta0 = 1;
            if (a.charging && (((sj & ST_CHARGE) ? 1u : 0u) == cv)) continue;  // L17
            topn_insert<NN>(top, make_key(x, j));
        }
        // merge the G partial lists; OR the flags
        topn_merge_group<NN, G>(top);
#pragma unroll
        for (int off = G / 2; off >= 1; off >>= 1) {
            theta0 |= __shfl_xor_sync(0xffffffffu, theta0, off);
            dbits |= __shfl_xor_sync(0xffffffffu, dbits, off);
        }
        if (valid && !deferred && li == 0) {
            const int need = NN - deg;
            int32_t* pj = a.prop_j + (int64_t)v * NN;
            float* pv = a.prop_v + (int64_t)v * NN;
            int np = 0;
#pragma unroll
            for (int s = 0; s < NN; s++) {
                if (s < need && top[s] != 0) {
                    pj[s] = key_col(top[s]);
                    pv[s] = key_val(top[s]);
                    np++;
                } else {
                    pj[s] = (s == 0 && !theta0) ? PROP_RETIRED : -1;
                }
            }
            if (a.diag) a.diag[v] = __uint_as_float(dbits);
            if (theta0) {
                my_live += 1;
                my_nnz += (unsigned long long)(re - rs);
            }
            my_prop |= (np > 0);
        }
    }
    // one atomic per warp
#pragma unroll
    for (int off = 16; off >= 1; off >>= 1) {
        my_live += __shfl_xor_sync(0xffffffffu, my_live, off);
        my_nnz += __shfl_xor_sync(0xffffffffu, my_nnz, off);
        my_prop |= __shfl_xor_sync(0xffffffffu, my_prop, off);
    }
    if (lane == 0) {
        const int slot = (int)(warp_global & 63);
        if (a.live_rows && my_live) atomicAdd(a.live_rows + slot, my_live);
        if (a.live_nnz && my_nnz) atomicAdd(a.live_nnz + slot, my_nnz);
        if (my_prop && *(volatile int*)a.proposed == 0) atomicOr(a.proposed, 1);
    }
}

template <int NN, int G>
__global__ void __launch_bounds__(256) k_propose(ProposeArgs a) {
    LF_TL(g_tl_factor, 1);
    pdl_wait();
    pdl_trigger();
    propose_phase<NN, G>(a);
}

// Round 0 (every row proposes; Alg. 2 L14-L22 at k = 0) as a tiled streaming kernel: a
// CTA takes PT/G consecutive rows, stages their col/val range into shared memory with
// coalesced 16-byte loads, and scans each row from shared memory with G lanes (G = 1:
// thread per row).  A tile whose entry span exceeds ETILE (a hub row) is scanned from
// global memory instead.  Same per-row semantics and outputs as k_propose.
constexpr int PT = 256;
constexpr int ETILE = 4096;

// sorted-descending top-NN insertion with an early exit: most candidates lose against
// the current last slot, so the common path is one 64-bit compare
template <int NN>
__device__ __forceinline__ void topn_insert_fast(uint64_t (&t)[NN], uint64_t x) {
    if (x <= t[NN - 1]) return;
#pragma unroll
    for (int i = NN - 1; i > 0; i--) {
        if (x > t[i - 1]) t[i] = t[i - 1];
        else { t[i] = x; return; }
    }
    t[0] = x;
}

// branch-free insertion network: t stays sorted descending; x = 0 leaves it unchanged
template <int NN>
__device__ __forceinline__ void topn_insert_net(uint64_t (&t)[NN], uint64_t x) {
#pragma unroll
    for (int i = 0; i < NN; i++) {
        const uint64_t h = t[i] > x ? t[i] : x;
        x = t[i] > x ? x : t[i];
        t[i] = h;
    }
}

// the same network guarded by a predicate (no key masking, one 64-bit compare per slot):
// the round-0 stream is ALU-bound, and this is most of its per-entry work
template <int NN>
__device__ __forceinline__ void topn_insert_pred(uint64_t (&t)[NN], uint64_t x, bool ok) {
#pragma unroll
    for (int i = 0; i < NN; i++) {
        const bool c = ok && x > t[i];
        const uint64_t h = c ? x : t[i];
        x = c ? t[i] : x;
        t[i] = h;
    }
}

#if defined(LF_TILE_MINB) && LF_TILE_MINB > 0
#define LF_TILE_BOUNDS __launch_bounds__(PT, LF_TILE_MINB)
#else
#define LF_TILE_BOUNDS __launch_bounds__(PT)
#endif
#ifdef LF_BRANCHFREE
#define TOPN_INS topn_insert
#else
#define TOPN_INS topn_insert_fast
#endif
template <int NN, int G, bool CHARGED>
__global__ void LF_TILE_BOUNDS k_propose_tile(ProposeArgs a) {
    constexpr int R = PT / G;
    __shared__ __align__(16) int2 sent[ETILE];  // interleaved (col, value bits)
    __shared__ int64_t srp[R + 1];
    const int tid = threadIdx.x;
    const int64_t r0 = (int64_t)blockIdx.x * R;
    for (int i = tid; i <= R; i += PT) {
        const int64_t r = r0 + i < a.N ? r0 + i : a.N;
        srp[i] = __ldg(a.rowptr + r);
    }
    __syncthreads();
    const int64_t e0 = srp[0], e1 = srp[R];
    const int64_t a0 = e0 & ~(int64_t)3;
    const bool staged = (e1 - a0) <= ETILE;
    if (staged) {
        const int64_t v1 = e1 & ~(int64_t)3;
        const int nvec = (int)((v1 - a0) >> 2);
        const int4* c4 = reinterpret_cast<const int4*>(a.col + a0);
        const int4* f4 = reinterpret_cast<const int4*>(a.val + a0);
        for (int i = tid; i < nvec; i += PT) {
            const int4 c = __ldg(c4 + i);
            const int4 f = __ldg(f4 + i);
            int4* d = reinterpret_cast<int4*>(sent + 4 * i);
            d[0] = make_int4(c.x, f.x, c.y, f.y);
            d[1] = make_int4(c.z, f.z, c.w, f.w);
        }
        for (int64_t e = v1 + tid; e < e1; e += PT)
            sent[e - a0] = make_int2(__ldg(a.col + e), __float_as_int(__ldg(a.val + e)));
    }
    __syncthreads();
    const int lr = tid / G, li = tid % G;
    const int64_t row = r0 + lr;
    const bool valid = row < a.N;
    const int32_t v = (int32_t)(a.row_base + row);
    const int64_t rs = srp[lr];
    int64_t re = valid ? srp[lr + 1] : rs;
    const bool deferred = valid && (re - rs) > a.defer_len;
    defer_append(a, deferred && li == 0, v);
    if (deferred) re = rs;
    uint32_t cv = 0;
    if (CHARGED && valid) cv = (a.state[v] & ST_CHARGE) ? 1u : 0u;
    uint64_t top[NN];
#pragma unroll
    for (int s = 0; s < NN; s++) top[s] = 0;
    uint32_t theta0 = 0, dbits = 0;
    if (staged) {
        const int hi = (int)(re - a0);
        for (int e = (int)(rs - a0) + li; e < hi; e += G) {
            const int2 ent = sent[e];
            const int32_t j = ent.x;
            const uint32_t xb = (uint32_t)ent.y;
            if (j == v) { dbits = xb; continue; }                        // diagonal (L231)
            const uint32_t ab = xb & 0x7FFFFFFFu;
            if (ab == 0u) continue;                                      // zero (L31)
            theta0 = 1;                 // round 0: nothing saturated, nothing confirmed
            if (CHARGED && (((a.state[j] & ST_CHARGE) ? 1u : 0u) == cv)) continue;  // L17
            TOPN_INS<NN>(top, ((uint64_t)ab << 32) | (((0x7FFFFFFFu - (uint32_t)j) << 1) | (xb >> 31)));
        }
    } else {
        for (int64_t e = rs + li; e < re; e += G) {
            const int32_t j = __ldg(a.col + e);
            const uint32_t xb = __float_as_uint(__ldg(a.val + e));
            if (j == v) { dbits = xb; continue; }
            const uint32_t ab = xb & 0x7FFFFFFFu;
            if (ab == 0u) continue;
            theta0 = 1;
            if (CHARGED && (((a.state[j] & ST_CHARGE) ? 1u : 0u) == cv)) continue;
            TOPN_INS<NN>(top, ((uint64_t)ab << 32) | (((0x7FFFFFFFu - (uint32_t)j) << 1) | (xb >> 31)));
        }
    }
    if (G > 1) {
        topn_merge_group<NN, G>(top);
#pragma unroll
        for (int off = G / 2; off >= 1; off >>= 1) {
            theta0 |= __shfl_xor_sync(0xffffffffu, theta0, off);
            dbits |= __shfl_xor_sync(0xffffffffu, dbits, off);
        }
    }
    unsigned long long my_live = 0, my_nnz = 0;
    int my_prop = 0;
    if (valid && !deferred && li == 0) {
        int32_t pj[NN];
        float pv[NN];
        int np = 0;
#pragma unroll
        for (int s = 0; s < NN; s++) {
            if (top[s] != 0) { pj[s] = key_col(top[s]); pv[s] = key_val(top[s]); np++; }
            else { pj[s] = (s == 0 && !theta0) ? PROP_RETIRED : -1; pv[s] = 0.0f; }
        }
        if (NN == 2) {
            reinterpret_cast<int2*>(a.prop_j)[v] = make_int2(pj[0], pj[NN > 1 ? 1 : 0]);
            reinterpret_cast<float2*>(a.prop_v)[v] = make_float2(pv[0], pv[NN > 1 ? 1 : 0]);
        } else if (NN == 4) {
            reinterpret_cast<int4*>(a.prop_j)[v] = make_int4(pj[0], pj[NN > 1 ? 1 : 0], pj[NN > 2 ? 2 : 0], pj[NN > 3 ? 3 : 0]);
            reinterpret_cast<float4*>(a.prop_v)[v] = make_float4(pv[0], pv[NN > 1 ? 1 : 0], pv[NN > 2 ? 2 : 0], pv[NN > 3 ? 3 : 0]);
        } else {
#pragma unroll
            for (int s = 0; s < NN; s++) {
                a.prop_j[(int64_t)v * NN + s] = pj[s];
                a.prop_v[(int64_t)v * NN + s] = pv[s];
            }
        }
        if (a.diag) a.diag[v] = __uint_as_float(dbits);
        if (theta0) { my_live = 1; my_nnz = (unsigned long long)(re - rs); }
        my_prop = np > 0;
    }
#pragma unroll
    for (int off = 16; off >= 1; off >>= 1) {
        my_live += __shfl_xor_sync(0xffffffffu, my_live, off);
        my_nnz += __shfl_xor_sync(0xffffffffu, my_nnz, off);
        my_prop |= __shfl_xor_sync(0xffffffffu, my_prop, off);
    }
    __shared__ unsigned long long red[3][PT / 32];
    if ((tid & 31) == 0) {
        red[0][tid >> 5] = my_live;
        red[1][tid >> 5] = my_nnz;
        red[2][tid >> 5] = (unsigned long long)my_prop;
    }
    __syncthreads();
    if (tid == 0) {
        unsigned long long l = 0, z = 0, pr = 0;
#pragma unroll
        for (int w = 0; w < PT / 32; w++) { l += red[0][w]; z += red[1][w]; pr |= red[2][w]; }
        // counters spread over 64 slots (one L2 atomic per CTA), summed by k_finalize
        if (a.live_rows && l) atomicAdd(a.live_rows + (blockIdx.x & 63), l);
        if (a.live_nnz && z) atomicAdd(a.live_nnz + (blockIdx.x & 63), z);
        if (pr && *(volatile int*)a.proposed == 0) atomicOr(a.proposed, 1);
    }
}

// ---------------------------------------------------------------------------
// Round 0 as a pipelined stream: persistent CTAs walk their tiles while cp.async (LDGSTS)
// copies the next tile's col/val range and the row pointers of the one after into the
// other shared-memory stage, so HBM reads overlap the row scans.
// ---------------------------------------------------------------------------
__device__ __forceinline__ void cp16(void* smem, const void* gmem) {
    const unsigned d = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(d), "l"(gmem));
}
__device__ __forceinline__ void cp8(void* smem, const void* gmem) {
    const unsigned d = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8;\n" ::"r"(d), "l"(gmem));
}
__device__ __forceinline__ void cp4(void* smem, const void* gmem) {
    const unsigned d = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;\n" ::"r"(d), "l"(gmem));
}
__device__ __forceinline__ void cp_commit() { asm volatile("cp.async.commit_group;\n" ::); }
__device__ __forceinline__ void cp_wait_all() { asm volatile("cp.async.wait_group 0;\n" ::: "memory"); }

#ifndef LF_SETILE
#define LF_SETILE 2048   // 38 KB of stages: 5 CTAs per SM (4096: 3), more bytes in flight
#endif
#ifndef LF_SPT
#define LF_SPT 256
#endif
constexpr int SPT = LF_SPT;         // threads
constexpr int SETILE = LF_SETILE;   // entries per stage (sparse rows; denser rows: kSetileBig)
#ifndef LF_SETILE_BIG
#define LF_SETILE_BIG 8192
#endif
constexpr int kSetileBig = LF_SETILE_BIG;  // 27-entry rows one lane each: 256 rows per tile fit a stage

template <int SE>
struct StreamSmem {
    int32_t col[2][SE];
    float val[2][SE];
    int64_t rp[3][SPT + 2];   // +2: rows of 16-byte multiples (bulk copies)
    int64_t a0[2];            // aligned start of the staged range per stage (or -1)
    unsigned long long bar[2];  // mbarriers of the bulk copies, one per prefetch batch parity
};

// one-thread bulk copies (TMA engine, no per-thread address arithmetic: the round-0 stream is
// ALU-bound and per-thread cp.async staging was a quarter of its instructions)
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init1(unsigned long long* b) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(b)) : "memory");
}
__device__ __forceinline__ void mbar_arrive_tx(unsigned long long* b, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait_parity(unsigned long long* b, uint32_t parity) {
    asm volatile(
        "{\n\t.reg .pred p;\n"
        "LF_MBW_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
        "@!p bra LF_MBW_%=;\n}" ::"r"(smem_u32(b)), "r"(parity) : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, unsigned long long* b) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(b)) : "memory");
}

template <int R>
__device__ __forceinline__ void issue_rowptr(const ProposeArgs& a, int64_t t, int64_t* dst) {
    const int64_t r0 = t * R;
    const int64_t cnt = (r0 + R <= a.N) ? R + 1 : a.N + 1 - r0;
    for (int i = threadIdx.x; i < cnt; i += blockDim.x) cp8(dst + i, a.rowptr + r0 + i);
}

// stage the entry range of a tile whose row pointers are in rp; returns false if too long
template <int SE>
__device__ __forceinline__ void issue_entries(const ProposeArgs& a, int64_t e0, int64_t e1, int32_t* scol,
                                              float* sval, int64_t* a0_out) {
    const int64_t a0 = e0 & ~(int64_t)3;
    if (e1 - a0 > SE) {
        if (threadIdx.x == 0) *a0_out = -1;
        return;
    }
    if (threadIdx.x == 0) *a0_out = a0;
    if ((((uintptr_t)a.col | (uintptr_t)a.val) & 15) != 0) {  // offset views: 4-byte copies
        for (int64_t e = e0 + threadIdx.x; e < e1; e += blockDim.x) {
            cp4(scol + (e - a0), a.col + e);
            cp4(sval + (e - a0), a.val + e);
        }
        return;
    }
    const int64_t v1 = e1 & ~(int64_t)3;
    const int nvec = (int)((v1 - a0) >> 2);
    for (int i = threadIdx.x; i < nvec; i += blockDim.x) {
        cp16(scol + 4 * i, a.col + a0 + 4 * i);
        cp16(sval + 4 * i, a.val + a0 + 4 * i);
    }
    for (int64_t e = v1 + threadIdx.x; e < e1; e += blockDim.x) {
        cp4(scol + (e - a0), a.col + e);
        cp4(sval + (e - a0), a.val + e);
    }
}

template <int NN, int G, bool CHARGED, int SE, int T = SPT>
__global__ void __launch_bounds__(T) k_propose_stream(ProposeArgs a) {
    LF_TL(g_tl_factor, 0);
    constexpr int R = T / G;
    extern __shared__ __align__(16) unsigned char sraw[];
    StreamSmem<SE>& S = *reinterpret_cast<StreamSmem<SE>*>(sraw);
    // small graphs: the long-row pass may launch and wait meanwhile (hides its launch); large
    // ones trigger at exit -- early-launched dependents sharing the SMs with this persistent
    // kernel cost more than the launch they hide (C5 graph replay 54.0 vs 45.1 ms without)
    if (a.N < ((int64_t)1 << 22)) pdl_trigger();
    const int tid = threadIdx.x;
    const int64_t ntiles = (a.N + R - 1) / R;
    const int64_t t0 = blockIdx.x;
    unsigned long long my_live = 0, my_nnz = 0;
    int my_prop = 0;
    // a prefetch batch: the entries of tile te (row pointers rpe, already staged) into stage
    // sb and the row pointers of tile tr (if any) into rps, on mbarrier bar; ranges the bulk
    // engine cannot take (the arrays' ends) fall back to per-thread cp.async
    const int64_t nnz = __ldg(a.rowptr + a.N);
    // bulk copies need 16-byte aligned sources (the caller's arrays may be offset views)
    const bool aligned_cv = (((uintptr_t)a.col | (uintptr_t)a.val) & 15) == 0;
    auto issue_batch = [&](int64_t te, const int64_t* rpe, int sb, int64_t tr, int64_t* rps,
                           unsigned long long* bar) {
        const int64_t rle = (te * R + R <= a.N) ? R : a.N - te * R;
        const int64_t e0 = rpe[0], e1 = rpe[rle];
        const int64_t ea = e0 & ~(int64_t)3, eb = (e1 + 3) & ~(int64_t)3;
        const bool fits = e1 - ea <= SE;
        const bool bulkE = fits && aligned_cv && eb <= nnz && eb - ea <= SE;
        const bool hasR = tr < ntiles;
        const int64_t r0 = tr * R;
        const int64_t rc = hasR ? ((r0 + R + 1 <= a.N + 1) ? R + 1 : a.N + 1 - r0) : 0;
        const int64_t rc2 = (rc + 1) & ~(int64_t)1;
        const bool bulkR = hasR && r0 + rc2 <= a.N + 1 && ((uintptr_t)(a.rowptr + r0) & 15) == 0;
        if (tid == 0) {
            S.a0[sb] = fits ? ea : -1;
            const uint32_t bytes = (bulkE ? (uint32_t)(eb - ea) * 8u : 0u) + (bulkR ? (uint32_t)rc2 * 8u : 0u);
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            mbar_arrive_tx(bar, bytes);
            if (bulkE) {
                bulk_g2s(S.col[sb], a.col + ea, (uint32_t)(eb - ea) * 4u, bar);
                bulk_g2s(S.val[sb], a.val + ea, (uint32_t)(eb - ea) * 4u, bar);
            }
            if (bulkR) bulk_g2s(rps, a.rowptr + r0, (uint32_t)rc2 * 8u, bar);
        }
        if (fits && !bulkE) {
            int64_t dummy;
            issue_entries<SE>(a, e0, e1, S.col[sb], S.val[sb], &dummy);
        }
        if (hasR && !bulkR) issue_rowptr<R>(a, tr, rps);
        cp_commit();
    };
    if (t0 < ntiles) {
        if (tid == 0) {
            mbar_init1(&S.bar[0]);
            mbar_init1(&S.bar[1]);
            asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        }
        // prologue: row pointers of the first tile (waited), then batch 0: its entries and
        // the next tile's row pointers
        issue_rowptr<R>(a, t0, S.rp[0]);
        cp_commit();
        cp_wait_all();
        __syncthreads();
        issue_batch(t0, S.rp[0], 0, t0 + gridDim.x, S.rp[1], &S.bar[0]);
    }
    int i = 0;
    for (int64_t t = t0; t < ntiles; t += gridDim.x, i++) {
        cp_wait_all();
        mbar_wait_parity(&S.bar[i & 1], (uint32_t)((i >> 1) & 1));
        __syncthreads();
        const int b = i & 1;
        const int64_t* rp = S.rp[i % 3];
        const int64_t tn = t + gridDim.x;
        if (tn < ntiles)  // prefetch: entries of the next tile, row pointers of the one after
            issue_batch(tn, S.rp[(i + 1) % 3], b ^ 1, tn + gridDim.x, S.rp[(i + 2) % 3], &S.bar[(i + 1) & 1]);
        const int64_t a0 = S.a0[b];
        const bool staged = a0 >= 0;
        const int32_t* scol = S.col[b];
        const float* sval = S.val[b];
        const int lr = tid / G, li = tid % G;
        const int64_t row = t * R + lr;
        const bool valid = row < a.N;
        const int32_t v = (int32_t)(a.row_base + row);
        const int64_t rs = valid ? rp[lr] : 0;
        int64_t re = valid ? rp[lr + 1] : 0;
        const bool deferred = valid && (re - rs) > a.defer_len;
        defer_append(a, deferred && li == 0, v);
        if (deferred) re = rs;
        uint32_t cv = 0;
        if (CHARGED && valid) cv = (a.state[v] & ST_CHARGE) ? 1u : 0u;
        uint64_t top[NN];
#pragma unroll
        for (int s2 = 0; s2 < NN; s2++) top[s2] = 0;
        uint32_t theta0 = 0, dbits = 0;
        if (staged) {
            // branch-free scan of the staged row: 32-bit smem offsets, a rejected entry
            // becomes key 0, which the insertion network never keeps
            const int lo = (int)(rs - a0) + li, hi = (int)(re - a0);
#pragma unroll 4
            for (int e = lo; e < hi; e += G) {
                const int32_t j = scol[e];
                const uint32_t xb = __float_as_uint(sval[e]);
                const uint32_t ab = xb & 0x7FFFFFFFu;
                const bool isd = j == v;                                 // diagonal (L231)
                dbits = isd ? xb : dbits;
                bool ok = !isd && ab != 0u;                              // zero (L31)
                if (CHARGED) {
                    theta0 |= ok ? 1u : 0u;
                    ok = ok && (((a.state[j] & ST_CHARGE) ? 1u : 0u) != cv);  // L17
                }
                const uint64_t key = ((uint64_t)ab << 32) | (((0x7FFFFFFFu - (uint32_t)j) << 1) | (xb >> 31));
                topn_insert_pred<NN>(top, key, ok);
            }
            // uncharged: every eligible entry entered the top list, so theta0 (some
            // eligible entry, L19) is "the list is not empty"; lanes merge it below
            if (!CHARGED) theta0 |= top[0] != 0 ? 1u : 0u;
        } else {
            for (int64_t e = rs + li; e < re; e += G) {
                const int32_t j = __ldg(a.col + e);
                const uint32_t xb = __float_as_uint(__ldg(a.val + e));
                if (j == v) { dbits = xb; continue; }                    // diagonal (L231)
                const uint32_t ab = xb & 0x7FFFFFFFu;
                if (ab == 0u) continue;                                  // zero (L31)
                theta0 = 1;
                if (CHARGED && (((a.state[j] & ST_CHARGE) ? 1u : 0u) == cv)) continue;  // L17
                topn_insert_fast<NN>(top, ((uint64_t)ab << 32) | (((0x7FFFFFFFu - (uint32_t)j) << 1) | (xb >> 31)));
            }
        }
        if (G > 1) {
            topn_merge_group<NN, G>(top);
#pragma unroll
            for (int off = G / 2; off >= 1; off >>= 1) {
                theta0 |= __shfl_xor_sync(0xffffffffu, theta0, off);
                dbits |= __shfl_xor_sync(0xffffffffu, dbits, off);
            }
        }
        if (valid && !deferred && li == 0) {
            int32_t pj[NN];
            float pv[NN];
            int np = 0;
#pragma unroll
            for (int s2 = 0; s2 < NN; s2++) {
                if (top[s2] != 0) { pj[s2] = key_col(top[s2]); pv[s2] = key_val(top[s2]); np++; }
                else { pj[s2] = (s2 == 0 && !theta0) ? PROP_RETIRED : -1; pv[s2] = 0.0f; }
            }
            if (NN == 2) {
                reinterpret_cast<int2*>(a.prop_j)[v] = make_int2(pj[0], pj[NN > 1 ? 1 : 0]);
                reinterpret_cast<float2*>(a.prop_v)[v] = make_float2(pv[0], pv[NN > 1 ? 1 : 0]);
            } else {
#pragma unroll
                for (int s2 = 0; s2 < NN; s2++) {
                    a.prop_j[(int64_t)v * NN + s2] = pj[s2];
                    a.prop_v[(int64_t)v * NN + s2] = pv[s2];
                }
            }
            if (a.diag) a.diag[v] = __uint_as_float(dbits);
            if (theta0) { my_live++; my_nnz += (unsigned long long)(re - rs); }
            my_prop |= np > 0;
        }
        __syncthreads();  // stage b and rp[i % 3] are reused two iterations later
    }
#pragma unroll
    for (int off = 16; off >= 1; off >>= 1) {
        my_live += __shfl_xor_sync(0xffffffffu, my_live, off);
        my_nnz += __shfl_xor_sync(0xffffffffu, my_nnz, off);
        my_prop |= __shfl_xor_sync(0xffffffffu, my_prop, off);
    }
    if ((tid & 31) == 0) {
        const int slot = (int)((blockIdx.x * (T / 32) + (tid >> 5)) & 63);
        if (a.live_rows && my_live) atomicAdd(a.live_rows + slot, my_live);
        if (a.live_nnz && my_nnz) atomicAdd(a.live_nnz + slot, my_nnz);
        if (my_prop && *(volatile int*)a.proposed == 0) atomicOr(a.proposed, 1);
    }
}

struct MutualArgs {
    int64_t N;                       // rows in all-rows mode (round 0)
    int64_t row_base;                // vertex of row r in all-rows mode: row_base + r
    int64_t gid_off;                 // global id of an own vertex v: v + gid_off (charges)
    const int32_t* __restrict__ wl;  // NULL = all rows (round 0)
    const int32_t* __restrict__ wl_count;
    const int32_t* __restrict__ prop_j;
    const float* __restrict__ prop_v;
    uint8_t* __restrict__ state;
    int32_t* __restrict__ pi;
    float* __restrict__ pi_w;
    float* __restrict__ pi_val;      // NULL if not requested
    int32_t* __restrict__ wl_next;   // NULL in the last round
    int32_t* __restrict__ wl_next_count;
    int32_t* __restrict__ wl_zero;   // count slot to reset for round k+2 (NULL: none)
    int fresh;                       // round 0 from scratch: state/pi not initialised yet
    int pad_state;                   // k_mutual0 also zeroes state[N..N+3] (whole-graph runs:
                                     // the rows mode fetches state bytes as aligned words)
    int next_charging;
    uint32_t next_k;
    uint32_t seed;
    unsigned long long thr;
};

template <int NN>
__device__ __forceinline__ void mutual_phase(const MutualArgs& a) {
    const int64_t count = a.wl_count ? (int64_t)*a.wl_count : a.N;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    if (a.wl_zero && blockIdx.x == 0 && threadIdx.x == 0) *a.wl_zero = 0;
    const int lane = threadIdx.x & 31;
    // warp-uniform trip count so that the warp-aggregated append is safe
    for (int64_t base = (int64_t)blockIdx.x * blockDim.x + (threadIdx.x & ~31); base < count;
         base += stride) {
        const int64_t idx = base + lane;
        bool keep = false;
        int32_t v = -1;
        if (idx < count) {
            v = a.wl ? __ldg(a.wl + idx) : (int32_t)(a.row_base + idx);
            int32_t pj[NN];
#pragma unroll
            for (int s = 0; s < NN; s++) pj[s] = a.prop_j[(int64_t)v * NN + s];
            int deg = 0;
            if (!a.fresh) deg = a.state[v] & ST_DEG;
            const bool retired = pj[0] == PROP_RETIRED;
            // Alg. 2 L27: keep w in prop(v) iff v in prop(w).  Confirmed slots are not in
            // prop_j (which holds only this round's new proposals) and always survive.
            uint64_t conf[NN];
            int nconf = 0;
#pragma unroll
            for (int s = 0; s < NN; s++) {
                conf[s] = 0;
                const int32_t w = pj[s];
                if (w >= 0) {
                    bool mutual = false;
#pragma unroll
                    for (int t = 0; t < NN; t++) mutual |= (a.prop_j[(int64_t)w * NN + t] == v);
                    if (mutual) {
                        conf[s] = make_key(a.prop_v[(int64_t)v * NN + s], w);
                        nconf++;
                    }
                }
            }
            if (nconf > 0 || a.fresh) {
                uint64_t t[NN];
#pragma unroll
                for (int s = 0; s < NN; s++) t[s] = 0;
                if (deg > 0) {
#pragma unroll
                    for (int s = 0; s < NN; s++) {
                        if (s < deg) {
                            const int32_t w = a.pi[(int64_t)v * NN + s];
                            const float aw = a.pi_w[(int64_t)v * NN + s];
                            uint32_t sg = 0;
                            if (a.pi_val) sg = __float_as_uint(a.pi_val[(int64_t)v * NN + s]) >> 31;
                            t[s] = make_key_abs(aw, sg, w);
                        }
                    }
                }
#pragma unroll
                for (int s = 0; s < NN; s++)
                    if (conf[s]) topn_insert<NN>(t, conf[s]);
#pragma unroll
                for (int s = 0; s < NN; s++) {
                    const int64_t o = (int64_t)v * NN + s;
                    if (t[s]) {
                        a.pi[o] = key_col(t[s]);
                        a.pi_w[o] = key_abs(t[s]);
                        if (a.pi_val) a.pi_val[o] = key_val(t[s]);
                    } else {
                        a.pi[o] = -1;
                        a.pi_w[o] = 0.0f;
                        if (a.pi_val) a.pi_val[o] = 0.0f;
                    }
                }
                deg += nconf;
            }
            if (a.wl_next) {
                uint32_t ch = 0;
                keep = !retired && deg < NN;
                if (keep && a.next_charging) ch = charge_bit((uint32_t)(v + a.gid_off), a.next_k, a.seed, a.thr);
                a.state[v] = (uint8_t)(deg | (ch ? ST_CHARGE : 0) | (keep ? ST_LIVE : 0));
            } else if (a.fresh || nconf > 0) {
                a.state[v] = (uint8_t)deg;
            }
        }
        if (a.wl_next) {
            // warp-aggregated append to the next worklist
            const unsigned m = __ballot_sync(0xffffffffu, keep);
            int32_t basepos = 0;
            if (lane == 0 && m) basepos = atomicAdd(a.wl_next_count, __popc(m));
            basepos = __shfl_sync(0xffffffffu, basepos, 0);
            if (keep) a.wl_next[basepos + __popc(m & ((1u << lane) - 1u))] = v;
        }
    }
}

template <int NN>
__global__ void __launch_bounds__(256) k_mutual(MutualArgs a) {
    pdl_wait();
    mutual_phase<NN>(a);
}

// NN consecutive slots of one row in one load (NN = 2, 4: 8- / 16-byte vector)
template <int NN, class T>
__device__ __forceinline__ void load_slots(const T* __restrict__ p, T (&o)[NN]) {
    if constexpr (NN == 2 && sizeof(T) == 4) {
        const uint2 x = *reinterpret_cast<const uint2*>(p);
        o[0] = *reinterpret_cast<const T*>(&x.x); o[1] = *reinterpret_cast<const T*>(&x.y);
    } else if constexpr (NN == 4 && sizeof(T) == 4) {
        const uint4 x = *reinterpret_cast<const uint4*>(p);
        o[0] = *reinterpret_cast<const T*>(&x.x); o[1] = *reinterpret_cast<const T*>(&x.y);
        o[2] = *reinterpret_cast<const T*>(&x.z); o[3] = *reinterpret_cast<const T*>(&x.w);
    } else {
#pragma unroll
        for (int s = 0; s < NN; s++) o[s] = p[s];
    }
}
template <int NN, class T>
__device__ __forceinline__ void store_slots(T* __restrict__ p, const T (&o)[NN]) {
    if constexpr (NN == 2 && sizeof(T) == 4) {
        uint2 x;
        x.x = *reinterpret_cast<const uint32_t*>(&o[0]); x.y = *reinterpret_cast<const uint32_t*>(&o[1]);
        *reinterpret_cast<uint2*>(p) = x;
    } else if constexpr (NN == 4 && sizeof(T) == 4) {
        uint4 x;
        x.x = *reinterpret_cast<const uint32_t*>(&o[0]); x.y = *reinterpret_cast<const uint32_t*>(&o[1]);
        x.z = *reinterpret_cast<const uint32_t*>(&o[2]); x.w = *reinterpret_cast<const uint32_t*>(&o[3]);
        *reinterpret_cast<uint4*>(p) = x;
    } else {
#pragma unroll
        for (int s = 0; s < NN; s++) p[s] = o[s];
    }
}

// Round 0's confirmation (Alg. 2 L26-L28 at k = 0) over all rows: the same outputs as
// mutual_phase with fresh = 1, with MB rows per thread whose loads are all issued before
// any result is used (the proposal gathers are the latency chain of this pass).  In a
// fresh round pi is empty and the proposals are already in key order, so the confirmed
// ones are copied in place order without a merge.
#ifndef LF_M0ROWS
// one worklist atomic per CTA: the warps' counts (warp-uniform tot) are combined in shared
// memory (a per-warp atomic put ~10^6 atomics on one counter per C5 round: its L2 line
// became the bottleneck of the mutual kernels); returns the warp's base position
__device__ __forceinline__ int block_append_base(int tot, int32_t* counter) {
    __shared__ int s_w[32];
    __shared__ int s_base;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    if (lane == 0) s_w[wid] = tot;
    __syncthreads();
    if (threadIdx.x == 0) {
        int t = 0;
        for (int q = 0; q < (int)(blockDim.x >> 5); q++) { const int x = s_w[q]; s_w[q] = t; t += x; }
        s_base = t ? atomicAdd(counter, t) : 0;
    }
    __syncthreads();
    const int b = s_base + s_w[wid];
    __syncthreads();  // s_w / s_base are reused by the next call
    return b;
}

#define LF_M0ROWS 4
#endif
constexpr int kMutual0Rows = LF_M0ROWS;  // rows per thread of k_mutual0 (loads in flight)

template <int NN, int MB>
__global__ void __launch_bounds__(256) k_mutual0(MutualArgs a) {
    LF_TL(g_tl_factor, 2);
    pdl_wait();
    if (a.wl_zero && blockIdx.x == 0 && threadIdx.x == 0) *a.wl_zero = 0;
    if (a.pad_state && blockIdx.x == 0 && threadIdx.x < 4) a.state[a.N + threadIdx.x] = 0;
    const int lane = threadIdx.x & 31;
    const int64_t chunk = (int64_t)blockDim.x * MB;
    for (int64_t c0 = (int64_t)blockIdx.x * chunk; c0 < a.N; c0 += (int64_t)gridDim.x * chunk) {
        int32_t pj[MB][NN], pw[MB][NN][NN];
        float pv[MB][NN];
#pragma unroll
        for (int b = 0; b < MB; b++) {
            const int64_t r = c0 + threadIdx.x + (int64_t)b * blockDim.x;
            if (r < a.N) {
                const int64_t v = a.row_base + r;
                load_slots<NN>(a.prop_j + v * NN, pj[b]);
                load_slots<NN>(a.prop_v + v * NN, pv[b]);
            } else {
#pragma unroll
                for (int s = 0; s < NN; s++) pj[b][s] = -1;
            }
        }
#pragma unroll
        for (int b = 0; b < MB; b++)
#pragma unroll
            for (int s = 0; s < NN; s++) {
                if (pj[b][s] >= 0) {
                    load_slots<NN>(a.prop_j + (int64_t)pj[b][s] * NN, pw[b][s]);
                } else {
#pragma unroll
                    for (int t = 0; t < NN; t++) pw[b][s][t] = -1;
                }
            }
        bool keepb[MB];
#pragma unroll
        for (int b = 0; b < MB; b++) {
            const int64_t r = c0 + threadIdx.x + (int64_t)b * blockDim.x;
            const int32_t v = (int32_t)(a.row_base + r);
            int32_t oj[NN];
            float ow[NN], ov[NN];
            int deg = 0;
#pragma unroll
            for (int s = 0; s < NN; s++) { oj[s] = -1; ow[s] = 0.0f; ov[s] = 0.0f; }
#pragma unroll
            for (int s = 0; s < NN; s++) {
                bool mutual = false;
#pragma unroll
                for (int t = 0; t < NN; t++) mutual |= (pw[b][s][t] == v);
                if (pj[b][s] >= 0 && mutual) {
                    // deg <= s: write the confirmed slot at position deg (predicated moves)
#pragma unroll
                    for (int q = 0; q < NN; q++)
                        if (q == deg) { oj[q] = pj[b][s]; ov[q] = pv[b][s]; ow[q] = fabsf(pv[b][s]); }
                    deg++;
                }
            }
            bool keep = false;
            if (r < a.N) {
                store_slots<NN>(a.pi + (int64_t)v * NN, oj);
                store_slots<NN>(a.pi_w + (int64_t)v * NN, ow);
                if (a.pi_val) store_slots<NN>(a.pi_val + (int64_t)v * NN, ov);
                uint32_t ch = 0;
                if (a.wl_next) {
                    keep = pj[b][0] != PROP_RETIRED && deg < NN;
                    if (keep && a.next_charging) ch = charge_bit((uint32_t)(v + a.gid_off), a.next_k, a.seed, a.thr);
                }
                a.state[v] = (uint8_t)(deg | (ch ? ST_CHARGE : 0) | (keep ? ST_LIVE : 0));
            }
            keepb[b] = keep;
        }
        if (a.wl_next) {  // one worklist atomic per CTA for all MB row batches
            unsigned m[MB];
            int tot = 0;
#pragma unroll
            for (int b = 0; b < MB; b++) { m[b] = __ballot_sync(0xffffffffu, keepb[b]); tot += __popc(m[b]); }
            int32_t basepos = block_append_base(tot, a.wl_next_count);
#pragma unroll
            for (int b = 0; b < MB; b++) {
                const int64_t r = c0 + threadIdx.x + (int64_t)b * blockDim.x;
                if (keepb[b]) a.wl_next[basepos + __popc(m[b] & ((1u << lane) - 1u))] = (int32_t)(a.row_base + r);
                basepos += __popc(m[b]);
            }
        }
    }
}

// Alg. 2 L23-L24 / L30: rounds = k+1 for the first uncharged round without proposals;
// also sums the live-row counter slots into live[k], live[M+k]
__device__ __forceinline__ void finalize_body(const int* flags, int M, int m, int k_m, int32_t* rounds,
                                              const unsigned long long* part, int64_t* live) {
    if (threadIdx.x == 0 && rounds) {
        int r = M;
        for (int k = 0; k < M; k++)
            if ((k % m) == k_m && flags[k] == 0) {
                r = k + 1;
                break;
            }
        *rounds = r;
    }
    if (live) {  // one warp per counter: lanes sum two of its 64 slots
        const int lane = threadIdx.x & 31;
        for (int i = threadIdx.x >> 5; i < 2 * M; i += blockDim.x >> 5) {
            const int k = i % M, which = i / M;
            const unsigned long long* q = part + (size_t)k * 128 + which * 64;
            unsigned long long t = q[lane] + q[lane + 32];
#pragma unroll
            for (int o = 16; o; o >>= 1) t += __shfl_xor_sync(0xffffffffu, t, o);
            if (lane == 0) live[i] = (int64_t)t;
        }
    }
}

__global__ void k_finalize(const int* flags, int M, int m, int k_m, int32_t* rounds,
                           const unsigned long long* part, int64_t* live) {
    pdl_wait();
    finalize_body(flags, M, m, k_m, rounds, part, live);
}

// Rounds 1..M-1 in one cooperative persistent kernel: after round 0 only the live rows
// (2-40% of them) remain, and separate launches would be latency-bound.  Per round:
// propose over the worklist | long rows warp-per-row | mutual, separated by grid barriers.
struct FusedArgs {
    ProposeArgs pa;      // round-independent fields (CSR, state, pi, prop, live slots base)
    MutualArgs ma;
    int32_t* wl[2];
    int32_t* counts;     // [3] worklist sizes (ring)
    int* flags;
    int32_t* long_rows;
    int32_t* long_count;
    unsigned long long* live_part;
    int M, m, k_m;
    int G;
    int32_t* rounds;     // finalize outputs (k_finalize's work, done by CTA 0 in the last round)
    int64_t* live;
    int cached;          // try the shared-memory cached mode (rounds_cached) first
    int32_t* bail;       // grid-wide "does not fit" flag of the cached mode (zeroed per run)
};

#ifndef LF_FUSED_T
#define LF_FUSED_T 512
#endif
#ifndef LF_FUSED_GRID_SM
#define LF_FUSED_GRID_SM 1   // one CTA per SM: grid barriers scale with the CTA count
#endif
#ifndef LF_FUSED_GRID
#define LF_FUSED_GRID 0      // > 0: absolute CTA count of the fused rounds kernel
#endif
// ---------------------------------------------------------------------------
// Cached mode of rounds 1..M-1: every CTA owns a fixed slice of the round-1 worklist L1
// (the rows mutual(0) kept) and keeps those rows -- state, confirmed keys and their CSR
// entries as keys -- in shared memory for all rounds.  Rows outside L1 never propose
// again and are never proposed to, so the slices cover every row the
// rounds touch.  Per round only two gathers remain: the state bytes of the entries'
// targets (before propose, L15/L17) and the partners' proposals (before mutual, L27),
// each one L2 level with every load of a CTA in flight together, instead of the
// worklist -> rowptr -> col -> state chains of the uncached phases.  The semantics are
// those of propose_phase/mutual_phase entry for entry (same eligibility tests in the same
// order, same keys), so the factor is bit-identical.  A slice that does not fit (too many
// rows, entries or a row longer than kCacheMaxRow) makes the whole grid bail out (a
// grid-wide flag) before anything global is written; the uncached loop then runs.
// ---------------------------------------------------------------------------
constexpr int kCacheMaxRow = 256;
template <int NN>
struct CacheCap {
    static constexpr int R = 1024;    // rows per CTA
    static constexpr int E = 6144;    // CSR entries per CTA
};
template <int NN>
struct CacheSmem {
    uint64_t pik[CacheCap<NN>::R * NN];   // confirmed keys per row, descending (0 = empty)
    uint64_t prk[CacheCap<NN>::R * NN];   // this round's proposals (keys; 0 = none)
    uint64_t ek[CacheCap<NN>::E];         // entry keys make_key(a_vj, j); 0 = not an edge
    int64_t rs[CacheCap<NN>::R];          // CSR start of each row
    int32_t gid[CacheCap<NN>::R];
    int32_t rlen[CacheCap<NN>::R];        // CSR row length (live-nnz counter)
    int32_t est[CacheCap<NN>::R];         // first pool entry of each row
    int16_t erow[CacheCap<NN>::E];        // row of each pool entry
    uint8_t esj[CacheCap<NN>::E];         // state byte of the entry's target (this round)
    uint8_t st[CacheCap<NN>::R];          // state byte (degree | charge)
    uint8_t act[CacheCap<NN>::R];         // bit 0: in this round's worklist, bit 1: retired
    int pool, ovf;
    unsigned long long red[3][LF_FUSED_T / 32];
};
template <int NN>
constexpr size_t cache_smem_bytes() { return sizeof(CacheSmem<NN>); }

template <int NN>
__device__ bool rounds_cached(const FusedArgs& f, cg::grid_group& grid) {
    using Cap = CacheCap<NN>;
    constexpr int T = LF_FUSED_T;
    constexpr int RPT = Cap::R / T;   // rows per thread
    constexpr int EPT = Cap::E / T;   // pool entries per thread
    extern __shared__ __align__(16) unsigned char fz_smem[];
    CacheSmem<NN>& S = *reinterpret_cast<CacheSmem<NN>*>(fz_smem);
    const int tid = threadIdx.x;
    const ProposeArgs& pa = f.pa;
#ifdef LF_CACHE_TIMING
    unsigned long long tm[24];
    int ntm = 0;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(tm[ntm++]));
#define CC_MARK() do { __syncthreads(); asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(tm[ntm < 23 ? ntm++ : 23])); } while (0)
#else
#define CC_MARK() do { } while (0)
#endif
    const int L = *(volatile const int32_t*)&f.counts[1];   // round-1 worklist (mutual(0))
    const int C = gridDim.x;
    const int RPC = (L + C - 1) / C;
    const int base = blockIdx.x * RPC;
    const int nmine = max(0, min(L - base, RPC));
    const int32_t* wl1 = f.wl[1];
    if (tid == 0) { S.pool = 0; S.ovf = RPC > Cap::R || f.M > kMaxFlagRounds; }
    __syncthreads();
    // A. own rows: id, state, confirmed keys, row extent
#pragma unroll
    for (int q = 0; q < RPT; q++) {
        const int s = tid + q * T;
        if (s >= nmine || s >= Cap::R) continue;
        const int32_t v = __ldcg(wl1 + base + s);
        const uint8_t stt = __ldcg(f.ma.state + v);
        int32_t pj[NN];
        float pw[NN], pv[NN];
#pragma unroll
        for (int t = 0; t < NN; t++) {
            const int64_t o = (int64_t)v * NN + t;
            pj[t] = f.ma.pi[o];
            pw[t] = f.ma.pi_w[o];
            pv[t] = f.ma.pi_val ? f.ma.pi_val[o] : 0.0f;
        }
        const int64_t r0 = __ldg(pa.rowptr + v), r1 = __ldg(pa.rowptr + v + 1);
        S.gid[s] = v;
        S.st[s] = stt;
        S.act[s] = 1;
        const int deg = stt & ST_DEG;
#pragma unroll
        for (int t = 0; t < NN; t++)
            S.pik[s * NN + t] = t < deg ? make_key_abs(pw[t], __float_as_uint(pv[t]) >> 31, pj[t]) : 0ull;
        const int len = (int)(r1 - r0);
        S.rs[s] = r0;
        S.rlen[s] = len;
        const int off = atomicAdd(&S.pool, len);
        S.est[s] = off;
        if (len > kCacheMaxRow || off + len > Cap::E) S.ovf = 1;
    }
    __syncthreads();
    CC_MARK();
    if (tid == 0 && S.ovf) atomicOr(f.bail, 1);
    grid.sync();
    CC_MARK();
    if (*(volatile int32_t*)f.bail) return false;   // uniform: nothing global written yet
#pragma unroll
    for (int q = 0; q < RPT; q++) {
        const int s = tid + q * T;
        if (s >= nmine) continue;
        const int e0 = S.est[s], len = S.rlen[s];
        for (int e = 0; e < len; e++) S.erow[e0 + e] = (int16_t)s;
    }
    __syncthreads();
    const int P = S.pool;
    // B. the rows' entries as keys (diagonal and zeros -- not edges, L31/L231 -- as key 0)
    {
        int32_t j[EPT];
        float x[EPT];
#pragma unroll
        for (int q = 0; q < EPT; q++) {
            const int p = tid + q * T;
            if (p >= P) continue;
            const int sr = S.erow[p];
            const int64_t e = S.rs[sr] + (p - S.est[sr]);
            j[q] = __ldg(pa.col + e);
            x[q] = __ldg(pa.val + e);
        }
#pragma unroll
        for (int q = 0; q < EPT; q++) {
            const int p = tid + q * T;
            if (p >= P) continue;
            const bool edge = j[q] != S.gid[S.erow[p]] && (__float_as_uint(x[q]) & 0x7FFFFFFFu) != 0u;
            S.ek[p] = edge ? make_key(x[q], j[q]) : 0ull;
        }
    }
    __syncthreads();  // the entry keys
    CC_MARK();
    for (int k = 1; k < f.M; k++) {
        const bool charging = (k % f.m) != f.k_m;
        const bool last = k == f.M - 1;
        // the targets' state bytes (round k), every load of the CTA in flight together
        {
            uint8_t sj[EPT];
#pragma unroll
            for (int q = 0; q < EPT; q++) {
                const int p = tid + q * T;
                sj[q] = (uint8_t)NN;
                if (p >= P) continue;
                const uint64_t key = S.ek[p];
                if (key && (S.act[S.erow[p]] & 1)) sj[q] = __ldcg(f.ma.state + key_col(key));
            }
#pragma unroll
            for (int q = 0; q < EPT; q++) {
                const int p = tid + q * T;
                if (p < P) S.esj[p] = sj[q];
            }
        }
        __syncthreads();  // the targets' states
        CC_MARK();
        // propose (Alg. 2 L13-L22), the tests of propose_phase in its order
        unsigned long long my_live = 0, my_nnz = 0, my_prop = 0;
#pragma unroll
        for (int q = 0; q < RPT; q++) {
            const int s = tid + q * T;
            if (s >= nmine || !(S.act[s] & 1)) continue;
            const uint8_t stt = S.st[s];
            const int deg = stt & ST_DEG;
            const uint32_t cv = (stt & ST_CHARGE) ? 1u : 0u;
            int32_t pc[NN];
#pragma unroll
            for (int t = 0; t < NN; t++) pc[t] = t < deg ? key_col(S.pik[s * NN + t]) : -1;
            uint64_t top[NN];
#pragma unroll
            for (int t = 0; t < NN; t++) top[t] = 0;
            bool theta0 = false;
            const int e0 = S.est[s], e1 = e0 + S.rlen[s];
            for (int e = e0; e < e1; e++) {
                const uint64_t key = S.ek[e];
                if (!key) continue;                              // diagonal / zero
                const uint32_t sj = S.esj[e];
                if ((int)(sj & ST_DEG) == NN) continue;          // saturated (L15)
                const int32_t j = key_col(key);
                bool in_pi = false;
#pragma unroll
                for (int t = 0; t < NN; t++) in_pi |= (pc[t] == j);
                if (in_pi) continue;                             // L19
                theta0 = true;
                if (charging && (((sj & ST_CHARGE) ? 1u : 0u) == cv)) continue;  // L17
                topn_insert<NN>(top, key);
            }
            const int need = NN - deg;
            const int32_t v = S.gid[s];
            int np = 0;
#pragma unroll
            for (int t = 0; t < NN; t++) {
                const uint64_t tk = (t < need) ? top[t] : 0ull;
                S.prk[s * NN + t] = tk;
                pa.prop_j[(int64_t)v * NN + t] = tk ? key_col(tk) : -1;
                np += tk != 0;
            }
            S.act[s] = theta0 ? 1 : 3;
            if (theta0) { my_live += 1; my_nnz += (unsigned long long)S.rlen[s]; }
            my_prop |= (np > 0);
        }
#pragma unroll
        for (int o = 16; o; o >>= 1) {
            my_live += __shfl_xor_sync(0xffffffffu, my_live, o);
            my_nnz += __shfl_xor_sync(0xffffffffu, my_nnz, o);
            my_prop |= __shfl_xor_sync(0xffffffffu, my_prop, o);
        }
        if ((tid & 31) == 0) { S.red[0][tid >> 5] = my_live; S.red[1][tid >> 5] = my_nnz; S.red[2][tid >> 5] = my_prop; }
        __syncthreads();
        if (tid < 32) {
            unsigned long long a0 = tid < T / 32 ? S.red[0][tid] : 0, a1 = tid < T / 32 ? S.red[1][tid] : 0,
                               a2 = tid < T / 32 ? S.red[2][tid] : 0;
#pragma unroll
            for (int o = 16; o; o >>= 1) {
                a0 += __shfl_xor_sync(0xffffffffu, a0, o);
                a1 += __shfl_xor_sync(0xffffffffu, a1, o);
                a2 |= __shfl_xor_sync(0xffffffffu, a2, o);
            }
            if (tid == 0) {
                const int slot = blockIdx.x & 63;
                if (f.live_part && a0) atomicAdd(f.live_part + (size_t)k * 128 + slot, a0);
                if (f.live_part && a1) atomicAdd(f.live_part + (size_t)k * 128 + 64 + slot, a1);
                if (a2) atomicOr(&f.flags[k], 1);
            }
        }
        CC_MARK();
        grid.sync();  // every proposal of round k is visible
        CC_MARK();
        // mutual (Alg. 2 L26-L28): keep w iff v is in prop(w); w proposed this round
#pragma unroll
        for (int q = 0; q < RPT; q++) {
            const int s = tid + q * T;
            if (s >= nmine || !(S.act[s] & 1)) continue;
            const int32_t v = S.gid[s];
            int32_t pw[NN][NN];
#pragma unroll
            for (int u = 0; u < NN; u++) {
                const uint64_t tk = S.prk[s * NN + u];
#pragma unroll
                for (int x = 0; x < NN; x++) pw[u][x] = -1;
                if (!tk) continue;
                const int32_t* q2 = pa.prop_j + (int64_t)key_col(tk) * NN;
#pragma unroll
                for (int x = 0; x < NN; x++) pw[u][x] = __ldcg(q2 + x);
            }
            uint64_t t[NN];
#pragma unroll
            for (int u = 0; u < NN; u++) t[u] = S.pik[s * NN + u];
            int nconf = 0;
#pragma unroll
            for (int u = 0; u < NN; u++) {
                bool mutual = false;
#pragma unroll
                for (int x = 0; x < NN; x++) mutual |= (pw[u][x] == v);
                if (mutual) { topn_insert<NN>(t, S.prk[s * NN + u]); nconf++; }
            }
            int deg = S.st[s] & ST_DEG;
            if (nconf) {
#pragma unroll
                for (int u = 0; u < NN; u++) S.pik[s * NN + u] = t[u];
                deg += nconf;
            }
            if (!last) {
                const bool keep = !(S.act[s] & 2) && deg < NN;
                uint32_t ch = 0;
                if (keep && ((k + 1) % f.m) != f.k_m) ch = charge_bit((uint32_t)v, (uint32_t)(k + 1), f.ma.seed, f.ma.thr);
                const uint8_t ns = (uint8_t)(deg | (ch ? ST_CHARGE : 0));
                S.st[s] = ns;
                f.ma.state[v] = ns;
                S.act[s] = keep ? 1 : 0;
            } else if (nconf) {
                S.st[s] = (uint8_t)deg;
            }
        }
        CC_MARK();
        if (!last) grid.sync();  // round k+1's states visible; round k's proposals consumed
        CC_MARK();
    }
    // write back the rows' factor slots and state
#pragma unroll
    for (int q = 0; q < RPT; q++) {
        const int s = tid + q * T;
        if (s >= nmine) continue;
        const int32_t v = S.gid[s];
#pragma unroll
        for (int u = 0; u < NN; u++) {
            const uint64_t key = S.pik[s * NN + u];
            const int64_t o = (int64_t)v * NN + u;
            f.ma.pi[o] = key ? key_col(key) : -1;
            f.ma.pi_w[o] = key ? key_abs(key) : 0.0f;
            if (f.ma.pi_val) f.ma.pi_val[o] = key ? key_val(key) : 0.0f;
        }
        f.ma.state[v] = S.st[s];
    }
    // every CTA's counters of the last round were added before the last barrier
    if (blockIdx.x == 0 && (f.rounds || f.live))
        finalize_body(f.flags, f.M, f.m, f.k_m, f.rounds, f.live_part, f.live);
#ifdef LF_CACHE_TIMING
    CC_MARK();
    if (tid == 0 && (blockIdx.x == 0 || blockIdx.x == 100)) {
        printf("cached blk %d L=%d nmine=%d P=%d:", blockIdx.x, L, nmine, P);
        for (int i = 1; i < ntm; i++) printf(" %llu", tm[i] - tm[i - 1]);
        printf("\n");
    }
#endif
    return true;
}

static bool cached_rounds_enabled() { return getenv("LF_NO_CACHED_ROUNDS") == nullptr; }

// Rounds 1..M-1, step 1: the cached mode (small live sets).  When the round-1 worklist does
// not fit (or the mode is disabled) the kernel only raises the bail flag, and the rows-mode
// kernel k_rounds_rows that follows it on the stream runs the rounds instead.
template <int NN>
__global__ void __launch_bounds__(LF_FUSED_T) k_rounds_fused(FusedArgs f) {
    LF_TL(g_tl_factor, 3);
    pdl_trigger();  // k_rounds_rows may launch and wait meanwhile
    cg::grid_group grid = cg::this_grid();
    if (f.cached && rounds_cached<NN>(f, grid)) return;
    if (!f.cached && blockIdx.x == 0 && threadIdx.x == 0) *f.bail = 1;
}

// ---------------------------------------------------------------------------
// Rows mode of rounds 1..M-1 (live sets too large for the cached mode: C2 with n = 1, 3,
// C3, C4, C5).  The rows still live at a round's start carry ST_LIVE in their state byte
// (set by the previous mutual phase for exactly the rows the worklist would hold), and
// every phase streams the rows in natural order, skipping the others after one coalesced
// state load: neighbouring rows' entries are adjacent in HBM and their targets' state
// bytes are L2-local, instead of the worklist's scattered order and its extra dependent
// load.  One cooperative kernel at full occupancy (the cached mode needs one CTA per SM);
// per round: propose | long rows (a CTA per row) | mutual, separated by grid barriers.
// Semantics per row are those of propose_phase / mutual_phase (same tests, same order,
// same keys), so the factor is bit-identical.
// ---------------------------------------------------------------------------
struct RowsArgs {
    int64_t N;
    const int64_t* __restrict__ rowptr;
    const int32_t* __restrict__ col;
    const float* __restrict__ val;
    uint8_t* __restrict__ state;
    int32_t* __restrict__ pi;
    float* __restrict__ pi_w;
    float* __restrict__ pi_val;
    int32_t* __restrict__ prop_j;
    float* __restrict__ prop_v;
    int* flags;
    unsigned long long* live_part;   // NULL: no counters
    int32_t* long_rows;
    int32_t* long_count;             // [kMaxFlagRounds]
    int64_t defer_len;
    int M, m, k_m;
    uint32_t seed;
    unsigned long long thr;
    const int32_t* bail;             // the cached mode's flag: 0 = it already ran the rounds
    int32_t* rounds;
    int64_t* live;
    int only_k, only_phase;          // > 0: run only phase only_phase (0 propose, 1 long rows,
                                     // 2 mutual) of round only_k (per-phase profiling launches)
    int32_t* wl[2];                  // worklists: round k's live rows in wl[k & 1] (mutual(k-1)
    int32_t* counts;                 //   appends them, roughly in id order), sizes counts[k % 3]
    int64_t row_base;                // partitioned runs: CSR row of vertex v is v - row_base,
    int64_t gid_off;                 //   its global id (charges) v + gid_off; NULL bail = always run
};
constexpr int kRowsT = 4;  // entries per lane per pass (loads in flight per lane)

// top-NN proposal of one row by the G lanes of a group (lane index li), entries [rs, re):
// the eligibility tests of propose_phase in its order; returns the merged list in top
template <int NN, int G>
__device__ __forceinline__ void row_topn(const RowsArgs& a, int32_t v, int64_t rs, int64_t re, int li,
                                         const int32_t (&p)[NN], uint32_t cv, bool charging,
                                         uint64_t (&top)[NN], uint32_t& theta0) {
#pragma unroll
    for (int s = 0; s < NN; s++) top[s] = 0;
    theta0 = 0;
    for (int64_t b = rs; b < re; b += G * kRowsT) {
        int32_t j[kRowsT];
        uint32_t xb[kRowsT];
#pragma unroll
        for (int t = 0; t < kRowsT; t++) {
            const int64_t e = b + li + t * G;
            const bool in = e < re;
            j[t] = in ? __ldg(a.col + e) : v;
            xb[t] = in ? __float_as_uint(__ldg(a.val + e)) : 0u;
        }
        uint32_t sj[kRowsT];
#pragma unroll
        for (int t = 0; t < kRowsT; t++) {
            const bool edge = j[t] != v && (xb[t] & 0x7FFFFFFFu) != 0u;  // A' = |A| - diag, zeros (L31, L231)
            sj[t] = edge ? (a.state ? (uint32_t)__ldcg(a.state + j[t]) : 0u) : (uint32_t)NN;
        }
#pragma unroll
        for (int t = 0; t < kRowsT; t++) {
            if ((int)(sj[t] & ST_DEG) == NN) continue;  // not an edge, or j saturated (L15)
            bool in_pi = false;
#pragma unroll
            for (int s = 0; s < NN; s++) in_pi |= (p[s] == j[t]);
            if (in_pi) continue;  // L19: W \ pi(v)
            theta0 = 1;
            if (charging && (((sj[t] & ST_CHARGE) ? 1u : 0u) == cv)) continue;  // L17
            topn_insert<NN>(top, ((uint64_t)(xb[t] & 0x7FFFFFFFu) << 32) |
                                     (((0x7FFFFFFFu - (uint32_t)j[t]) << 1) | (xb[t] >> 31)));
        }
    }
    topn_merge_group<NN, G>(top);
#pragma unroll
    for (int off = G / 2; off >= 1; off >>= 1) theta0 |= __shfl_xor_sync(0xffffffffu, theta0, off);
}

template <int NN>
__device__ __forceinline__ void write_prop(const RowsArgs& a, int32_t v, int deg, const uint64_t (&top)[NN],
                                           uint32_t theta0, int& np) {
    const int need = NN - deg;
    np = 0;
#pragma unroll
    for (int s = 0; s < NN; s++) {
        const uint64_t tk = s < need ? top[s] : 0ull;
        a.prop_j[(int64_t)v * NN + s] = tk ? key_col(tk) : ((s == 0 && !theta0) ? PROP_RETIRED : -1);
        a.prop_v[(int64_t)v * NN + s] = tk ? key_val(tk) : 0.0f;
        np += tk != 0;
    }
}

// propose (Alg. 2 L13-L22) of round k over its worklist (the rows still live, appended by
// the previous mutual phase roughly in id order), one row per lane.  A warp takes 32
// worklist entries, loads their state, row extent and confirmed slots (one round trip; the
// next 32 entries' ids are already in flight) and queues the rows in shared memory; every
// batch of queued rows whose aligned ranges fit the warp's slice is staged with 16-byte
// cp.async (all rows in flight), then every entry's target state word is fetched with a
// 4-byte cp.async (all in flight), then each lane reduces its row from shared memory with
// the tests of propose_phase and a branch-free top-n network.
#ifndef LF_ROWS_T
#define LF_ROWS_T 256
#endif
#ifndef LF_ROWS_BUD
#define LF_ROWS_BUD 640
#endif
constexpr int kRowsBud = LF_ROWS_BUD;  // staged entries per warp (640: 3 CTAs of 8 warps per SM)
constexpr int kRowsWarps = LF_ROWS_T / 32;
template <int BUD, int NQ = 4>
struct RowsWarpSmemT {
    int32_t col[BUD];
    uint32_t val[BUD];
    uint32_t sjw[BUD];  // the 4-byte state word holding byte col & 3
    int64_t qrs[64];      // queue of live rows: CSR start
    int32_t qv[64];       //   vertex
    int32_t qlen[64];     //   entries
    int32_t qp[64][NQ];   //   confirmed slots
    uint8_t qst[64];      //   state byte
};
using RowsWarpSmem = RowsWarpSmemT<kRowsBud>;
struct RowsSmem {
    RowsWarpSmem w[kRowsWarps];
};
// the per-round propose kernel of large graphs: 4 warps per CTA, whole 32-row batches; the
// queue keeps n confirmed slots per row, so that 4 CTAs (16 warps) fit an SM for n <= 2
// (with 4 slots: 3 CTAs, 12 warps)
#ifndef LF_ROWSK_BUD
#define LF_ROWSK_BUD 1024
#endif
constexpr int kRowsBudK = LF_ROWSK_BUD, kRowsTK = 128;
template <int NN>
struct RowsSmemK {
    RowsWarpSmemT<kRowsBudK, NN> w[kRowsTK / 32];
};

// one batch: the longest prefix of the queue whose aligned ranges fit; returns its size
template <int NN, int BUD, int NQ>
__device__ __forceinline__ int rows_batch(const RowsArgs& a, RowsWarpSmemT<BUD, NQ>& S, int qcnt, bool charging,
                                          bool bulk_ok, int64_t nnz, unsigned long long& my_live,
                                          unsigned long long& my_nnz, int& my_prop) {
    const int lane = threadIdx.x & 31;
    const bool has = lane < qcnt;
    int64_t rs = 0;
    int len = 0;
    if (has) { rs = S.qrs[lane]; len = S.qlen[lane]; }
    const int64_t as = rs & ~(int64_t)3, ae = (rs + len + 3) & ~(int64_t)3;
    const int plen = has ? (int)(ae - as) : 0;
    int incl = plen;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int y = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += y;
    }
    const bool take = has && incl <= BUD;
    const int nb = __popc(__ballot_sync(0xffffffffu, take));
    const int boff = incl - plen;
    const int q0 = boff + (int)(rs - as), q1 = q0 + len;
    if (take) {  // stage the row (16-byte copies of its aligned range, else per entry)
        if (bulk_ok && ae <= nnz) {
            for (int c = 0; c < plen; c += 4) {
                cp16(&S.col[boff + c], a.col + as + c);
                cp16(&S.val[boff + c], a.val + as + c);
            }
        } else {
            for (int e = 0; e < len; e++) {
                cp4(&S.col[q0 + e], a.col + rs + e);
                cp4(&S.val[q0 + e], a.val + rs + e);
            }
        }
    }
    cp_commit();
    cp_wait_all();
    __syncwarp();
    if (take) {  // the targets' state words (L15/L17), every entry's copy in flight
        for (int q = q0; q < q1; q++) cp4(&S.sjw[q], a.state + (S.col[q] & ~3));
    }
    cp_commit();
    cp_wait_all();
    __syncwarp();
    if (take) {
        const int32_t v = S.qv[lane];
        const uint32_t sv = S.qst[lane];
        int32_t p[NN];
#pragma unroll
        for (int s2 = 0; s2 < NN; s2++) p[s2] = S.qp[lane][s2];
        const uint32_t cv = (sv & ST_CHARGE) ? 1u : 0u;
        uint64_t top[NN];
#pragma unroll
        for (int s2 = 0; s2 < NN; s2++) top[s2] = 0;
        uint32_t theta0 = 0;
        for (int q = q0; q < q1; q++) {
            const int32_t j = S.col[q];
            const uint32_t xb = S.val[q];
            const uint32_t sj = (S.sjw[q] >> (8 * (j & 3))) & 0xffu;
            bool in_pi = false;
#pragma unroll
            for (int s2 = 0; s2 < NN; s2++) in_pi |= (p[s2] == j);
            // A' = |A| - diag and zeros (L31, L231); j saturated (L15); W \ pi(v) (L19)
            const bool elig = j != v && (xb & 0x7FFFFFFFu) != 0u && (int)(sj & ST_DEG) != NN && !in_pi;
            theta0 |= elig ? 1u : 0u;
            const bool ok = elig && !(charging && (((sj & ST_CHARGE) ? 1u : 0u) == cv));  // L17
            topn_insert_pred<NN>(top, ((uint64_t)(xb & 0x7FFFFFFFu) << 32) |
                                          (((0x7FFFFFFFu - (uint32_t)j) << 1) | (xb >> 31)), ok);
        }
        int np;
        write_prop<NN>(a, v, sv & ST_DEG, top, theta0, np);
        if (theta0) { my_live++; my_nnz += (unsigned long long)len; }
        my_prop |= np > 0;
    }
    __syncwarp();
    // drop the batch from the queue (slots nb..qcnt-1 move down)
    int64_t mrs[2];
    int32_t mv[2], ml[2], mp[2][NN];
    uint8_t mst[2];
#pragma unroll
    for (int h = 0; h < 2; h++) {
        const int src = nb + lane + 32 * h;
        if (src < qcnt) {
            mrs[h] = S.qrs[src]; mv[h] = S.qv[src]; ml[h] = S.qlen[src]; mst[h] = S.qst[src];
#pragma unroll
            for (int s2 = 0; s2 < NN; s2++) mp[h][s2] = S.qp[src][s2];
        }
    }
    __syncwarp();
#pragma unroll
    for (int h = 0; h < 2; h++) {
        const int src = nb + lane + 32 * h;
        if (src < qcnt) {
            const int d = lane + 32 * h;
            S.qrs[d] = mrs[h]; S.qv[d] = mv[h]; S.qlen[d] = ml[h]; S.qst[d] = mst[h];
#pragma unroll
            for (int s2 = 0; s2 < NN; s2++) S.qp[d][s2] = mp[h][s2];
        }
    }
    __syncwarp();
    return nb;
}

template <int NN, int G, int BUD, int NQ = 4>
__device__ __forceinline__ void rows_propose(const RowsArgs& a, int k, bool charging, RowsWarpSmemT<BUD, NQ>& S) {
    const int lane = threadIdx.x & 31;
    const int64_t wg = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const int64_t nnz = __ldg(a.rowptr + a.N);
    const bool bulk_ok = ((((uintptr_t)a.col) | ((uintptr_t)a.val)) & 15) == 0;
    const int32_t* __restrict__ wl = a.wl[k & 1];
    const int64_t cnt = __ldcg(a.counts + k % 3);
    unsigned long long my_live = 0, my_nnz = 0;
    int my_prop = 0;
    int qcnt = 0;
    // a two-deep software pipeline over the worklist: the next 32 rows' state, row extent and
    // confirmed slots are loaded while this iteration's batches run (the loads only block at
    // the loop's back edge), and the ids after them are in flight as well
    auto fetch = [&](int32_t v, uint32_t& st, int64_t& rs, int64_t& re, int32_t (&p)[NN]) {
        st = 0;
        rs = re = 0;
#pragma unroll
        for (int s2 = 0; s2 < NN; s2++) p[s2] = -1;
        if (v >= 0) {  // live: deg < n, so pi's unused slots hold -1
            st = __ldcg(a.state + v);
            rs = __ldg(a.rowptr + (v - a.row_base));
            re = __ldg(a.rowptr + (v - a.row_base) + 1);
#pragma unroll
            for (int s2 = 0; s2 < NN; s2++) p[s2] = __ldcg(a.pi + (int64_t)v * NN + s2);
        }
    };
    int64_t i0 = wg * 32;
    int32_t vc = (i0 + lane < cnt) ? __ldcg(wl + i0 + lane) : -1;
    int32_t vn = (i0 + nw * 32 + lane < cnt) ? __ldcg(wl + i0 + nw * 32 + lane) : -1;
    uint32_t stc;
    int64_t rsc, rec;
    int32_t pc[NN];
    fetch(vc, stc, rsc, rec, pc);
    for (; i0 < cnt; i0 += nw * 32) {
        const int32_t v = vc;
        const bool valid = v >= 0;
        const uint32_t st = stc;
        const int64_t rs = rsc, re = rec;
        int32_t p[NN];
#pragma unroll
        for (int s2 = 0; s2 < NN; s2++) p[s2] = pc[s2];
        // the next iteration's rows (ids already here) and the ids after them
        const int64_t i2 = i0 + 2 * nw * 32;
        const int32_t vnn = (i2 + lane < cnt) ? __ldcg(wl + i2 + lane) : -1;
        fetch(vn, stc, rsc, rec, pc);
        vc = vn;
        vn = vnn;
        const bool lng = valid && (re - rs) > a.defer_len;
        {   // long rows: a CTA per row after the barrier
            const unsigned m = __ballot_sync(0xffffffffu, lng);
            if (m) {
                int base = 0;
                if (lane == 0) base = atomicAdd(&a.long_count[k], __popc(m));
                base = __shfl_sync(0xffffffffu, base, 0);
                if (lng) a.long_rows[base + __popc(m & ((1u << lane) - 1u))] = v;
            }
        }
        const bool enq = valid && !lng;
        const unsigned m = __ballot_sync(0xffffffffu, enq);
        if (enq) {
            const int pos = qcnt + __popc(m & ((1u << lane) - 1u));
            S.qrs[pos] = rs;
            S.qv[pos] = v;
            S.qlen[pos] = (int)(re - rs);
            S.qst[pos] = (uint8_t)st;
#pragma unroll
            for (int s2 = 0; s2 < NN; s2++) S.qp[pos][s2] = p[s2];
        }
        qcnt += __popc(m);
        __syncwarp();
        while (qcnt >= 32) qcnt -= rows_batch<NN, BUD, NQ>(a, S, qcnt, charging, bulk_ok, nnz, my_live, my_nnz, my_prop);
    }
    while (qcnt > 0) qcnt -= rows_batch<NN, BUD, NQ>(a, S, qcnt, charging, bulk_ok, nnz, my_live, my_nnz, my_prop);
#pragma unroll
    for (int off = 16; off >= 1; off >>= 1) {
        my_live += __shfl_xor_sync(0xffffffffu, my_live, off);
        my_nnz += __shfl_xor_sync(0xffffffffu, my_nnz, off);
        my_prop |= __shfl_xor_sync(0xffffffffu, my_prop, off);
    }
    if (lane == 0) {
        const int slot = (int)(wg & 63);
        if (a.live_part && my_live) atomicAdd(a.live_part + (size_t)k * 128 + slot, my_live);
        if (a.live_part && my_nnz) atomicAdd(a.live_part + (size_t)k * 128 + 64 + slot, my_nnz);
        if (my_prop && *(volatile int*)&a.flags[k] == 0) atomicOr(&a.flags[k], 1);
    }
}

// one long row per CTA (hub rows of power-law graphs): the CTA's threads stride the row,
// warps merge their lists with shuffles, warp 0 merges the warps' lists
template <int NN>
__device__ __forceinline__ void block_row_topn(const RowsArgs& a, int32_t v, int64_t rs, int64_t re, const int32_t (&p)[NN],
                               uint32_t cv, bool charging, uint64_t (&top)[NN], uint32_t& theta0) {
    __shared__ uint64_t wk[32][NN];
    __shared__ uint32_t wth[32];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nwarp = blockDim.x >> 5;
    uint64_t t[NN];
    uint32_t th = 0;
#pragma unroll
    for (int s = 0; s < NN; s++) t[s] = 0;
    for (int64_t b = rs + w * 32 * kRowsT; b < re; b += (int64_t)blockDim.x * kRowsT) {
        uint64_t tt[NN];
        uint32_t th2;
        row_topn<NN, 32>(a, v, b, (b + 32 * kRowsT < re ? b + 32 * kRowsT : re), lane, p, cv, charging, tt, th2);
        th |= th2;
#pragma unroll
        for (int s = 0; s < NN; s++) topn_insert<NN>(t, tt[s]);
    }
    if (lane == 0) {
#pragma unroll
        for (int s = 0; s < NN; s++) wk[w][s] = t[s];
        wth[w] = th;
    }
    __syncthreads();
#pragma unroll
    for (int s = 0; s < NN; s++) top[s] = 0;
    theta0 = 0;
    for (int q = 0; q < nwarp; q++) {
#pragma unroll
        for (int s = 0; s < NN; s++) topn_insert<NN>(top, wk[q][s]);
        theta0 |= wth[q];
    }
    __syncthreads();  // wk reused by the next row
}

template <int NN>
__device__ __forceinline__ void rows_long(const RowsArgs& a, int k, bool charging) {
    const int cnt = *(volatile int32_t*)&a.long_count[k];
    unsigned long long my_live = 0, my_nnz = 0;
    int my_prop = 0;
    for (int i = blockIdx.x; i < cnt; i += gridDim.x) {
        const int32_t v = __ldcg(a.long_rows + i);
        const uint32_t sv = __ldcg(a.state + v);
        const int64_t rs = __ldg(a.rowptr + (v - a.row_base)), re = __ldg(a.rowptr + (v - a.row_base) + 1);
        const int deg = sv & ST_DEG;
        int32_t p[NN];
#pragma unroll
        for (int s = 0; s < NN; s++) p[s] = deg > 0 ? __ldcg(a.pi + (int64_t)v * NN + s) : -1;
        uint64_t top[NN];
        uint32_t theta0;
        block_row_topn<NN>(a, v, rs, re, p, (sv & ST_CHARGE) ? 1u : 0u, charging, top, theta0);
        if (threadIdx.x == 0) {
            int np;
            write_prop<NN>(a, v, deg, top, theta0, np);
            if (theta0) { my_live++; my_nnz += (unsigned long long)(re - rs); }
            my_prop |= np > 0;
        }
    }
    if (threadIdx.x == 0) {
        const int slot = blockIdx.x & 63;
        if (a.live_part && my_live) atomicAdd(a.live_part + (size_t)k * 128 + slot, my_live);
        if (a.live_part && my_nnz) atomicAdd(a.live_part + (size_t)k * 128 + 64 + slot, my_nnz);
        if (my_prop && *(volatile int*)&a.flags[k] == 0) atomicOr(&a.flags[k], 1);
    }
}

// mutual (Alg. 2 L26-L28) of round k over its worklist, MB rows per thread in flight; the
// rows that stay live are appended to round k+1's worklist (one atomic per warp)
template <int NN, int MB>
__device__ __forceinline__ void rows_mutual(const RowsArgs& a, int k, bool last) {
    const int64_t chunk = (int64_t)blockDim.x * MB;
    const bool next_charging = ((k + 1) % a.m) != a.k_m;
    const int32_t* __restrict__ wl = a.wl[k & 1];
    int32_t* wn = a.wl[(k + 1) & 1];
    int32_t* cn = a.counts + (k + 1) % 3;
    const int64_t cnt = __ldcg(a.counts + k % 3);
    if (!last && blockIdx.x == 0 && threadIdx.x == 0) a.counts[(k + 2) % 3] = 0;  // round k+2's appends
    const int lane = threadIdx.x & 31;
    for (int64_t c0 = (int64_t)blockIdx.x * chunk; c0 < cnt; c0 += (int64_t)gridDim.x * chunk) {
        int32_t vv[MB];
        uint32_t st[MB];
        int32_t pj[MB][NN], pw[MB][NN][NN];
#pragma unroll
        for (int b = 0; b < MB; b++) {
            const int64_t i = c0 + threadIdx.x + (int64_t)b * blockDim.x;
            vv[b] = i < cnt ? __ldcg(wl + i) : -1;
        }
#pragma unroll
        for (int b = 0; b < MB; b++) {
            st[b] = vv[b] >= 0 ? (uint32_t)__ldcg(a.state + vv[b]) : 0u;
#pragma unroll
            for (int s = 0; s < NN; s++) pj[b][s] = vv[b] >= 0 ? __ldcg(a.prop_j + (int64_t)vv[b] * NN + s) : -1;
        }
#pragma unroll
        for (int b = 0; b < MB; b++)
#pragma unroll
            for (int s = 0; s < NN; s++)
#pragma unroll
                for (int t = 0; t < NN; t++)
                    pw[b][s][t] = pj[b][s] >= 0 ? __ldcg(a.prop_j + (int64_t)pj[b][s] * NN + t) : -1;
        bool keepb[MB];
#pragma unroll
        for (int b = 0; b < MB; b++) {
            keepb[b] = false;
            const int32_t v32 = vv[b];
            if (v32 < 0) continue;
            const int64_t v = v32;
            uint64_t conf[NN];
            int nconf = 0;
#pragma unroll
            for (int s = 0; s < NN; s++) {
                conf[s] = 0;
                bool mutual = false;
#pragma unroll
                for (int t = 0; t < NN; t++) mutual |= (pw[b][s][t] == v32);
                if (pj[b][s] >= 0 && mutual) {
                    conf[s] = make_key(__ldcg(a.prop_v + v * NN + s), pj[b][s]);
                    nconf++;
                }
            }
            int deg = st[b] & ST_DEG;
            if (nconf > 0) {
                uint64_t t[NN];
#pragma unroll
                for (int s = 0; s < NN; s++) {
                    t[s] = 0;
                    if (s < deg) {
                        const int64_t o = v * NN + s;
                        const uint32_t sg = a.pi_val ? (__float_as_uint(a.pi_val[o]) >> 31) : 0u;
                        t[s] = make_key_abs(a.pi_w[o], sg, a.pi[o]);
                    }
                }
#pragma unroll
                for (int s = 0; s < NN; s++)
                    if (conf[s]) topn_insert<NN>(t, conf[s]);
#pragma unroll
                for (int s = 0; s < NN; s++) {
                    const int64_t o = v * NN + s;
                    a.pi[o] = t[s] ? key_col(t[s]) : -1;
                    a.pi_w[o] = t[s] ? key_abs(t[s]) : 0.0f;
                    if (a.pi_val) a.pi_val[o] = t[s] ? key_val(t[s]) : 0.0f;
                }
                deg += nconf;
            }
            uint32_t ns = (uint32_t)deg;
            if (!last) {
                keepb[b] = pj[b][0] != PROP_RETIRED && deg < NN;
                if (keepb[b]) {
                    ns |= ST_LIVE;
                    if (next_charging && charge_bit((uint32_t)(v + a.gid_off), (uint32_t)(k + 1), a.seed, a.thr)) ns |= ST_CHARGE;
                }
            }
            if (ns != st[b]) a.state[v] = (uint8_t)ns;
        }
        if (!last) {  // one worklist atomic per CTA for all MB row batches
            unsigned m[MB];
            int tot = 0;
#pragma unroll
            for (int b = 0; b < MB; b++) { m[b] = __ballot_sync(0xffffffffu, keepb[b]); tot += __popc(m[b]); }
            int32_t basepos = block_append_base(tot, cn);
#pragma unroll
            for (int b = 0; b < MB; b++) {
                if (keepb[b]) wn[basepos + __popc(m[b] & ((1u << lane) - 1u))] = vv[b];
                basepos += __popc(m[b]);
            }
        }
    }
}

template <int NN, int G>
__global__ void __launch_bounds__(LF_ROWS_T, 3) k_rounds_rows(RowsArgs a) {
    LF_TL(g_tl_factor, 4);
    extern __shared__ __align__(16) unsigned char rows_smem[];
    RowsWarpSmem& S = reinterpret_cast<RowsSmem*>(rows_smem)->w[threadIdx.x >> 5];
    pdl_wait();
    if (a.bail && *(volatile const int32_t*)a.bail == 0) return;  // the cached mode ran the rounds
    if (a.only_k > 0) {
        const int k = a.only_k;
        const bool charging = (k % a.m) != a.k_m;
        const bool last = k == a.M - 1;
        if (a.only_phase == 0) rows_propose<NN, G, kRowsBud>(a, k, charging, S);
        if (a.only_phase == 1 && *(volatile int32_t*)&a.long_count[k] > 0) rows_long<NN>(a, k, charging);
        if (a.only_phase == 2) {
            if (last && blockIdx.x == 0 && (a.rounds || a.live))
                finalize_body(a.flags, a.M, a.m, a.k_m, a.rounds, a.live_part, a.live);
            rows_mutual<NN, 2>(a, k, last);
        }
        return;
    }
    cg::grid_group grid = cg::this_grid();
    for (int k = 1; k < a.M; k++) {
        const bool charging = (k % a.m) != a.k_m;
        const bool last = k == a.M - 1;
        rows_propose<NN, G, kRowsBud>(a, k, charging, S);
        grid.sync();
        if (*(volatile int32_t*)&a.long_count[k] > 0) {
            rows_long<NN>(a, k, charging);
            grid.sync();
        }
        if (last && blockIdx.x == 0 && (a.rounds || a.live))
            finalize_body(a.flags, a.M, a.m, a.k_m, a.rounds, a.live_part, a.live);
        rows_mutual<NN, 2>(a, k, last);
        if (!last) grid.sync();
    }
}

// Deferred long rows of a per-round propose (hub rows of power-law graphs; C4's reach 44 k
// entries): a CTA per row instead of a warp, with propose_phase's semantics for one row
// (round 0 also captures the diagonal; state / pi may be NULL in a fresh round 0).
template <int NN>
__global__ void __launch_bounds__(256) k_propose_long_blk(ProposeArgs pa) {
    LF_TL(g_tl_factor, 7);
    pdl_wait();
    pdl_trigger();
    const int cnt = *(volatile const int32_t*)pa.wl_count;
    RowsArgs ra;
    memset(&ra, 0, sizeof(ra));
    ra.col = pa.col;
    ra.val = pa.val;
    ra.state = const_cast<uint8_t*>(pa.state);
    unsigned long long my_live = 0, my_nnz = 0;
    int my_prop = 0;
    for (int i = blockIdx.x; i < cnt; i += gridDim.x) {
        const int32_t v = __ldcg(pa.wl + i);
        const int64_t row = (int64_t)v - pa.row_base;
        const int64_t rs = __ldg(pa.rowptr + row), re = __ldg(pa.rowptr + row + 1);
        const uint32_t sv = pa.state ? (uint32_t)__ldcg(pa.state + v) : 0u;
        const int deg = sv & ST_DEG;
        int32_t p[NN];
#pragma unroll
        for (int s2 = 0; s2 < NN; s2++) p[s2] = (pa.pi && deg > 0) ? __ldcg(pa.pi + (int64_t)v * NN + s2) : -1;
        if (pa.diag) {  // the diagonal entry (L231: not an edge), at most one per row
            for (int64_t e = rs + threadIdx.x; e < re; e += blockDim.x)
                if (__ldg(pa.col + e) == v) pa.diag[v] = __ldg(pa.val + e);
        }
        uint64_t top[NN];
        uint32_t theta0;
        block_row_topn<NN>(ra, v, rs, re, p, (sv & ST_CHARGE) ? 1u : 0u, pa.charging != 0, top, theta0);
        if (threadIdx.x == 0) {
            const int need = NN - deg;
            int np = 0;
#pragma unroll
            for (int s2 = 0; s2 < NN; s2++) {
                const uint64_t tk = s2 < need ? top[s2] : 0ull;
                pa.prop_j[(int64_t)v * NN + s2] = tk ? key_col(tk) : ((s2 == 0 && !theta0) ? PROP_RETIRED : -1);
                pa.prop_v[(int64_t)v * NN + s2] = tk ? key_val(tk) : 0.0f;
                np += tk != 0;
            }
            if (theta0) { my_live++; my_nnz += (unsigned long long)(re - rs); }
            my_prop |= np > 0;
        }
    }
    if (threadIdx.x == 0) {
        const int slot = blockIdx.x & 63;
        if (pa.live_rows && my_live) atomicAdd(pa.live_rows + slot, my_live);
        if (pa.live_nnz && my_nnz) atomicAdd(pa.live_nnz + slot, my_nnz);
        if (my_prop && *(volatile int*)pa.proposed == 0) atomicOr(pa.proposed, 1);
    }
}

// Rows mode of large graphs as three kernels per round (propose | long rows | mutual): the
// propose kernel runs 4-warp CTAs with whole 32-row batches in shared memory, the mutual
// kernel needs no shared memory and runs at full occupancy with 4 rows per thread in
// flight -- one cooperative kernel would hold both at the propose kernel's occupancy.
template <int NN>
__global__ void __launch_bounds__(kRowsTK) k_rows_propose_k(RowsArgs a) {
    LF_TL(g_tl_factor, 5);
    extern __shared__ __align__(16) unsigned char rows_smem_k[];
    auto& S = reinterpret_cast<RowsSmemK<NN>*>(rows_smem_k)->w[threadIdx.x >> 5];
    pdl_wait();
    if (a.bail && *(volatile const int32_t*)a.bail == 0) return;  // the cached mode ran the rounds
    rows_propose<NN, 1, kRowsBudK, NN>(a, a.only_k, (a.only_k % a.m) != a.k_m, S);
}
template <int NN>
__global__ void __launch_bounds__(256) k_rows_long_k(RowsArgs a) {
    pdl_wait();
    if (a.bail && *(volatile const int32_t*)a.bail == 0) return;
    if (*(volatile int32_t*)&a.long_count[a.only_k] > 0) rows_long<NN>(a, a.only_k, (a.only_k % a.m) != a.k_m);
}
template <int NN>
#ifndef LF_RMUT_MINB
#define LF_RMUT_MINB 1
#endif
#ifndef LF_RMUT_MB
#define LF_RMUT_MB 2  // rows in flight per thread (C5 rounds 1-4: 2 -> 6.86 ms, 4 -> 7.09 ms)
#endif
__global__ void __launch_bounds__(256, LF_RMUT_MINB) k_rows_mutual_k(RowsArgs a) {
    LF_TL(g_tl_factor, 6);
    pdl_wait();
    if (a.bail && *(volatile const int32_t*)a.bail == 0) return;
    const int k = a.only_k;
    const bool last = k == a.M - 1;
    if (last && blockIdx.x == 0 && (a.rounds || a.live))
        finalize_body(a.flags, a.M, a.m, a.k_m, a.rounds, a.live_part, a.live);
    rows_mutual<NN, LF_RMUT_MB>(a, k, last);
}

// state of round 0 when round 0 is charged (k_m != 0): degree 0 + charge(v, 0)
__global__ void k_init_state(int64_t NL, uint8_t* state, uint32_t seed, unsigned long long thr,
                             const int32_t* __restrict__ l2g) {
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < NL;
         v += (int64_t)gridDim.x * blockDim.x) {
        const uint32_t g = l2g ? (uint32_t)l2g[v] : (uint32_t)v;
        state[v] = charge_bit(g, 0u, seed, thr) ? ST_CHARGE : 0;
    }
}

// diagonal only (M = 0: no round streams the rows)
__global__ void k_diag(int64_t N, const int64_t* __restrict__ rowptr, const int32_t* __restrict__ col,
                       const float* __restrict__ val, float* diag, int64_t row_base) {
    for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < N;
         r += (int64_t)gridDim.x * blockDim.x) {
        const int32_t v = (int32_t)(row_base + r);
        float d = 0.0f;
        for (int64_t e = rowptr[r]; e < rowptr[r + 1]; e++)
            if (col[e] == v) d = val[e];
        diag[v] = d;
    }
}

// ---------------------------------------------------------------------------
// host side
// ---------------------------------------------------------------------------

template <int NN>
static void launch_propose(int G, const ProposeArgs& pa, int grid, cudaStream_t s) {
    switch (G) {
        case 1: k_propose<NN, 1><<<grid, 256, 0, s>>>(pa); break;
        case 2: k_propose<NN, 2><<<grid, 256, 0, s>>>(pa); break;
        case 4: k_propose<NN, 4><<<grid, 256, 0, s>>>(pa); break;
        case 8: k_propose<NN, 8><<<grid, 256, 0, s>>>(pa); break;
        case 16: k_propose<NN, 16><<<grid, 256, 0, s>>>(pa); break;
        default: k_propose<NN, 32><<<grid, 256, 0, s>>>(pa); break;
    }
}

template <int NN, int G, bool CH, int SE, int T = SPT>
static void launch_stream_one(const ProposeArgs& pa, cudaStream_t s) {
    static bool attr = false;
    const int smem = (int)sizeof(StreamSmem<SE>);
    if (!attr) {
        cudaFuncSetAttribute((const void*)k_propose_stream<NN, G, CH, SE, T>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
        attr = true;
    }
    const int grid = persistent_grid((const void*)k_propose_stream<NN, G, CH, SE, T>, T, smem);
    k_propose_stream<NN, G, CH, SE, T><<<grid, T, smem, s>>>(pa);
}

// G lanes per row and the stage size: (1, SETILE) for sparse rows (C1, C2), one lane per row
// with big stages up to 32 entries per row (C3-C5: no merge shuffles; 9.5 -> 6.0 ms on C5),
// then 2 and 8 lanes
template <int NN, bool CH>
static void launch_stream_g(int G, const ProposeArgs& pa, cudaStream_t s) {
    switch (G) {
        case 0: launch_stream_one<NN, 1, CH, SETILE>(pa, s); break;
        // 128 threads with 4096-entry stages: 3 CTAs per SM instead of one (C5: 6.0 -> 5.5 ms,
        // 91% of the measured copy peak; C3 0.061 -> 0.053 ms)
        case 1: launch_stream_one<NN, 1, CH, kSetileBig / 2, 128>(pa, s); break;
        case 2: launch_stream_one<NN, 2, CH, kSetileBig>(pa, s); break;
        case 3: launch_stream_one<NN, 2, CH, SETILE>(pa, s); break;
        default: launch_stream_one<NN, 8, CH, kSetileBig>(pa, s); break;
    }
}

template <int NN>
static void launch_propose_stream(int G, const ProposeArgs& pa, cudaStream_t s) {
    if (pa.N == 0) return;
    if (pa.charging) launch_stream_g<NN, true>(G, pa, s);
    else launch_stream_g<NN, false>(G, pa, s);
}

template <int NN>
static void launch_propose_tile(int G, const ProposeArgs& pa, int64_t N, cudaStream_t s) {
    const int R = PT / G;
    const int grid = (int)((N + R - 1) / R);
    if (grid == 0) return;
    if (pa.charging) {
        switch (G) {
            case 1: k_propose_tile<NN, 1, true><<<grid, PT, 0, s>>>(pa); break;
            case 2: k_propose_tile<NN, 2, true><<<grid, PT, 0, s>>>(pa); break;
            case 4: k_propose_tile<NN, 4, true><<<grid, PT, 0, s>>>(pa); break;
            default: k_propose_tile<NN, 8, true><<<grid, PT, 0, s>>>(pa); break;
        }
    } else {
        switch (G) {
            case 1: k_propose_tile<NN, 1, false><<<grid, PT, 0, s>>>(pa); break;
            case 2: k_propose_tile<NN, 2, false><<<grid, PT, 0, s>>>(pa); break;
            case 4: k_propose_tile<NN, 4, false><<<grid, PT, 0, s>>>(pa); break;
            default: k_propose_tile<NN, 8, false><<<grid, PT, 0, s>>>(pa); break;
        }
    }
}

// lanes-per-row code of the round-0 stream (launch_stream_g): an average tile (256 / G
// rows) fits a stage; 0 = one lane with small stages, 1 = one lane with big stages
static int tile_lanes(double avg) {
    if (avg <= 7) return 0;
    if (avg <= 14) return 3;  // (2 lanes, small stages): C4's skewed rows
    if (avg <= 30) return 1;
    if (avg <= 60) return 2;
    return 8;
}

// lanes per row of the rows-mode rounds: kRowsT entries per lane cover an average row
static int rows_lanes(double avg) {
    if (avg <= 4) return 1;
    if (avg <= 8) return 2;
    if (avg <= 16) return 4;
    if (avg <= 32) return 8;
    return 16;
}

static int lanes_per_row(double avg) {
    // enough lanes to cover an average row in one or two passes
    if (avg <= 3) return 2;
    if (avg <= 7.5) return 4;
    if (avg <= 16) return 8;
    if (avg <= 40) return 16;
    return 32;
}

template <int NN>
static int factor_impl(const lf_csr_t* A, const lf_factor_opts_t* o, int32_t* pi, float* pi_w,
                       float* pi_val, float* diag, int32_t* rounds_dev, int64_t* live,
                       const FactorWs& w, cudaStream_t s, const PartCtx* part) {
    const int64_t N = A->n;                        // CSR rows
    const int64_t NL = part ? part->NL : N;        // vertex-indexed array length
    const int64_t row_base = part ? part->row_base : 0;
    const int64_t gid_off = part ? part->gid_off : 0;
    if (part && o->until_maximal) return set_error(LF_EINVAL, "partitioned factor: until_maximal unsupported");
    const int M = o->until_maximal ? 0x7fffffff : o->M;
    const double pthr = (double)o->p * 4294967296.0;
    unsigned long long thr = pthr <= 0 ? 0ull : (pthr >= 4294967296.0 ? 4294967296ull
                                                                      : (unsigned long long)ceil(pthr));
    const int G = lanes_per_row(N > 0 ? (double)A->nnz / (double)N : 1.0);
    const int grid_p = persistent_grid((const void*)k_propose<NN, 32>, 256);
    const int grid_m = persistent_grid((const void*)k_mutual<NN>, 256);

    {  // one memset for the contiguous control block (counts, flags, long_count, live_part)
        const bool lv = live && !o->until_maximal && o->M > 0;
        const char* end = lv ? (const char*)(w.live_part + (size_t)128 * o->M) : (const char*)w.live_part;
        LF_CUDA(cudaMemsetAsync(w.counts, 0, (size_t)(end - (const char*)w.counts), s));
    }
    if ((N == 0 && !part) || (!o->until_maximal && o->M == 0)) {
        // no rounds: empty factor (a partition with no rows still takes part in the
        // exchanges below, so it only returns here when there are no rounds at all)
        if (NL > 0) {
            LF_CUDA(cudaMemsetAsync(pi, 0xff, sizeof(int32_t) * NL * NN, s));
            LF_CUDA(cudaMemsetAsync(pi_w, 0, sizeof(float) * NL * NN, s));
            if (pi_val) LF_CUDA(cudaMemsetAsync(pi_val, 0, sizeof(float) * NL * NN, s));
        }
        if (N > 0 && diag) {
            LF_PROF("diag", -1, s);
            k_diag<<<persistent_grid((const void*)k_diag, 256), 256, 0, s>>>(N, A->rowptr, A->col, A->val, diag,
                                                                           row_base);
            LF_CUDA(cudaGetLastError());
        }
        if (rounds_dev) LF_CUDA(cudaMemsetAsync(rounds_dev, 0, sizeof(int32_t), s));
        return LF_OK;
    }
    const bool charged0 = (0 % o->m) != o->k_m;
    if (charged0) {
        LF_PROF("init_state", -1, s);
        k_init_state<<<persistent_grid((const void*)k_init_state, 256), 256, 0, s>>>(
            NL, w.state, o->seed, thr, part ? part->l2g : nullptr);
        LF_CUDA(cudaGetLastError());
    }
    int rounds_host = -1;
    // partitioned runs (rounds cannot be fused: two halo exchanges per round) use the rows-mode
    // kernels per round for large row ranges (LF_PART_ROWS=0/1 overrides)
    RowsArgs pr;
    memset(&pr, 0, sizeof(pr));
    const char* prs = getenv("LF_PART_ROWS");
    const bool rows_part = part && !o->until_maximal && o->M <= kMaxFlagRounds &&
                           (prs ? strcmp(prs, "0") != 0 : N >= ((int64_t)1 << 20));
    if (rows_part) {
        pr.N = N;
        pr.rowptr = A->rowptr;
        pr.col = A->col;
        pr.val = A->val;
        pr.state = w.state;
        pr.pi = pi;
        pr.pi_w = pi_w;
        pr.pi_val = pi_val;
        pr.prop_j = w.prop_j;
        pr.prop_v = w.prop_v;
        pr.flags = w.flags;
        pr.live_part = live ? w.live_part : nullptr;
        pr.long_rows = w.long_rows;
        pr.long_count = w.long_count;
        pr.defer_len = 128;
        pr.M = o->M;
        pr.m = o->m;
        pr.k_m = o->k_m;
        pr.seed = o->seed;
        pr.thr = thr;
        pr.bail = nullptr;    // always run
        pr.rounds = nullptr;  // the host's pre_finalize hook reduces the flags first: k_finalize
        pr.live = nullptr;
        pr.wl[0] = w.wl[0];
        pr.wl[1] = w.wl[1];
        pr.counts = w.counts;
        pr.row_base = row_base;
        pr.gid_off = gid_off;
        static bool pattr = false;
        if (!pattr) {
            LF_CUDA(cudaFuncSetAttribute((const void*)k_rows_propose_k<NN>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         (int)sizeof(RowsSmemK<NN>)));
            pattr = true;
        }
    }
    // rounds 1..M-1 in one cooperative kernel unless the host must check maximality
    const bool fuse = !o->until_maximal && o->M > 1 && !part;
    const int M_loop = fuse ? 1 : M;
    for (int k = 0; k < M_loop; k++) {
        const bool charging = (k % o->m) != o->k_m;
        const bool fresh = (k == 0);
        if (part && (k > 0 || charged0)) {  // halo: ghost degrees and charges of round k
            const int rc = part->pre_propose(part->ctx, k, s);
            if (rc) return rc;
        }
        ProposeArgs pa;
        pa.N = N;
        pa.row_base = row_base;
        pa.rowptr = A->rowptr;
        pa.col = A->col;
        pa.val = A->val;
        pa.state = (fresh && !charged0) ? nullptr : w.state;
        pa.pi = fresh ? nullptr : pi;
        pa.wl = fresh ? nullptr : w.wl[k & 1];
        pa.wl_count = fresh ? nullptr : &w.counts[k % 3];
        pa.prop_j = w.prop_j;
        pa.prop_v = w.prop_v;
        pa.diag = fresh ? diag : nullptr;
        pa.charging = charging ? 1 : 0;
        const bool rec = live && !o->until_maximal;
        pa.live_rows = rec ? w.live_part + (size_t)k * 128 : nullptr;
        pa.live_nnz = rec ? w.live_part + (size_t)k * 128 + 64 : nullptr;
        pa.proposed = &w.flags[k % kMaxFlagRounds];
        pa.defer_list = w.long_rows;
        pa.defer_count = &w.long_count[k % kMaxFlagRounds];
        if (o->until_maximal && k >= kMaxFlagRounds) {
            LF_CUDA(cudaMemsetAsync(pa.proposed, 0, sizeof(int), s));
            LF_CUDA(cudaMemsetAsync(pa.defer_count, 0, sizeof(int32_t), s));
        }
        {
            LF_PROF("propose", k, s);
            if (fresh) {
                const int Gt = tile_lanes(N > 0 ? (double)A->nnz / (double)N : 1.0);
                pa.defer_len = Gt == 0 ? 32 : (Gt == 1 ? 128 : (Gt == 3 ? 64 : 32 * Gt));
#ifdef LF_TILE_PLAIN
                launch_propose_tile<NN>(Gt <= 1 ? 1 : (Gt == 3 ? 2 : Gt), pa, N, s);
#else
                launch_propose_stream<NN>(Gt, pa, s);
#endif
            } else if (rows_part) {
                pr.only_k = k;
                LF_CUDA(launch_pdl(k_rows_propose_k<NN>,
                                   persistent_grid((const void*)k_rows_propose_k<NN>, kRowsTK, sizeof(RowsSmemK<NN>)),
                                   kRowsTK, sizeof(RowsSmemK<NN>), s, pr));
            } else {
                pa.defer_len = 32 * G;
                launch_propose<NN>(G, pa, grid_p, s);
            }
            LF_CUDA(cudaGetLastError());
        }
        {
            // long rows of this round: one CTA per row
            LF_PROF("propose_long", k, s);
            ProposeArgs pl = pa;
            pl.wl = w.long_rows;
            pl.wl_count = pa.defer_count;
            pl.defer_len = INT64_MAX;
            LF_CUDA(launch_pdl(k_propose_long_blk<NN>, persistent_grid((const void*)k_propose_long_blk<NN>, 256),
                               256, 0, s, pl));
        }

        if (o->until_maximal && (k % o->m) == o->k_m) {
            // L23-L25 checked on the host in this mode (one sync per m rounds)
            int f = 0;
            LF_CUDA(cudaMemcpyAsync(&f, pa.proposed, sizeof(int), cudaMemcpyDeviceToHost, s));
            LF_CUDA(cudaStreamSynchronize(s));
            if (f == 0) {
                rounds_host = k + 1;
                if (fresh) {
                    // nothing proposed at all: export the empty factor
                    MutualArgs ma{};
                    ma.N = N; ma.row_base = row_base; ma.gid_off = gid_off; ma.prop_j = w.prop_j; ma.prop_v = w.prop_v; ma.state = w.state;
                    ma.pi = pi; ma.pi_w = pi_w; ma.pi_val = pi_val; ma.fresh = 1;
                    k_mutual<NN><<<grid_m, 256, 0, s>>>(ma);
                    LF_CUDA(cudaGetLastError());
                }
                break;
            }
        }
        if (part) {  // halo: ghost proposals of round k
            const int rc = part->pre_mutual(part->ctx, k, s);
            if (rc) return rc;
        }
        const bool last = !o->until_maximal && (k == M - 1);
        MutualArgs ma;
        ma.wl_zero = nullptr;
        ma.N = N;
        ma.row_base = row_base;
        ma.gid_off = gid_off;
        ma.wl = fresh ? nullptr : w.wl[k & 1];
        ma.wl_count = fresh ? nullptr : &w.counts[k % 3];
        ma.prop_j = w.prop_j;
        ma.prop_v = w.prop_v;
        ma.state = w.state;
        ma.pi = pi;
        ma.pi_w = pi_w;
        ma.pi_val = pi_val;
        ma.wl_next = last ? nullptr : w.wl[(k + 1) & 1];
        ma.wl_next_count = last ? nullptr : &w.counts[(k + 1) % 3];
        ma.wl_zero = last ? nullptr : &w.counts[(k + 2) % 3];
        ma.fresh = fresh ? 1 : 0;
        ma.pad_state = (fresh && !part) ? 1 : 0;
        ma.next_charging = ((k + 1) % o->m) != o->k_m;
        ma.next_k = (uint32_t)(k + 1);
        ma.seed = o->seed;
        ma.thr = thr;
        {
            LF_PROF("mutual", k, s);
            // all-rows round 0: batched kernel with vector slot loads (needs aligned slots)
            const uintptr_t amask = (NN == 2 ? 7 : (NN == 4 ? 15 : 3));
            const bool aligned = ((uintptr_t)pi & amask) == 0 && ((uintptr_t)pi_w & amask) == 0 &&
                                 (!pi_val || ((uintptr_t)pi_val & amask) == 0);
            if (fresh && aligned && N > 0) {
                const int64_t per = 256 * (int64_t)kMutual0Rows;
                const int64_t g = (N + per - 1) / per;
                LF_CUDA(launch_pdl(k_mutual0<NN, kMutual0Rows>, (int)(g < (1 << 20) ? g : (1 << 20)), 256, 0, s, ma));
            } else if (rows_part && !fresh) {
                pr.only_k = k;
                LF_CUDA(launch_pdl(k_rows_mutual_k<NN>, persistent_grid((const void*)k_rows_mutual_k<NN>, 256), 256, 0,
                                   s, pr));
            } else {
                LF_CUDA(launch_pdl(k_mutual<NN>, grid_m, 256, 0, s, ma));
            }
        }
    }
    if (fuse) {
        FusedArgs f;
        memset(&f, 0, sizeof(f));
        ProposeArgs& pa = f.pa;
        pa.N = N;
        pa.row_base = 0;
        pa.rowptr = A->rowptr;
        pa.col = A->col;
        pa.val = A->val;
        pa.state = w.state;
        pa.pi = pi;
        pa.prop_j = w.prop_j;
        pa.prop_v = w.prop_v;
        pa.diag = nullptr;
        pa.defer_list = w.long_rows;
        MutualArgs& ma = f.ma;
        ma.N = N;
        ma.row_base = 0;
        ma.gid_off = 0;
        ma.prop_j = w.prop_j;
        ma.prop_v = w.prop_v;
        ma.state = w.state;
        ma.pi = pi;
        ma.pi_w = pi_w;
        ma.pi_val = pi_val;
        ma.seed = o->seed;
        ma.thr = thr;
        f.wl[0] = w.wl[0];
        f.wl[1] = w.wl[1];
        f.counts = w.counts;
        f.flags = w.flags;
        f.long_rows = w.long_rows;
        f.long_count = w.long_count;
        f.live_part = (live && !o->until_maximal) ? w.live_part : nullptr;
        f.M = o->M;
        f.m = o->m;
        f.k_m = o->k_m;
        f.rounds = rounds_dev;
        f.live = live;
        f.cached = cached_rounds_enabled() ? 1 : 0;
        f.bail = &w.counts[3];
        {
            LF_PROF("rounds_fused", -1, s);
            void* args[] = {&f};
            const void* kfn = (const void*)k_rounds_fused<NN>;
            const size_t smem = f.cached ? cache_smem_bytes<NN>() : 0;
            if (f.cached) {
                static bool attr = false;
                if (!attr) {
                    LF_CUDA(cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
                    attr = true;
                }
            }
            int grid = LF_FUSED_GRID > 0 ? LF_FUSED_GRID : sm_count() * LF_FUSED_GRID_SM;  // fewer CTAs: cheaper barriers
            const int cap = persistent_grid(kfn, LF_FUSED_T, smem);
            if (grid > cap) grid = cap;
            LF_CUDA(cudaLaunchCooperativeKernel(kfn, grid, LF_FUSED_T, args, smem, s));
        }
        {
            RowsArgs r;
            memset(&r, 0, sizeof(r));
            r.N = N;
            r.rowptr = A->rowptr;
            r.col = A->col;
            r.val = A->val;
            r.state = w.state;
            r.pi = pi;
            r.pi_w = pi_w;
            r.pi_val = pi_val;
            r.prop_j = w.prop_j;
            r.prop_v = w.prop_v;
            r.flags = w.flags;
            r.live_part = f.live_part;
            r.long_rows = w.long_rows;
            r.long_count = w.long_count;
            r.M = o->M;
            r.m = o->m;
            r.k_m = o->k_m;
            r.seed = o->seed;
            r.thr = thr;
            r.bail = f.bail;
            r.rounds = rounds_dev;
            r.live = live;
            r.wl[0] = w.wl[0];
            r.wl[1] = w.wl[1];
            r.counts = w.counts;
            const int Gr = rows_lanes(N > 0 ? (double)A->nnz / (double)N : 1.0);
            r.defer_len = 128;  // longer rows: a CTA per row (and 32 padded rows of <= 24 fit kRowsBud)
            const void* kfn;
            switch (Gr) {
                case 1: kfn = (const void*)k_rounds_rows<NN, 1>; break;
                case 2: kfn = (const void*)k_rounds_rows<NN, 2>; break;
                case 4: kfn = (const void*)k_rounds_rows<NN, 4>; break;
                case 8: kfn = (const void*)k_rounds_rows<NN, 8>; break;
                default: kfn = (const void*)k_rounds_rows<NN, 16>; break;
            }
            const int rsm = (int)sizeof(RowsSmem);
            {
                static bool attr[5] = {false, false, false, false, false};
                const int gi = Gr == 1 ? 0 : Gr == 2 ? 1 : Gr == 4 ? 2 : Gr == 8 ? 3 : 4;
                if (!attr[gi]) {
                    LF_CUDA(cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, rsm));
                    attr[gi] = true;
                }
            }
            cudaLaunchConfig_t cfg = {};
            cfg.gridDim = dim3(persistent_grid(kfn, LF_ROWS_T, rsm));
            cfg.blockDim = dim3(LF_ROWS_T);
            cfg.dynamicSmemBytes = rsm;
            cfg.stream = s;
            cudaLaunchAttribute at[2];
            at[0].id = cudaLaunchAttributeCooperative;
            at[0].val.cooperative = 1;
            at[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
            at[1].val.programmaticStreamSerializationAllowed = 1;
            cfg.attrs = at;
            cfg.numAttrs = pdl_enabled() ? 2 : 1;
            void* args[] = {&r};
            // large graphs: three kernels per round (k_rows_*_k); others: one cooperative kernel
            const char* sp = getenv("LF_ROWS_SPLIT");
            const bool split = sp ? strcmp(sp, "0") != 0 : N >= ((int64_t)1 << 22);
            if (split) {
                const void* kp = (const void*)k_rows_propose_k<NN>;
                const int psm = (int)sizeof(RowsSmemK<NN>);
                static bool pattr = false;
                if (!pattr) {
                    LF_CUDA(cudaFuncSetAttribute(kp, cudaFuncAttributeMaxDynamicSharedMemorySize, psm));
                    pattr = true;
                }
                cudaLaunchConfig_t c2 = cfg;
                c2.attrs = at + 1;  // PDL only
                c2.numAttrs = pdl_enabled() ? 1 : 0;
                const void* kl = (const void*)k_rows_long_k<NN>;
                const void* km = (const void*)k_rows_mutual_k<NN>;
                for (int k = 1; k < o->M; k++) {
                    r.only_k = k;
                    {
                        LF_PROF("rows_propose", k, s);
                        c2.gridDim = dim3(persistent_grid(kp, kRowsTK, psm));
                        c2.blockDim = dim3(kRowsTK);
                        c2.dynamicSmemBytes = psm;
                        LF_CUDA(cudaLaunchKernelExC(&c2, kp, args));
                    }
                    {
                        LF_PROF("rows_long", k, s);
                        c2.gridDim = dim3(persistent_grid(kl, 256));
                        c2.blockDim = dim3(256);
                        c2.dynamicSmemBytes = 0;
                        LF_CUDA(cudaLaunchKernelExC(&c2, kl, args));
                    }
                    {
                        LF_PROF("rows_mutual", k, s);
                        c2.gridDim = dim3(persistent_grid(km, 256));
                        LF_CUDA(cudaLaunchKernelExC(&c2, km, args));
                    }
                }
            } else {
                LF_PROF("rounds_rows", -1, s);
                LF_CUDA(cudaLaunchKernelExC(&cfg, kfn, args));
            }
        }
    }
    if (o->until_maximal) {
        if (rounds_dev) {
            LF_CUDA(cudaMemcpyAsync(rounds_dev, &rounds_host, sizeof(int32_t), cudaMemcpyHostToDevice, s));
            LF_CUDA(cudaStreamSynchronize(s));
        }
    } else if (!fuse && (rounds_dev || live)) {
        if (part && part->pre_finalize) {  // global maximality flags / counters
            const int rc = part->pre_finalize(part->ctx, s);
            if (rc) return rc;
        }
        LF_PROF("finalize", -1, s);
        LF_CUDA(launch_pdl(k_finalize, 1, 32, 0, s, (const int*)w.flags, o->M, o->m, o->k_m, rounds_dev,
                           (const unsigned long long*)w.live_part, live));
    }
    return LF_OK;
}

int factor_dispatch(const lf_csr_t* A, int n, const lf_factor_opts_t* o, int32_t* pi, float* pi_w,
                    float* pi_val, float* diag, int32_t* rounds_dev, int64_t* live, const FactorWs& w,
                    cudaStream_t s, const PartCtx* part) {
    switch (n) {
        case 1: return factor_impl<1>(A, o, pi, pi_w, pi_val, diag, rounds_dev, live, w, s, part);
        case 2: return factor_impl<2>(A, o, pi, pi_w, pi_val, diag, rounds_dev, live, w, s, part);
        case 3: return factor_impl<3>(A, o, pi, pi_w, pi_val, diag, rounds_dev, live, w, s, part);
        case 4: return factor_impl<4>(A, o, pi, pi_w, pi_val, diag, rounds_dev, live, w, s, part);
        default: return set_error(LF_EINVAL, "n must be in [1,4]");
    }
}

#ifdef LF_TIMELINE
int timeline_factor(unsigned long long* out, int reset) {
    if (reset) {
        unsigned long long h[16];
        for (int i = 0; i < 16; i += 2) { h[i] = ~0ull; h[i + 1] = 0; }
        return cudaMemcpyToSymbol(g_tl_factor, h, sizeof(h)) == cudaSuccess ? 0 : -1;
    }
    return cudaMemcpyFromSymbol(out, g_tl_factor, sizeof(g_tl_factor)) == cudaSuccess ? 0 : -1;
}
#else
int timeline_factor(unsigned long long*, int) { return -1; }
#endif
}  // namespace lf
