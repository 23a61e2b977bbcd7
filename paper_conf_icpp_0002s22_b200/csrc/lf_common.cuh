// lf_common.cuh -- device helpers shared by the sm_100a kernels of liblf.so.
//
// Nothing here is shared with oracle/ (the CPU oracle is an independent C file).
#pragma once

#include <cstdint>
#include <cuda_runtime.h>

#include "../../include/lf.h"

namespace lf {

// ---------------------------------------------------------------------------
// Proposal keys (Table 1 accumulator of (|a_vj|, j) pairs, L207-L214, L235).
// One 64-bit key orders the candidates of a row totally: |a| descending, then j
// ascending (DESIGN.md §3 reading c1), so a top-n reduction in ANY order gives the same
// result.  The signed value travels in bit 0 (never decides the order: no row holds
// the same j twice):
//   bits 62..32  |a| (fp32 bits without sign: order-preserving for finite |a| > 0)
//   bits 31..1   0x7FFFFFFF - j
//   bit  0       sign of a
// key 0 = "empty" (every real key has |a| bits >= 1).
// ---------------------------------------------------------------------------
__device__ __forceinline__ uint64_t make_key(float a, int32_t j) {
    uint32_t b = __float_as_uint(a);
    uint32_t lo = ((0x7FFFFFFFu - (uint32_t)j) << 1) | (b >> 31);
    return ((uint64_t)(b & 0x7FFFFFFFu) << 32) | lo;
}
__device__ __forceinline__ int32_t key_col(uint64_t k) {
    return (int32_t)(0x7FFFFFFFu - ((uint32_t)k >> 1));
}
__device__ __forceinline__ float key_abs(uint64_t k) { return __uint_as_float((uint32_t)(k >> 32)); }
__device__ __forceinline__ float key_val(uint64_t k) {
    return __uint_as_float((uint32_t)(k >> 32) | (((uint32_t)k & 1u) << 31));
}
// key from stored (|w|, signed value, j): used to merge existing confirmed slots
__device__ __forceinline__ uint64_t make_key_abs(float absw, uint32_t sign, int32_t j) {
    uint32_t lo = ((0x7FFFFFFFu - (uint32_t)j) << 1) | (sign & 1u);
    return ((uint64_t)__float_as_uint(absw) << 32) | lo;
}

// Sorted (descending) top-NN insertion, branch-free bubble.
template <int NN>
__device__ __forceinline__ void topn_insert(uint64_t (&t)[NN], uint64_t x) {
#pragma unroll
    for (int i = 0; i < NN; i++) {
        uint64_t hi = t[i] > x ? t[i] : x;
        x = t[i] > x ? x : t[i];
        t[i] = hi;
    }
}

// Butterfly merge of sorted top-NN lists across G consecutive lanes (G power of 2).
template <int NN, int G>
__device__ __forceinline__ void topn_merge_group(uint64_t (&t)[NN]) {
#pragma unroll
    for (int off = G / 2; off >= 1; off >>= 1) {
        uint64_t y[NN];
#pragma unroll
        for (int i = 0; i < NN; i++) y[i] = __shfl_xor_sync(0xffffffffu, t[i], off);
#pragma unroll
        for (int i = 0; i < NN; i++) topn_insert<NN>(t, y[i]);
    }
}

// ---------------------------------------------------------------------------
// charge(v,k): MD5 round 1 over the 12-byte message (v, k, seed) ("a part
// of the MD5 algorithm"; DESIGN.md §3 reading c2).  '+' iff a + 0x67452301 < p*2^32.
// Written from RFC 1321 independently of oracle/.
// ---------------------------------------------------------------------------
__device__ __forceinline__ uint32_t md5r1_step(uint32_t a, uint32_t b, uint32_t c, uint32_t d,
                                               uint32_t x, uint32_t t, int s) {
    uint32_t f = (b & c) | (~b & d);
    return b + __funnelshift_l(a + f + x + t, a + f + x + t, s);
}

__device__ __forceinline__ uint32_t charge_hash(uint32_t v, uint32_t k, uint32_t seed) {
    uint32_t a = 0x67452301u, b = 0xefcdab89u, c = 0x98badcfeu, d = 0x10325476u;
    // message words: v, k, seed, 0x80 (padding), 0..., 96 (bit length) at word 14
    a = md5r1_step(a, b, c, d, v, 0xd76aa478u, 7);
    d = md5r1_step(d, a, b, c, k, 0xe8c7b756u, 12);
    c = md5r1_step(c, d, a, b, seed, 0x242070dbu, 17);
    b = md5r1_step(b, c, d, a, 0x80u, 0xc1bdceeeu, 22);
    a = md5r1_step(a, b, c, d, 0u, 0xf57c0fafu, 7);
    d = md5r1_step(d, a, b, c, 0u, 0x4787c62au, 12);
    c = md5r1_step(c, d, a, b, 0u, 0xa8304613u, 17);
    b = md5r1_step(b, c, d, a, 0u, 0xfd469501u, 22);
    a = md5r1_step(a, b, c, d, 0u, 0x698098d8u, 7);
    d = md5r1_step(d, a, b, c, 0u, 0x8b44f7afu, 12);
    c = md5r1_step(c, d, a, b, 0u, 0xffff5bb1u, 17);
    b = md5r1_step(b, c, d, a, 0u, 0x895cd7beu, 22);
    a = md5r1_step(a, b, c, d, 0u, 0x6b901122u, 7);
    d = md5r1_step(d, a, b, c, 0u, 0xfd987193u, 12);
    c = md5r1_step(c, d, a, b, 96u, 0xa679438eu, 17);
    b = md5r1_step(b, c, d, a, 0u, 0x49b40821u, 22);
    return a + 0x67452301u;
}

// threshold: charge '+' iff hash < thr, thr = floor(p * 2^32) clamped (host computes it)
__device__ __forceinline__ uint32_t charge_bit(uint32_t v, uint32_t k, uint32_t seed,
                                               uint64_t thr) {
    return (uint64_t)charge_hash(v, k, seed) < thr ? 1u : 0u;
}

// vertex state byte: bits 0..2 = number of confirmed edges (0..4),
// bit 3 = charge of v in the current round, bit 4 = live (below).
constexpr uint8_t ST_DEG = 0x7;
constexpr uint8_t ST_CHARGE = 0x8;
// bit 4: v is live at the current round's start (deg < n and not retired) -- the rows mode
// of the rounds streams the rows carrying it (lf_factor.cu k_rounds_rows)
constexpr uint8_t ST_LIVE = 0x10;

// prop_j slot value for a row whose charge-free candidate set is empty (retired)
constexpr int32_t PROP_RETIRED = -2;

// PDL (see launch_pdl): wait until the stream predecessor grid has completed and its
// writes are visible (a no-op for an ordinary launch); let the successor grid launch early
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }

// Diagnostic timeline (builds with -DLF_TIMELINE only): earliest CTA start / latest CTA
// exit of each kernel of the step, on the global timer; read by lf_debug_timeline.
#ifdef LF_TIMELINE
__device__ __forceinline__ unsigned long long tl_now() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
struct TlScope {
    unsigned long long* slot;
    __device__ explicit TlScope(unsigned long long* s) : slot(s) {
        if (threadIdx.x == 0) atomicMin(slot, tl_now());
    }
    __device__ ~TlScope() {
        if (threadIdx.x == 0) atomicMax(slot + 1, tl_now());
    }
};
#define LF_TL(arr, id) ::lf::TlScope lf_tl_scope_(&(arr)[2 * (id)])
#else
#define LF_TL(arr, id) do { } while (0)
#endif

}  // namespace lf
