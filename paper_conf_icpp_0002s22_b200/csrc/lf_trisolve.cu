// lf_trisolve.cu -- apply the tridiagonal preconditioner: y = T^{-1} x for the (a, b, c)
// that lf_tridiag writes (§1 "Tridiagonal systems can be
// inverted at the bandwidth limit of the GPU [21]", §6).
//
// T is block diagonal: row r is uncoupled from row r-1 exactly when a[r] = c[r-1] = 0,
// which is the case at every path boundary of the linear forest (L219).  Each such
// segment is an independent tridiagonal system.  Two paths, both always launched; a
// device flag (TriCtl::seq, set by the partition path's checks) makes one of them exit:
//   - partition path (diagonally dominant T; k_part_pass1 / k_part_chain / k_part_pass2,
//     below): fixed 32-row chunks, a reduced system of two unknowns per chunk swept per
//     chain of coupled chunks, then one more pass per chunk;
//   - sequential path (any other T): k_seg_solve, one thread per segment (found by a
//     grid-stride scan of the rows), Gaussian elimination with scaled partial pivoting
//     (the pivoting strategy of [21]; reading f2-1) streaming down the segment
//     with the pending row in registers, U rows with their right-hand side stored as one
//     float4, then back substitution upwards.
// fp32 throughout (the paper's GPU path is fp32).
#include <cuda_runtime.h>

#include <cstdint>

#include "lf_common.cuh"
#include "lf_internal.h"

namespace lf {

struct TriCtl {
    unsigned int seq;    // 1: use the sequential pivoting path
};

__device__ __forceinline__ bool seg_start(int64_t r, const float* __restrict__ a,
                                          const float* __restrict__ c) {
    return r == 0 || (__ldg(a + r) == 0.0f && __ldg(c + r - 1) == 0.0f);
}

__device__ __forceinline__ float row_scale(float l, float d, float u) {
    return fmaxf(fabsf(l), fmaxf(fabsf(d), fabsf(u)));
}

__global__ void __launch_bounds__(128) k_seg_solve(int64_t N, const float* __restrict__ a,
                                                   const float* __restrict__ b,
                                                   const float* __restrict__ c,
                                                   const float* __restrict__ x,
                                                   const TriCtl* __restrict__ ctl,
                                                   float4* __restrict__ U, float* __restrict__ y) {
    pdl_wait();
    if (!ctl->seq) return;
    // grid-stride over rows; the thread that owns a segment's first row solves it
    for (int64_t s = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; s < N;
         s += (int64_t)gridDim.x * blockDim.x) {
        if (!seg_start(s, a, c)) continue;
        // pending row i: p*y[i] + q*y[i+1] = rr, scale sc of the original row it came from
        float p = __ldg(b + s), q = __ldg(c + s), rr = __ldg(x + s);
        float sc = row_scale(s > 0 ? __ldg(a + s) : 0.0f, p, q);
        float cprev = q;  // original c[i] (for the segment-end test)
        int64_t i = s;
        for (;;) {
            const int64_t nx = i + 1;
            if (nx >= N) break;
            const float l = __ldg(a + nx);
            if (l == 0.0f && cprev == 0.0f) break;  // nx starts the next segment
            const float d = __ldg(b + nx), u = __ldg(c + nx), xn = __ldg(x + nx);
            const float sn = row_scale(l, d, u);
            if (fabsf(p) * sn >= fabsf(l) * sc) {  // |p|/sc >= |l|/sn: keep row i as pivot
                U[i] = make_float4(p, q, 0.0f, rr);
                const float f = l / p;
                p = fmaf(-f, q, d);
                q = u;
                rr = fmaf(-f, rr, xn);
                sc = sn;
            } else {  // interchange: row nx is the pivot row of column i
                U[i] = make_float4(l, d, u, xn);
                const float f = p / l;
                p = fmaf(-f, d, q);
                q = -f * u;
                rr = fmaf(-f, xn, rr);
            }
            cprev = u;
            i = nx;
        }
        // back substitution, rows i (= segment end) .. s
        float y1 = rr / p, y2 = 0.0f;
        y[i] = y1;
        for (int64_t k = i - 1; k >= s; --k) {
            const float4 w = U[k];
            const float yk = (w.w - w.y * y1 - w.z * y2) / w.x;
            y[k] = yk;
            y2 = y1;
            y1 = yk;
        }
    }
}

// ---------------------------------------------------------------------------------------
// Partition path (diagonally dominant T): fixed chunks of PK rows, one
// thread per chunk, PB chunks per block staged through shared memory with coalesced loads.
//   pass 1: each chunk solves T_j z = rhs for rhs = x_j, -a[s] e_1, -c[e] e_K (Thomas,
//           no pivoting: stable under diagonal dominance) and keeps the first and last
//           entries of the three solutions: y_j = P + G y[s-1] + H y[e+1].
//   chain:  one thread per chain of coupled chunks sweeps the 2-unknowns-per-chunk reduced
//           system (F_j = y[s], L_j = y[e]) forward and back.
//   pass 2: each chunk re-solves with x[s] -= a[s] L_{j-1}, x[e] -= c[e] F_{j+1}.
// Pass 1 also checks |b| >= |a| + |c|, b != 0 on every row and a nonzero Thomas pivot; any
// failure sets ctl->seq and the partition results are overwritten by the pivoting path.
// ---------------------------------------------------------------------------------------
#ifndef LF_TS_PK
#define LF_TS_PK 32
#endif
#ifndef LF_TS_CB
#define LF_TS_CB 8
#endif
constexpr int PK = LF_TS_PK;  // rows per chunk
constexpr int PB = 64;        // chunks (threads) per block
constexpr int PS = PK + 1;  // padded smem row stride (conflict-free column walks)
constexpr unsigned TS_SPLIT = 1, TS_DEC = 2, TS_DECNEXT = 4;

// reciprocal without the IEEE slow path: MUFU approximation + one Newton step (about
// 1 ulp; no branch, two dependent FMAs instead of __frcp_rn's checked sequence)
__device__ __forceinline__ float rcp_nr(float m) {
    float r;
    asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(m));
    return fmaf(r, fmaf(-m, r, 1.0f), r);
}

struct ChunkSmem {
    float a[PB * PS], b[PB * PS], c[PB * PS], x[PB * PS];
};

// staging of rows [r0, r0 + PB*PK) into the padded [thread][PS] layout: 16-byte loads
// through registers when the block is full and the arrays are 16-byte aligned, else one
// 4-byte cp.async per element (coalesced across the block, all in flight at once);
// a[0] and c[N-1] are ignored (0) and rows past N become identity rows
__device__ __forceinline__ void cp_async4(float* dst, const float* src) {
    const unsigned d = (unsigned)__cvta_generic_to_shared(dst);
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(d), "l"(src) : "memory");
}

__device__ __forceinline__ void stage_chunks(int64_t N, int64_t r0, const float* __restrict__ a,
                                             const float* __restrict__ b,
                                             const float* __restrict__ c,
                                             const float* __restrict__ x, ChunkSmem& S) {
    const bool al16 = ((reinterpret_cast<uintptr_t>(a) | reinterpret_cast<uintptr_t>(b) |
                        reinterpret_cast<uintptr_t>(c) | reinterpret_cast<uintptr_t>(x)) & 15) == 0;
    if (r0 + PB * PK <= N && al16) {
        // full block, 16-byte aligned arrays: 16-byte loads, all 4 x 8 in flight per thread,
        // then scalar stores into the padded layout (a float4 never straddles a chunk and
        // the 32 lanes of a warp hit 32 distinct banks)
        constexpr int NV = PB * PK / 4 / PB;
        float4 va[NV], vb[NV], vc[NV], vx[NV];
        const float4* a4 = reinterpret_cast<const float4*>(a + r0);
        const float4* b4 = reinterpret_cast<const float4*>(b + r0);
        const float4* c4 = reinterpret_cast<const float4*>(c + r0);
        const float4* x4 = reinterpret_cast<const float4*>(x + r0);
#pragma unroll
        for (int n = 0; n < NV; ++n) {
            const int q = threadIdx.x + n * PB;
            va[n] = __ldg(a4 + q);
            vb[n] = __ldg(b4 + q);
            vc[n] = __ldg(c4 + q);
            vx[n] = __ldg(x4 + q);
        }
#pragma unroll
        for (int n = 0; n < NV; ++n) {
            const int k = 4 * (threadIdx.x + n * PB);
            const int o = (k / PK) * PS + (k % PK);
            S.a[o] = va[n].x, S.a[o + 1] = va[n].y, S.a[o + 2] = va[n].z, S.a[o + 3] = va[n].w;
            S.b[o] = vb[n].x, S.b[o + 1] = vb[n].y, S.b[o + 2] = vb[n].z, S.b[o + 3] = vb[n].w;
            S.c[o] = vc[n].x, S.c[o + 1] = vc[n].y, S.c[o + 2] = vc[n].z, S.c[o + 3] = vc[n].w;
            S.x[o] = vx[n].x, S.x[o + 1] = vx[n].y, S.x[o + 2] = vx[n].z, S.x[o + 3] = vx[n].w;
        }
    } else if (r0 + PB * PK <= N) {
#pragma unroll 8
        for (int k = threadIdx.x; k < PB * PK; k += PB) {
            const int o = (k / PK) * PS + (k % PK);
            cp_async4(S.a + o, a + r0 + k);
            cp_async4(S.b + o, b + r0 + k);
            cp_async4(S.c + o, c + r0 + k);
            cp_async4(S.x + o, x + r0 + k);
        }
    } else {
        for (int k = threadIdx.x; k < PB * PK; k += PB) {
            const int64_t r = r0 + k;
            const int o = (k / PK) * PS + (k % PK);
            if (r < N) {
                cp_async4(S.a + o, a + r);
                cp_async4(S.b + o, b + r);
                cp_async4(S.c + o, c + r);
                cp_async4(S.x + o, x + r);
            } else {
                S.a[o] = 0.0f;
                S.b[o] = 1.0f;
                S.c[o] = 0.0f;
                S.x[o] = 0.0f;
            }
        }
    }
    asm volatile("cp.async.wait_all;" ::: "memory");
    __syncthreads();
    if (threadIdx.x == 0) {
        if (r0 == 0) S.a[0] = 0.0f;
        if (r0 <= N - 1 && N - 1 < r0 + PB * PK) {
            const int k = (int)(N - 1 - r0);
            S.c[(k / PK) * PS + (k % PK)] = 0.0f;
        }
    }
}

__global__ void __launch_bounds__(PB) k_part_pass1(int64_t N, const float* __restrict__ a,
                                                   const float* __restrict__ b,
                                                   const float* __restrict__ c,
                                                   const float* __restrict__ x,
                                                   float4* __restrict__ pg, float4* __restrict__ hh,
                                                   TriCtl* __restrict__ ctl) {
    __shared__ ChunkSmem S;
    const int64_t r0 = (int64_t)blockIdx.x * PB * PK;
    stage_chunks(N, r0, a, b, c, x, S);
    __syncthreads();
    const int64_t j = (int64_t)blockIdx.x * PB + threadIdx.x;
    if (r0 + (int64_t)threadIdx.x * PK >= N) return;
    float* A = S.a + threadIdx.x * PS;
    float* B = S.b + threadIdx.x * PS;
    float* Cc = S.c + threadIdx.x * PS;
    float* X = S.x + threadIdx.x * PS;
    // chain flags (from the original rows, before they are overwritten):
    //   SPLIT: a[r] = c[r-1] = 0 for some r in (s, e] -- the chunk's head no longer sees
    //          y[e+1] and its tail no longer sees y[s-1] (G_last = H_first = 0 exactly);
    //   DEC / DECNEXT: no coupling to the previous / next chunk (or none exists)
    const int64_t s0 = r0 + (int64_t)threadIdx.x * PK, e0 = s0 + PK - 1;
    unsigned fl = 0;
    for (int i = 1; i < PK; ++i)
        if (A[i] == 0.0f && Cc[i - 1] == 0.0f) fl |= TS_SPLIT;
    if (s0 == 0 || (A[0] == 0.0f && __ldg(c + s0 - 1) == 0.0f)) fl |= TS_DEC;
    if (e0 + 1 >= N || (Cc[PK - 1] == 0.0f && __ldg(a + e0 + 1) == 0.0f)) fl |= TS_DECNEXT;
    bool ok = true;
    // Two eliminations of the same chunk, interleaved (independent chains, no stores):
    //  - top-down Thomas gives the LAST entries of the three solutions (rhs x, the G rhs
    //    -a[s] e_1, the H rhs -c[e] e_K);
    //  - bottom-up Thomas (the mirror: a and c swap roles) gives the FIRST entries.
    // Row 0's a and row PK-1's c are the couplings and stay out of both eliminations.
    float cp = 0.0f, dx = 0.0f, dg = 0.0f, mL = 1.0f;   // top-down
    float cq = 0.0f, ex = 0.0f, eh = 0.0f, m0 = 1.0f;   // bottom-up
#pragma unroll 8
    for (int i = 0; i < PK; ++i) {
        {  // top-down, row i
            const float ai = A[i], bi = B[i], ci = Cc[i];
            ok &= (fabsf(bi) >= fabsf(ai) + fabsf(ci)) && bi != 0.0f;
            const float l = (i == 0) ? 0.0f : ai;
            const float m = fmaf(-l, cp, bi);
            ok &= m != 0.0f;
            const float rm = rcp_nr(m);
            dx = fmaf(-l, dx, X[i]) * rm;
            dg = fmaf(-l, dg, (i == 0) ? -ai : 0.0f) * rm;
            cp = ci * rm;
            mL = rm;
        }
        {  // bottom-up, row k
            const int k = PK - 1 - i;
            const float ak = A[k], bk = B[k], ck = Cc[k];
            const float u = (k == PK - 1) ? 0.0f : ck;
            const float m = fmaf(-u, cq, bk);
            ok &= m != 0.0f;
            const float rm = rcp_nr(m);
            ex = fmaf(-u, ex, X[k]) * rm;
            eh = fmaf(-u, eh, (k == PK - 1) ? -ck : 0.0f) * rm;
            cq = ak * rm;
            m0 = rm;
        }
    }
    const float pL = dx, gL = dg, hL = -Cc[PK - 1] * mL;  // H's last entry: -c[e] / m_last
    const float zx = ex, zh = eh, zg = -A[0] * m0;          // G's first entry: -a[s] / m'_first
    pg[j] = make_float4(zx, zg, pL, gL);  // P_first, G_first, P_last, G_last
    hh[j] = make_float4(zh, hL, __uint_as_float(fl), 0.0f);  // H_first, H_last, flags
    ok &= isfinite(zx) && isfinite(zg) && isfinite(zh) && isfinite(pL);
    if (!ok) atomicOr(&ctl->seq, 1u);
}

// one thread per chain of coupled chunks: forward sweep over
//   F_j = pF + gF L_{j-1} + hF F_{j+1},  L_j = pL + gL L_{j-1} + hL F_{j+1}
// with L_{j-1} = u + v F_j, then back substitution F_j = alpha + beta F_{j+1}.
// A chain ends at chunk j when F_j no longer depends on F_{j+1} (SPLIT(j): hF = 0, or
// DECNEXT(j)); the next chain starts at j + 1 with L_j = pL_j + hL_j F_{j+1} (SPLIT, gL
// = 0) or with nothing (DEC).  Chains are therefore as short as the distance between
// path boundaries, not between chunk-aligned ones.
__device__ __forceinline__ unsigned ts_flags(const float4& h) { return __float_as_uint(h.z); }

__global__ void __launch_bounds__(128) k_part_chain(int64_t NC, const float4* __restrict__ pg,
                                                    const float4* __restrict__ hh,
                                                    float4* __restrict__ sweep,
                                                    float2* __restrict__ FL,
                                                    TriCtl* __restrict__ ctl) {
    pdl_wait();
    pdl_trigger();  // pass 2 may launch now and stage its (read-only) inputs meanwhile
    if (ctl->seq) return;
    for (int64_t j0 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j0 < NC;
         j0 += (int64_t)gridDim.x * blockDim.x) {
        const unsigned f0 = ts_flags(hh[j0]);
        const bool prev_split = j0 > 0 && (ts_flags(hh[j0 - 1]) & TS_SPLIT);
        if (!(f0 & TS_DEC) && !prev_split) continue;
        const bool from_split = !(f0 & TS_DEC);  // L_{j0-1} = pL + hL F_{j0}
        float u = 0.0f, v = 0.0f;
        if (from_split) {
            u = pg[j0 - 1].z;
            v = hh[j0 - 1].y;
        }
        int64_t j = j0;
        bool ok = true, end_dec = false;
        // the walk is a dependent chain; the next CB chunks' parameters are loaded as one
        // batch (independent loads) ahead of their use
        constexpr int CB = LF_TS_CB;
        float4 qb[CB], hb[CB];
        for (bool done = false; !done;) {
#pragma unroll
            for (int t = 0; t < CB; ++t) {
                if (j + t < NC) {
                    qb[t] = pg[j + t];
                    hb[t] = hh[j + t];
                }
            }
#pragma unroll
            for (int t = 0; t < CB; ++t) {
                const float4 q = qb[t];
                const float4 h = hb[t];
                const unsigned f = ts_flags(h);
                const float den = fmaf(-q.y, v, 1.0f);
                ok &= den != 0.0f;
                const float rd = rcp_nr(den);
                const float al = fmaf(q.y, u, q.x) * rd, be = h.x * rd;
                sweep[j] = make_float4(al, be, u, v);  // u, v: L_{j-1} = u + v F_j
                const float un = fmaf(q.w, fmaf(v, al, u), q.z);
                const float vn = fmaf(q.w * v, be, h.y);
                u = un;
                v = vn;
                if (f & (TS_SPLIT | TS_DECNEXT)) {
                    end_dec = (f & TS_DECNEXT) != 0;
                    done = true;
                    break;
                }
                ++j;
            }
        }
        // chain end j: F_j = alpha_j (beta_j = 0)
        float Fn = 0.0f;
#pragma unroll 4
        for (int64_t k = j; k >= j0; --k) {
            const float4 w = sweep[k];
            const float F = fmaf(w.y, Fn, w.x);
            FL[k].x = F;
            if (k > j0 || from_split) FL[k - 1].y = fmaf(w.w, F, w.z);  // L_{k-1} = u + v F_k
            Fn = F;
        }
        // L_j = u + v F_{j+1}: here if nothing follows (v = 0), else by the next chain
        if (end_dec) FL[j].y = u;
        ok &= isfinite(Fn) && isfinite(u);
        if (!ok) atomicOr(&ctl->seq, 1u);
    }
}

__global__ void __launch_bounds__(PB) k_part_pass2(int64_t N, int64_t NC,
                                                   const float* __restrict__ a,
                                                   const float* __restrict__ b,
                                                   const float* __restrict__ c,
                                                   const float* __restrict__ x,
                                                   const float2* __restrict__ FL,
                                                   float* __restrict__ y,
                                                   const TriCtl* __restrict__ ctl) {
    __shared__ ChunkSmem S;
    const int64_t r0 = (int64_t)blockIdx.x * PB * PK;
    stage_chunks(N, r0, a, b, c, x, S);  // inputs only: overlaps the chain kernel (PDL)
    __syncthreads();
    pdl_wait();
    if (ctl->seq) return;
    const int64_t j = (int64_t)blockIdx.x * PB + threadIdx.x;
    if (r0 + (int64_t)threadIdx.x * PK < N) {
        float* A = S.a + threadIdx.x * PS;
        float* B = S.b + threadIdx.x * PS;
        float* Cc = S.c + threadIdx.x * PS;
        float* X = S.x + threadIdx.x * PS;
        const float yl = j > 0 ? FL[j - 1].y : 0.0f;
        const float yr = j + 1 < NC ? FL[j + 1].x : 0.0f;
        // twisted factorisation: top-down over rows [0, H), bottom-up over [H, PK), both
        // chains interleaved; the two meet in a 2x2 system for y[H-1], y[H], then both
        // halves back-substitute outwards (serial length PK/2 + PK/2 instead of 2 PK)
        constexpr int H = PK / 2;
        const float x0 = fmaf(-A[0], yl, X[0]);
        const float xe = fmaf(-Cc[PK - 1], yr, X[PK - 1]);
        float cp = 0.0f, dx = 0.0f, cq = 0.0f, ex = 0.0f;
#pragma unroll 8
        for (int i = 0; i < H; ++i) {
            {
                const float l = (i == 0) ? 0.0f : A[i];
                const float rm = rcp_nr(fmaf(-l, cp, B[i]));
                dx = fmaf(-l, dx, (i == 0) ? x0 : X[i]) * rm;
                cp = Cc[i] * rm;
                Cc[i] = cp;
                X[i] = dx;
            }
            {
                const int k = PK - 1 - i;
                const float u = (k == PK - 1) ? 0.0f : Cc[k];
                const float rm = rcp_nr(fmaf(-u, cq, B[k]));
                ex = fmaf(-u, ex, (k == PK - 1) ? xe : X[k]) * rm;
                cq = A[k] * rm;
                A[k] = cq;
                X[k] = ex;
            }
        }
        // y[H-1] + cp y[H] = dx,  y[H] + cq y[H-1] = ex
        float zt = (dx - cp * ex) * rcp_nr(fmaf(-cp, cq, 1.0f));
        float zb = fmaf(-cq, zt, ex);
        X[H - 1] = zt;
        X[H] = zb;
#pragma unroll 8
        for (int i = 1; i < H; ++i) {
            zt = fmaf(-Cc[H - 1 - i], zt, X[H - 1 - i]);
            X[H - 1 - i] = zt;
            zb = fmaf(-A[H + i], zb, X[H + i]);
            X[H + i] = zb;
        }
    }
    __syncthreads();
    for (int k = threadIdx.x; k < PB * PK; k += PB) {
        const int64_t r = r0 + k;
        if (r < N) y[r] = S.x[(k / PK) * PS + (k % PK)];
    }
}

static inline size_t align256(size_t x) { return (x + 255) & ~(size_t)255; }

static inline int64_t n_chunks(int64_t N) { return (N + PK - 1) / PK; }

size_t trisolve_ws_bytes(int64_t N) {
    const int64_t NC = n_chunks(N);
    return 256 + align256((size_t)N * 16) + align256((size_t)NC * 16) * 3 +
           align256((size_t)NC * 8);
}

int trisolve_run(int64_t N, const float* a, const float* b, const float* c, const float* x,
                 float* y, void* ws, cudaStream_t s) {
    if (N == 0) return LF_OK;
    const int64_t NC = n_chunks(N);
    char* w = (char*)ws;
    TriCtl* ctl = (TriCtl*)w;
    w += 256;
    float4* U = (float4*)w;
    w += align256((size_t)N * 16);
    float4* pg = (float4*)w;
    w += align256((size_t)NC * 16);
    float4* sweep = (float4*)w;
    w += align256((size_t)NC * 16);
    float4* hh = (float4*)w;
    w += align256((size_t)NC * 16);
    float2* FL = (float2*)w;
    LF_CUDA(cudaMemsetAsync(ctl, 0, sizeof(TriCtl), s));
    const int pgrid = (int)((NC + PB - 1) / PB);
    {
        LF_PROF("trisolve_part1", -1, s);
        k_part_pass1<<<pgrid, PB, 0, s>>>(N, a, b, c, x, pg, hh, ctl);
        LF_CUDA(cudaGetLastError());
    }
    {
        LF_PROF("trisolve_chain", -1, s);
        const int64_t blocks = (NC + 127) / 128, cap = (int64_t)sm_count() * 16;
        LF_CUDA(launch_pdl(k_part_chain, (int)(blocks < cap ? blocks : cap), 128, 0, s, NC,
                           (const float4*)pg, (const float4*)hh, sweep, FL, ctl));
        LF_CUDA(cudaGetLastError());
    }
    {
        LF_PROF("trisolve_part2", -1, s);
        LF_CUDA(launch_pdl(k_part_pass2, pgrid, PB, 0, s, N, NC, a, b, c, x, (const float2*)FL, y,
                           (const TriCtl*)ctl));
        LF_CUDA(cudaGetLastError());
    }
    {
        LF_PROF("trisolve", -1, s);
        // a thread per segment, found by a grid-stride scan of the rows
        const int64_t blocks = (N + 127) / 128, cap = (int64_t)sm_count() * 8;
        const int grid = (int)(blocks < cap ? blocks : cap);
        LF_CUDA(launch_pdl(k_seg_solve, grid, 128, 0, s, N, a, b, c, x, (const TriCtl*)ctl, U, y));
        LF_CUDA(cudaGetLastError());
    }
    return LF_OK;
}

}  // namespace lf
