// lf_part.cu -- the factor rounds row-partitioned across GPUs.
//
// Each GPU owns a contiguous row range [lo, hi) of A (global column ids).  Setup relabels
// the columns into a local id space
//     [ghosts below lo | own rows lo..hi-1 | ghosts above hi]
// which is monotone in the global id, so the proposal keys' tie order (lower column
// index first, reading c1) is unchanged and the single-GPU kernels run as they are on
// the own rows.  Between rounds the owner of every boundary vertex sends
//   * before propose(k): its state byte (degree, round-k charge)    1 B per vertex
//   * before mutual(k):  its n proposals, translated to the receiver's local ids
// to the ranks whose rows reference it (a halo exchange; A is symmetric, so the sender
// knows its send lists from its own rows).  Rounds are synchronous, so the result is
// bit-identical to one GPU.  The exchange runs over NCCL (ncclSend/ncclRecv in a group
// on the compute stream) or, for tests, over an in-process loopback that runs G
// partitions on one GPU in lockstep.
#include <cuda_runtime.h>
#include <nccl.h>

#include <condition_variable>
#include <cstdio>
#include <cstring>
#include <cub/device/device_scan.cuh>
#include <mutex>
#include <string>
#include <thread>
#include <vector>

#include "lf_common.cuh"
#include "lf_internal.h"

namespace lf {

#define LF_NCCL(call)                                                                  \
    do {                                                                               \
        ncclResult_t r_ = (call);                                                      \
        if (r_ != ncclSuccess) {                                                       \
            char m_[256];                                                              \
            snprintf(m_, sizeof(m_), "NCCL error %s in %s", ncclGetErrorString(r_), #call); \
            return set_error(LF_ENCCL, m_);                                            \
        }                                                                              \
    } while (0)

// reusable barrier for the loopback driver's partition threads (with abort)
struct Barrier {
    std::mutex mu;
    std::condition_variable cv;
    int n = 0, waiting = 0;
    long gen = 0;
    bool aborted = false;
    bool wait() {
        std::unique_lock<std::mutex> lk(mu);
        if (aborted) return false;
        const long g = gen;
        if (++waiting == n) {
            waiting = 0;
            gen++;
            cv.notify_all();
            return true;
        }
        cv.wait(lk, [&] { return gen != g || aborted; });
        return !aborted;
    }
    void abort() {
        std::lock_guard<std::mutex> lk(mu);
        aborted = true;
        cv.notify_all();
    }
};

struct Part;

struct Comm {
    int kind = 0;  // 0: NCCL (one partition per process), 1: loopback (all partitions here)
    ncclComm_t nccl = nullptr;
    int nranks = 1, rank = 0;
    std::vector<Part*> parts;  // loopback: all partitions of the current run
    Barrier bar;
    bool own_nccl = false;
};

struct Part {
    int G = 1, rank = 0, n = 2;
    int64_t N = 0, lo = 0, hi = 0, n_own = 0, nnz = 0;
    int64_t nb = 0, na = 0, NL = 0;
    std::vector<int64_t> bounds;
    // device
    const int64_t* rowptr = nullptr;
    const float* val = nullptr;
    int32_t* col_local = nullptr;
    int32_t* l2g = nullptr;
    int32_t* send_idx = nullptr;   // local ids of own vertices to send, grouped by peer
    int8_t* send_peer = nullptr;   // destination rank per send entry
    int64_t* dpeer = nullptr;      // [3G]: lo, hi, nb of every rank (device copy)
    unsigned char* sbuf = nullptr;
    int32_t* pi = nullptr;
    float* pi_w = nullptr;
    float* pi_val = nullptr;
    float* diag = nullptr;
    int32_t* rounds = nullptr;
    int64_t* live = nullptr;
    void* ws = nullptr;
    size_t ws_bytes = 0;
    // host exchange plan
    std::vector<int64_t> send_off, send_cnt;  // per peer: first entry in send_idx, count
    std::vector<int64_t> recv_lid, recv_cnt;  // per peer: first local id of its ghosts, count
    std::vector<int64_t> peer_lo, peer_hi, peer_nb;
    int64_t send_total = 0;
    bool plan_checked = false;
    int32_t* ghost_list = nullptr;  // sorted global ids of ghosts
    int64_t n_ghost = 0;
    std::vector<int64_t> peer_send_total;
    // linear forest
    int32_t* pi2g = nullptr;     // [n_own*2] own factor slots, global ids (n = 2)
    float* pi2w = nullptr;
    float* pi2v = nullptr;
    float* pdiag = nullptr;
    int2* ghost_pi = nullptr;    // [NL] factor slots of ghosts (global ids)
    int32_t* ghost_iperm = nullptr;
    int32_t *forest = nullptr, *path_id = nullptr, *pos = nullptr, *iperm = nullptr;
    int64_t* n_cycles = nullptr;
    void* lws = nullptr;
    size_t lws_bytes = 0;
    ForestWs lw;
    ForestPartCtx fpc;
    bool lf_ready = false;
    // run
    Comm* comm = nullptr;
    FactorWs fws;
    int M = 5;
    std::vector<void*> allocs;
};

template <class T>
static int dalloc(Part* p, T** ptr, size_t count, cudaStream_t s) {
    void* q = nullptr;
    LF_CUDA(cudaMallocAsync(&q, (count ? count : 1) * sizeof(T), s));
    p->allocs.push_back(q);
    *ptr = (T*)q;
    return LF_OK;
}

// ---------------------------------------------------------------------------
// setup kernels
// ---------------------------------------------------------------------------
__global__ void k_mark_ghosts(int64_t nnz, const int32_t* __restrict__ col, int64_t lo, int64_t hi,
                              uint32_t* bits) {
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < nnz; e += (int64_t)gridDim.x * blockDim.x) {
        const int32_t j = col[e];
        if (j < lo || j >= hi) atomicOr(&bits[j >> 5], 1u << (j & 31));
    }
}

__global__ void k_popc(int64_t W, const uint32_t* __restrict__ bits, int32_t* pc) {
    for (int64_t w = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; w < W; w += (int64_t)gridDim.x * blockDim.x)
        pc[w] = __popc(bits[w]);
}

__device__ __forceinline__ int32_t bit_rank(const uint32_t* bits, const int32_t* wpre, int32_t x) {
    return wpre[x >> 5] + __popc(bits[x >> 5] & ((1u << (x & 31)) - 1u));
}

__global__ void k_ghost_list(int64_t W, const uint32_t* __restrict__ bits, const int32_t* __restrict__ wpre,
                             int32_t* ghost) {
    for (int64_t w = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; w < W; w += (int64_t)gridDim.x * blockDim.x) {
        uint32_t b = bits[w];
        int32_t r = wpre[w];
        while (b) {
            const int i = __ffs(b) - 1;
            ghost[r++] = (int32_t)(w * 32 + i);
            b &= b - 1;
        }
    }
}

// lower_bound of each of the G+1 rank bounds in the sorted ghost list
__global__ void k_ghost_bounds(const int32_t* __restrict__ ghost, int64_t ng, const int64_t* __restrict__ bounds,
                               int G, int64_t* out) {
    const int q = threadIdx.x;
    if (q > G) return;
    int64_t a = 0, b = ng;
    const int64_t x = bounds[q];
    while (a < b) {
        const int64_t m = (a + b) / 2;
        if (ghost[m] < x) a = m + 1; else b = m;
    }
    out[q] = a;
}

__global__ void k_l2g(int64_t NL, int64_t nb, int64_t n_own, int64_t lo, const int32_t* __restrict__ ghost,
                      int32_t* l2g) {
    for (int64_t L = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; L < NL; L += (int64_t)gridDim.x * blockDim.x) {
        if (L < nb) l2g[L] = ghost[L];
        else if (L < nb + n_own) l2g[L] = (int32_t)(lo + (L - nb));
        else l2g[L] = ghost[L - n_own];
    }
}

__global__ void k_relabel(int64_t nnz, const int32_t* __restrict__ col, int64_t lo, int64_t hi, int64_t nb,
                          int64_t n_own, const uint32_t* __restrict__ bits, const int32_t* __restrict__ wpre,
                          int32_t* col_local) {
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < nnz; e += (int64_t)gridDim.x * blockDim.x) {
        const int32_t j = col[e];
        if (j >= lo && j < hi) col_local[e] = (int32_t)(nb + (j - lo));
        else {
            const int32_t r = bit_rank(bits, wpre, j);
            col_local[e] = r < nb ? r : (int32_t)(r + n_own);
        }
    }
}

__device__ __forceinline__ int owner_of(int64_t j, const int64_t* bounds, int G) {
    int q = 0;
    while (q + 1 < G && j >= bounds[q + 1]) q++;
    return q;
}

// flags[q * n_own + r] = 1 if own row r references a column of rank q (q != rank)
__global__ void k_mark_send(int64_t n_own, const int64_t* __restrict__ rowptr, const int32_t* __restrict__ col,
                            const int64_t* __restrict__ bounds, int G, int rank, int32_t* flags) {
    for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < n_own; r += (int64_t)gridDim.x * blockDim.x) {
        for (int64_t e = rowptr[r]; e < rowptr[r + 1]; e++) {
            const int q = owner_of(col[e], bounds, G);
            if (q != rank) flags[(int64_t)q * n_own + r] = 1;
        }
    }
}

__global__ void k_compact_send(int64_t total, int64_t n_own, int64_t nb, const int32_t* __restrict__ flags,
                               const int32_t* __restrict__ pos, int32_t* send_idx, int8_t* send_peer) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
        if (flags[i]) {
            const int64_t q = i / n_own, r = i - q * n_own;
            send_idx[pos[i]] = (int32_t)(nb + r);
            send_peer[pos[i]] = (int8_t)q;
        }
    }
}

// ---------------------------------------------------------------------------
// halo packing
// ---------------------------------------------------------------------------
__global__ void k_pack_state(int64_t cnt, const int32_t* __restrict__ idx, const uint8_t* __restrict__ state,
                             uint8_t* out) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < cnt; i += (int64_t)gridDim.x * blockDim.x)
        out[i] = state[idx[i]];
}

// proposals of boundary vertices, as the receiver's local ids (-1: not a receiver vertex)
__global__ void k_pack_prop(int64_t cnt, int n, const int32_t* __restrict__ idx, const int8_t* __restrict__ peer,
                            const int32_t* __restrict__ prop_j, const int32_t* __restrict__ l2g,
                            const int64_t* __restrict__ dpeer, int G, int32_t* out) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < cnt; i += (int64_t)gridDim.x * blockDim.x) {
        const int32_t v = idx[i];
        const int q = peer[i];
        const int64_t qlo = dpeer[q], qhi = dpeer[G + q], qnb = dpeer[2 * G + q];
        for (int s = 0; s < n; s++) {
            const int32_t x = prop_j[(int64_t)v * n + s];
            int32_t y = -1;
            if (x >= 0) {
                const int64_t g = l2g[x];
                if (g >= qlo && g < qhi) y = (int32_t)(g - qlo + qnb);
            }
            out[i * n + s] = y;
        }
    }
}

// loopback reduction of the per-round flags (max) and live counters (sum)
__global__ void k_reduce_parts(int P, int M, int** flags, unsigned long long** live) {
    for (int i = threadIdx.x; i < M; i += blockDim.x) {
        int f = 0;
        for (int p = 0; p < P; p++) f = max(f, flags[p][i]);
        for (int p = 0; p < P; p++) flags[p][i] = f;
    }
    if (live[0]) {
        for (int i = threadIdx.x; i < M * 128; i += blockDim.x) {
            unsigned long long t = 0;
            for (int p = 0; p < P; p++) t += live[p][i];
            for (int p = 0; p < P; p++) live[p][i] = t;
        }
    }
}

// ---------------------------------------------------------------------------
// exchange
// ---------------------------------------------------------------------------
static int check_plan(Part* p, cudaStream_t s) {
    // the counts p sends to q must be what q expects from p (symmetric pattern)
    Comm* c = p->comm;
    if (p->plan_checked) return LF_OK;
    if (c->kind == 1) {
        p->peer_send_total.assign(p->G, 0);
        for (int q = 0; q < p->G; q++) {
            Part* o = c->parts[q];
            p->peer_send_total[q] = o->send_total;
            if (q == p->rank) continue;
            if (p->send_cnt[q] != o->recv_cnt[p->rank])
                return set_error(LF_EINPUT, "partition plan mismatch: A is not pattern-symmetric");
            p->peer_nb[q] = o->nb;
        }
    } else {
        const int G = p->G;
        int64_t *dsend = nullptr, *dall = nullptr;
        LF_CUDA(cudaMalloc(&dsend, sizeof(int64_t) * (G + 1)));
        LF_CUDA(cudaMalloc(&dall, sizeof(int64_t) * (G + 1) * G));
        std::vector<int64_t> mine(G + 1);
        for (int q = 0; q < G; q++) mine[q] = p->send_cnt[q];
        mine[G] = p->nb;
        // on the caller's stream (not the legacy default stream), then one host sync
        LF_CUDA(cudaMemcpyAsync(dsend, mine.data(), sizeof(int64_t) * (G + 1), cudaMemcpyHostToDevice, s));
        LF_NCCL(ncclAllGather(dsend, dall, G + 1, ncclInt64, c->nccl, s));
        std::vector<int64_t> all((size_t)(G + 1) * G);
        LF_CUDA(cudaMemcpyAsync(all.data(), dall, sizeof(int64_t) * all.size(), cudaMemcpyDeviceToHost, s));
        LF_CUDA(cudaStreamSynchronize(s));
        cudaFree(dsend);
        cudaFree(dall);
        p->peer_send_total.assign(G, 0);
        for (int q = 0; q < G; q++) {
            for (int r = 0; r < G; r++) p->peer_send_total[q] += all[(size_t)q * (G + 1) + r];
            p->peer_nb[q] = all[(size_t)q * (G + 1) + G];
            if (q != p->rank && all[(size_t)q * (G + 1) + p->rank] != p->recv_cnt[q])
                return set_error(LF_EINPUT, "partition plan mismatch: A is not pattern-symmetric");
        }
    }
    std::vector<int64_t> h(3 * p->G);
    for (int q = 0; q < p->G; q++) {
        h[q] = p->peer_lo[q];
        h[p->G + q] = p->peer_hi[q];
        h[2 * p->G + q] = p->peer_nb[q];
    }
    LF_CUDA(cudaMemcpy(p->dpeer, h.data(), sizeof(int64_t) * h.size(), cudaMemcpyHostToDevice));
    p->plan_checked = true;
    return LF_OK;
}

// move B bytes per entry: p's send buffer (grouped by peer) -> peers' dst + recv_lid * B
static int exchange(Part* p, unsigned char* dst, size_t B, cudaStream_t s) {
    Comm* c = p->comm;
    if (c->kind == 0) {
        LF_NCCL(ncclGroupStart());
        for (int q = 0; q < p->G; q++) {
            if (q == p->rank) continue;
            if (p->send_cnt[q])
                LF_NCCL(ncclSend(p->sbuf + p->send_off[q] * B, p->send_cnt[q] * B, ncclUint8, q, c->nccl, s));
            if (p->recv_cnt[q])
                LF_NCCL(ncclRecv(dst + p->recv_lid[q] * B, p->recv_cnt[q] * B, ncclUint8, q, c->nccl, s));
        }
        LF_NCCL(ncclGroupEnd());
        return LF_OK;
    }
    // loopback: every partition packed (barrier), copy the inbound slices, barrier
    if (!c->bar.wait()) return set_error(LF_ECUDA, "loopback exchange aborted");
    for (int q = 0; q < p->G; q++) {
        if (q == p->rank || !p->recv_cnt[q]) continue;
        Part* o = c->parts[q];
        LF_CUDA(cudaMemcpyAsync(dst + p->recv_lid[q] * B, o->sbuf + o->send_off[p->rank] * B, p->recv_cnt[q] * B,
                                cudaMemcpyDeviceToDevice, s));
    }
    if (!c->bar.wait()) return set_error(LF_ECUDA, "loopback exchange aborted");
    return LF_OK;
}

static int hook_pre_propose(void* ctx, int k, cudaStream_t s) {
    Part* p = (Part*)ctx;
    (void)k;
    if (p->send_total) {
        k_pack_state<<<persistent_grid((const void*)k_pack_state, 256), 256, 0, s>>>(p->send_total, p->send_idx,
                                                                                 p->fws.state, p->sbuf);
        LF_CUDA(cudaGetLastError());
    }
    LF_PROF("halo_state", k, s);
    return exchange(p, p->fws.state, 1, s);
}

static int hook_pre_mutual(void* ctx, int k, cudaStream_t s) {
    Part* p = (Part*)ctx;
    if (p->send_total) {
        k_pack_prop<<<persistent_grid((const void*)k_pack_prop, 256), 256, 0, s>>>(
            p->send_total, p->n, p->send_idx, p->send_peer, p->fws.prop_j, p->l2g, p->dpeer, p->G,
            (int32_t*)p->sbuf);
        LF_CUDA(cudaGetLastError());
    }
    LF_PROF("halo_prop", k, s);
    return exchange(p, (unsigned char*)p->fws.prop_j, sizeof(int32_t) * p->n, s);
}

static int hook_pre_finalize(void* ctx, cudaStream_t s) {
    Part* p = (Part*)ctx;
    Comm* c = p->comm;
    if (c->kind == 0) {
        LF_NCCL(ncclGroupStart());
        LF_NCCL(ncclAllReduce(p->fws.flags, p->fws.flags, p->M, ncclInt32, ncclMax, c->nccl, s));
        LF_NCCL(ncclAllReduce(p->fws.live_part, p->fws.live_part, (size_t)p->M * 128, ncclUint64, ncclSum,
                              c->nccl, s));
        LF_NCCL(ncclGroupEnd());
        return LF_OK;
    }
    if (!c->bar.wait()) return set_error(LF_ECUDA, "loopback reduce aborted");
    if (p->rank == 0) {
        const int P = (int)c->parts.size();
        std::vector<int*> f(P);
        std::vector<unsigned long long*> l(P);
        for (int q = 0; q < P; q++) {
            f[q] = c->parts[q]->fws.flags;
            l[q] = c->parts[q]->live ? c->parts[q]->fws.live_part : nullptr;
        }
        int** df = nullptr;
        unsigned long long** dl = nullptr;
        LF_CUDA(cudaMallocAsync(&df, sizeof(int*) * P, s));
        LF_CUDA(cudaMallocAsync(&dl, sizeof(void*) * P, s));
        LF_CUDA(cudaMemcpyAsync(df, f.data(), sizeof(int*) * P, cudaMemcpyHostToDevice, s));
        LF_CUDA(cudaMemcpyAsync(dl, l.data(), sizeof(void*) * P, cudaMemcpyHostToDevice, s));
        k_reduce_parts<<<1, 256, 0, s>>>(P, p->M, df, dl);
        LF_CUDA(cudaGetLastError());
        LF_CUDA(cudaFreeAsync(df, s));
        LF_CUDA(cudaFreeAsync(dl, s));
        LF_CUDA(cudaStreamSynchronize(s));  // host vectors go out of scope
    }
    if (!c->bar.wait()) return set_error(LF_ECUDA, "loopback reduce aborted");
    return LF_OK;
}

static int run_factor(Part* p, const lf_factor_opts_t* o, cudaStream_t s) {
    int rc = check_plan(p, s);
    if (rc) return rc;
    lf_csr_t A{p->n_own, p->nnz, p->rowptr, p->col_local, p->val};
    PartCtx pc;
    pc.row_base = p->nb;
    pc.gid_off = p->lo - p->nb;
    pc.NL = p->NL;
    pc.l2g = p->l2g;
    pc.ctx = p;
    pc.pre_propose = hook_pre_propose;
    pc.pre_mutual = hook_pre_mutual;
    pc.pre_finalize = hook_pre_finalize;
    p->M = o->M;
    return factor_dispatch(&A, p->n, o, p->pi, p->pi_w, p->pi_val, p->diag, p->rounds, p->live, p->fws, s, &pc);
}

__global__ void k_export(int64_t n_own, int n, int64_t nb, const int32_t* __restrict__ pi,
                         const float* __restrict__ pi_w, const float* __restrict__ pi_val,
                         const float* __restrict__ diag, const int32_t* __restrict__ l2g, int32_t* opi, float* opw,
                         float* opv, float* odiag) {
    for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < n_own; r += (int64_t)gridDim.x * blockDim.x) {
        const int64_t v = nb + r;
        for (int s = 0; s < n; s++) {
            const int32_t x = pi[v * n + s];
            if (opi) opi[r * n + s] = x >= 0 ? l2g[x] : -1;
            if (opw) opw[r * n + s] = pi_w[v * n + s];
            if (opv) opv[r * n + s] = pi_val[v * n + s];
        }
        if (odiag) odiag[r] = diag[v];
    }
}


// ---------------------------------------------------------------------------
// partitioned linear forest
// ---------------------------------------------------------------------------
__global__ void k_pack_pi(int64_t cnt, const int32_t* __restrict__ idx, int64_t nb, const int2* __restrict__ pi2g,
                          int2* out) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < cnt; i += (int64_t)gridDim.x * blockDim.x)
        out[i] = pi2g[idx[i] - nb];
}

__global__ void k_pack_i32(int64_t cnt, const int32_t* __restrict__ idx, int64_t nb, const int32_t* __restrict__ own,
                           int32_t* out) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < cnt; i += (int64_t)gridDim.x * blockDim.x)
        out[i] = own[idx[i] - nb];
}

__global__ void k_sum_parts_i64(int P, int count, int64_t** bufs) {
    for (int i = threadIdx.x; i < count; i += blockDim.x) {
        int64_t t = 0;
        for (int p = 0; p < P; p++) t += bufs[p][i];
        for (int p = 0; p < P; p++) bufs[p][i] = t;
    }
}

static int cb_allgather(void* ctx, const void* send, void* recv, size_t bytes, cudaStream_t s) {
    Part* p = (Part*)ctx;
    Comm* c = p->comm;
    if (c->kind == 0) {
        LF_NCCL(ncclAllGather(send, recv, bytes, ncclUint8, c->nccl, s));
        return LF_OK;
    }
    // loopback: every partition's send buffer is at the same place in its own context;
    // copy all of them into this partition's receive buffer (ordering by barriers)
    if (!c->bar.wait()) return set_error(LF_ECUDA, "loopback allgather aborted");
    const bool is_rec = send == p->fpc.rec_send;  // exit records, or published offsets
    if (!is_rec && send != (const void*)p->fpc.pub_send)
        return set_error(LF_EINVAL, "loopback allgather: unknown buffer");
    for (int q = 0; q < p->G; q++) {
        Part* o = c->parts[q];
        const void* src = is_rec ? o->fpc.rec_send : (const void*)o->fpc.pub_send;
        LF_CUDA(cudaMemcpyAsync((char*)recv + (size_t)q * bytes, src, bytes, cudaMemcpyDeviceToDevice, s));
    }
    if (!c->bar.wait()) return set_error(LF_ECUDA, "loopback allgather aborted");
    return LF_OK;
}

static int cb_allreduce_i64(void* ctx, int64_t* buf, int count, cudaStream_t s) {
    Part* p = (Part*)ctx;
    Comm* c = p->comm;
    if (c->kind == 0) {
        LF_NCCL(ncclAllReduce(buf, buf, count, ncclInt64, ncclSum, c->nccl, s));
        return LF_OK;
    }
    if (!c->bar.wait()) return set_error(LF_ECUDA, "loopback allreduce aborted");
    if (p->rank == 0) {
        const int P = (int)c->parts.size();
        const size_t off = buf - p->fpc.tot;
        std::vector<int64_t*> b(P);
        for (int q = 0; q < P; q++) b[q] = c->parts[q]->fpc.tot + off;
        int64_t** db = nullptr;
        LF_CUDA(cudaMallocAsync(&db, sizeof(void*) * P, s));
        LF_CUDA(cudaMemcpyAsync(db, b.data(), sizeof(void*) * P, cudaMemcpyHostToDevice, s));
        k_sum_parts_i64<<<1, 64, 0, s>>>(P, count, db);
        LF_CUDA(cudaGetLastError());
        LF_CUDA(cudaFreeAsync(db, s));
        LF_CUDA(cudaStreamSynchronize(s));
    }
    if (!c->bar.wait()) return set_error(LF_ECUDA, "loopback allreduce aborted");
    return LF_OK;
}

static int lf_setup(Part* p, cudaStream_t s) {
    if (p->lf_ready) return LF_OK;
    if (p->n != 2) return set_error(LF_EINVAL, "partitioned linear forest needs n = 2");
    const int64_t no = p->n_own > 0 ? p->n_own : 1;
    int rc;
#define TRYL(x) do { rc = (x); if (rc) return rc; } while (0)
    TRYL(dalloc(p, &p->pi2g, (size_t)no * 2, s));
    TRYL(dalloc(p, &p->pi2w, (size_t)no * 2, s));
    TRYL(dalloc(p, &p->pi2v, (size_t)no * 2, s));
    TRYL(dalloc(p, &p->pdiag, (size_t)no, s));
    TRYL(dalloc(p, &p->ghost_pi, (size_t)p->NL, s));
    TRYL(dalloc(p, &p->ghost_iperm, (size_t)p->NL, s));
    TRYL(dalloc(p, &p->forest, (size_t)no * 2, s));
    TRYL(dalloc(p, &p->path_id, (size_t)no, s));
    TRYL(dalloc(p, &p->pos, (size_t)no, s));
    TRYL(dalloc(p, &p->iperm, (size_t)no, s));
    TRYL(dalloc(p, &p->n_cycles, 1, s));
    {
        Carve c(nullptr, 0);
        p->lws_bytes = forest_ws_carve(c, no, nullptr, false) + 256;
        char* w = nullptr;
        TRYL(dalloc(p, &w, p->lws_bytes, s));
        p->lws = w;
        Carve c2(p->lws, p->lws_bytes);
        forest_ws_carve(c2, no, &p->lw, false);
    }
    ForestPartCtx& f = p->fpc;
    memset(&f, 0, sizeof(f));
    f.lo = p->lo;
    f.hi = p->hi;
    f.G = p->G;
    f.rank = p->rank;
    f.ghost_list = p->ghost_list;
    f.n_ghost = p->n_ghost;
    f.ghost_below = p->nb;
    f.ghost_nb = p->ghost_pi;
    int64_t cap = 1;
    for (int q = 0; q < p->G; q++) cap = p->peer_send_total[q] > cap ? p->peer_send_total[q] : cap;
    f.exit_cap = cap;
    const size_t N = (size_t)p->N + 1;
    for (int i = 0; i < 2; i++) {
        TRYL(dalloc(p, &f.gq[i], N, s));
        TRYL(dalloc(p, &f.gk[i], N, s));
        TRYL(dalloc(p, &f.gr[i], N, s));
    }
    const size_t NG = N > (size_t)p->G * cap ? N : (size_t)p->G * cap;  // glist positions
    TRYL(dalloc(p, &f.gcyc, NG, s));
    TRYL(dalloc(p, &f.gend, NG, s));
    TRYL(dalloc(p, &f.gdist, NG, s));
    TRYL(dalloc(p, &f.gbidx, N, s));
    TRYL(dalloc(p, &f.glist, (size_t)p->G * cap, s));
    TRYL(dalloc(p, &f.gcq, (size_t)p->G * cap, s));
    TRYL(dalloc(p, &f.gcq_k, (size_t)p->G * cap, s));
    TRYL(dalloc(p, &f.gctl, 256, s));
    char* rs = nullptr;
    TRYL(dalloc(p, &rs, exit_record_bytes() * cap, s));
    f.rec_send = rs;
    char* ra = nullptr;
    TRYL(dalloc(p, &ra, exit_record_bytes() * cap * p->G, s));
    f.rec_all = ra;
    TRYL(dalloc(p, &f.pub_send, (size_t)cap, s));
    TRYL(dalloc(p, &f.pub_all, (size_t)cap * p->G, s));
    TRYL(dalloc(p, &f.offG, N, s));
    TRYL(dalloc(p, &f.tot, (size_t)p->G + 2, s));
    f.ctx = p;
    f.allgather = cb_allgather;
    f.allreduce_i64 = cb_allreduce_i64;
#undef TRYL
    p->lf_ready = true;
    return LF_OK;
}

static int run_forest(Part* p, cudaStream_t s) {
    int rc = check_plan(p, s);
    if (rc) return rc;
    rc = lf_setup(p, s);
    if (rc) return rc;
    // own factor with global ids, and the factor slots of ghost vertices (halo)
    if (p->n_own > 0) {
        k_export<<<persistent_grid((const void*)k_export, 256), 256, 0, s>>>(p->n_own, 2, p->nb, p->pi, p->pi_w,
                                                                           p->pi_val, p->diag, p->l2g, p->pi2g,
                                                                           p->pi2w, p->pi2v, p->pdiag);
        LF_CUDA(cudaGetLastError());
    }
    if (p->send_total) {
        k_pack_pi<<<persistent_grid((const void*)k_pack_pi, 256), 256, 0, s>>>(p->send_total, p->send_idx, p->nb,
                                                                           (const int2*)p->pi2g, (int2*)p->sbuf);
        LF_CUDA(cudaGetLastError());
    }
    {
        LF_PROF("halo_pi", -1, s);
        rc = exchange(p, (unsigned char*)p->ghost_pi, sizeof(int2), s);
        if (rc) return rc;
    }
    return forest_part_run(p->N, p->pi2g, p->pi2w, p->forest, p->path_id, p->pos, p->iperm, p->n_cycles, p->lw,
                           p->fpc, s);
}

// tridiagonal coefficients of the own vertices (row iperm[v]); foreign neighbours' rows
// come from a halo exchange of iperm
__global__ void k_part_tridiag(int64_t lo, int64_t hi, const int2* __restrict__ forest, const int32_t* __restrict__ iperm,
                               const int2* __restrict__ pi2g, const float2* __restrict__ pi2v,
                               const float* __restrict__ diag, const int32_t* __restrict__ ghost_list, int64_t ng,
                               int64_t nbelow, const int32_t* __restrict__ ghost_iperm, float* a, float* b, float* c) {
    for (int64_t v = lo + (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < hi; v += (int64_t)gridDim.x * blockDim.x) {
        const int64_t i = v - lo;
        const int32_t r = iperm[i];
        const int2 f = forest[i];
        const int2 pn = pi2g[i];
        const float2 pv = pi2v[i];
        float ar = 0.0f, cr = 0.0f;
#pragma unroll
        for (int k = 0; k < 2; k++) {
            const int32_t w = k ? f.y : f.x;
            if (w < 0) continue;
            const float x = (pn.x == w) ? pv.x : pv.y;
            int32_t rw;
            if (w >= lo && w < hi) rw = iperm[w - lo];
            else {
                int64_t l = 0, h = ng;
                while (l < h) {
                    const int64_t m = (l + h) >> 1;
                    if (ghost_list[m] < w) l = m + 1; else h = m;
                }
                rw = ghost_iperm[l < nbelow ? l : l + (hi - lo)];
            }
            if (rw == r - 1) ar = x;
            else if (rw == r + 1) cr = x;
        }
        a[i] = ar;
        b[i] = diag[i];
        c[i] = cr;
    }
}

static int run_tridiag(Part* p, float* a, float* b, float* c, cudaStream_t s) {
    if (!p->lf_ready) return set_error(LF_EINVAL, "lf_part_tridiag: run lf_part_linear_forest first");
    if (p->send_total) {
        k_pack_i32<<<persistent_grid((const void*)k_pack_i32, 256), 256, 0, s>>>(p->send_total, p->send_idx, p->nb,
                                                                             p->iperm, (int32_t*)p->sbuf);
        LF_CUDA(cudaGetLastError());
    }
    int rc = exchange(p, (unsigned char*)p->ghost_iperm, sizeof(int32_t), s);
    if (rc) return rc;
    if (p->n_own > 0) {
        LF_PROF("tridiag", -1, s);
        k_part_tridiag<<<persistent_grid((const void*)k_part_tridiag, 256), 256, 0, s>>>(
            p->lo, p->hi, (const int2*)p->forest, p->iperm, (const int2*)p->pi2g, (const float2*)p->pi2v, p->pdiag,
            p->ghost_list, p->n_ghost, p->nb, p->ghost_iperm, a, b, c);
        LF_CUDA(cudaGetLastError());
    }
    return LF_OK;
}

// run fn on every partition of this process (loopback: lockstep threads)
template <class F>
static int for_parts(void** parts, int nparts, Comm* c, F fn) {
    if (c->kind == 0) {
        Part* p = (Part*)parts[0];
        p->comm = c;
        return fn(p);
    }
    c->parts.assign(nparts, nullptr);
    for (int i = 0; i < nparts; i++) {
        Part* p = (Part*)parts[i];
        c->parts[p->rank] = p;
        p->comm = c;
    }
    c->bar.n = nparts;
    c->bar.aborted = false;
    int dev = 0;
    cudaGetDevice(&dev);
    std::vector<int> rcs(nparts, 0);
    std::vector<std::string> errs(nparts);
    std::vector<std::thread> th;
    for (int i = 0; i < nparts; i++) {
        th.emplace_back([&, i] {
            cudaSetDevice(dev);
            const int rc = fn(c->parts[i]);
            if (rc) {
                errs[i] = lf_last_error();
                c->bar.abort();
            }
            rcs[i] = rc;
        });
    }
    for (auto& t : th) t.join();
    for (int i = 0; i < nparts; i++)
        if (rcs[i]) return set_error(rcs[i], errs[i].c_str());
    return LF_OK;
}

}  // namespace lf

using namespace lf;

extern "C" {

int lf_comm_nccl_unique_id(void* id128) {
    if (!id128) return set_error(LF_EINVAL, "lf_comm_nccl_unique_id: NULL");
    ncclUniqueId id;
    LF_NCCL(ncclGetUniqueId(&id));
    memcpy(id128, &id, sizeof(id));
    return LF_OK;
}

int lf_comm_create_nccl(const void* id128, int nranks, int rank, void** out) {
    if (!id128 || !out || nranks < 1 || rank < 0 || rank >= nranks)
        return set_error(LF_EINVAL, "lf_comm_create_nccl: bad arguments");
    Comm* c = new Comm();
    c->kind = 0;
    c->nranks = nranks;
    c->rank = rank;
    ncclUniqueId id;
    memcpy(&id, id128, sizeof(id));
    ncclResult_t r = ncclCommInitRank(&c->nccl, nranks, id, rank);
    if (r != ncclSuccess) {
        delete c;
        char m[256];
        snprintf(m, sizeof(m), "ncclCommInitRank: %s", ncclGetErrorString(r));
        return set_error(LF_ENCCL, m);
    }
    c->own_nccl = true;
    *out = c;
    return LF_OK;
}

int lf_comm_create_loopback(int nparts, void** out) {
    if (!out || nparts < 1) return set_error(LF_EINVAL, "lf_comm_create_loopback: bad arguments");
    Comm* c = new Comm();
    c->kind = 1;
    c->nranks = nparts;
    *out = c;
    return LF_OK;
}

int lf_comm_destroy(void* comm) {
    Comm* c = (Comm*)comm;
    if (!c) return LF_OK;
    if (c->own_nccl && c->nccl) ncclCommDestroy(c->nccl);
    delete c;
    return LF_OK;
}

int lf_part_create(int G, const int64_t* bounds, int rank, const lf_csr_t* A, int n, void** out, void* stream) {
    g_err_clear();
    if (G < 1 || G > 127 || !bounds || rank < 0 || rank >= G || !A || !out || n < 1 || n > 4)
        return set_error(LF_EINVAL, "lf_part_create: bad arguments");
    cudaStream_t s = (cudaStream_t)stream;
    Part* p = new Part();
    p->G = G;
    p->rank = rank;
    p->n = n;
    p->bounds.assign(bounds, bounds + G + 1);
    p->N = bounds[G];
    p->lo = bounds[rank];
    p->hi = bounds[rank + 1];
    p->n_own = p->hi - p->lo;
    p->nnz = A->nnz;
    p->rowptr = A->rowptr;
    p->val = A->val;
    if (A->n != p->n_own || p->N >= ((int64_t)1 << 31)) {
        delete p;
        return set_error(LF_EINVAL, "lf_part_create: A->n must equal bounds[rank+1]-bounds[rank]");
    }
    for (int q = 0; q < G; q++) {
        p->peer_lo.push_back(bounds[q]);
        p->peer_hi.push_back(bounds[q + 1]);
        p->peer_nb.push_back(0);
    }
    auto fail = [&](int rc) {
        for (void* a : p->allocs) cudaFreeAsync(a, s);
        delete p;
        return rc;
    };
#define TRY(x)                       \
    do {                             \
        int rc_ = (x);               \
        if (rc_) return fail(rc_);   \
    } while (0)
    const int64_t W = (p->N + 31) / 32;
    uint32_t* bits = nullptr;
    int32_t *pc = nullptr, *wpre = nullptr, *ghost = nullptr;
    int64_t *dbounds = nullptr, *gb = nullptr;
    TRY(set_cuda_rc(cudaMallocAsync(&bits, sizeof(uint32_t) * (W + 1), s), "alloc"));
    TRY(set_cuda_rc(cudaMallocAsync(&pc, sizeof(int32_t) * (W + 1), s), "alloc"));
    TRY(set_cuda_rc(cudaMallocAsync(&wpre, sizeof(int32_t) * (W + 1), s), "alloc"));
    TRY(set_cuda_rc(cudaMallocAsync(&dbounds, sizeof(int64_t) * (G + 1), s), "alloc"));
    TRY(set_cuda_rc(cudaMallocAsync(&gb, sizeof(int64_t) * (G + 1), s), "alloc"));
    TRY(set_cuda_rc(cudaMemcpyAsync(dbounds, bounds, sizeof(int64_t) * (G + 1), cudaMemcpyHostToDevice, s), "copy"));
    TRY(set_cuda_rc(cudaMemsetAsync(bits, 0, sizeof(uint32_t) * (W + 1), s), "memset"));
    const int grid = 148 * 8;
    k_mark_ghosts<<<grid, 256, 0, s>>>(p->nnz, A->col, p->lo, p->hi, bits);
    k_popc<<<grid, 256, 0, s>>>(W + 1, bits, pc);
    {
        size_t tb = 0;
        cub::DeviceScan::ExclusiveSum(nullptr, tb, pc, wpre, (int)(W + 1), s);
        void* tmp = nullptr;
        TRY(set_cuda_rc(cudaMallocAsync(&tmp, tb + 16, s), "alloc"));
        TRY(set_cuda_rc(cub::DeviceScan::ExclusiveSum(tmp, tb, pc, wpre, (int)(W + 1), s), "scan"));
        cudaFreeAsync(tmp, s);
    }
    int32_t ng32 = 0;
    TRY(set_cuda_rc(cudaMemcpyAsync(&ng32, wpre + W, sizeof(int32_t), cudaMemcpyDeviceToHost, s), "copy"));
    TRY(set_cuda_rc(cudaStreamSynchronize(s), "sync"));
    const int64_t ng = ng32;
    TRY(dalloc(p, &ghost, (size_t)(ng + 1), s));
    p->ghost_list = ghost;
    p->n_ghost = ng;
    k_ghost_list<<<grid, 256, 0, s>>>(W + 1, bits, wpre, ghost);
    k_ghost_bounds<<<1, 128, 0, s>>>(ghost, ng, dbounds, G, gb);
    std::vector<int64_t> hgb(G + 1);
    TRY(set_cuda_rc(cudaMemcpyAsync(hgb.data(), gb, sizeof(int64_t) * (G + 1), cudaMemcpyDeviceToHost, s), "copy"));
    TRY(set_cuda_rc(cudaStreamSynchronize(s), "sync"));
    p->nb = hgb[rank];
    p->na = ng - p->nb;
    p->NL = ng + p->n_own;
    // recv plan: ghosts of rank q are the sorted ghost ranks [hgb[q], hgb[q+1])
    p->recv_lid.assign(G, 0);
    p->recv_cnt.assign(G, 0);
    for (int q = 0; q < G; q++) {
        if (q == rank) continue;
        const int64_t a = hgb[q], b = hgb[q + 1];
        p->recv_cnt[q] = b - a;
        p->recv_lid[q] = a < p->nb ? a : a + p->n_own;
    }
    TRY(dalloc(p, &p->l2g, (size_t)p->NL, s));
    TRY(dalloc(p, &p->col_local, (size_t)p->nnz, s));
    k_l2g<<<grid, 256, 0, s>>>(p->NL, p->nb, p->n_own, p->lo, ghost, p->l2g);
    k_relabel<<<grid, 256, 0, s>>>(p->nnz, A->col, p->lo, p->hi, p->nb, p->n_own, bits, wpre, p->col_local);
    // send plan
    {
        const int64_t tot = (int64_t)G * p->n_own;
        int32_t *flags = nullptr, *pos = nullptr;
        TRY(set_cuda_rc(cudaMallocAsync(&flags, sizeof(int32_t) * (tot + 1), s), "alloc"));
        TRY(set_cuda_rc(cudaMallocAsync(&pos, sizeof(int32_t) * (tot + 1), s), "alloc"));
        TRY(set_cuda_rc(cudaMemsetAsync(flags, 0, sizeof(int32_t) * (tot + 1), s), "memset"));
        k_mark_send<<<grid, 256, 0, s>>>(p->n_own, A->rowptr, A->col, dbounds, G, rank, flags);
        size_t tb = 0;
        cub::DeviceScan::ExclusiveSum(nullptr, tb, flags, pos, (int)(tot + 1), s);
        void* tmp = nullptr;
        TRY(set_cuda_rc(cudaMallocAsync(&tmp, tb + 16, s), "alloc"));
        TRY(set_cuda_rc(cub::DeviceScan::ExclusiveSum(tmp, tb, flags, pos, (int)(tot + 1), s), "scan"));
        cudaFreeAsync(tmp, s);
        std::vector<int32_t> qpos(G + 1);
        for (int q = 0; q <= G; q++)
            TRY(set_cuda_rc(cudaMemcpyAsync(&qpos[q], pos + (int64_t)q * p->n_own, sizeof(int32_t),
                                            cudaMemcpyDeviceToHost, s), "copy"));
        TRY(set_cuda_rc(cudaStreamSynchronize(s), "sync"));
        p->send_total = qpos[G];
        p->send_off.assign(G, 0);
        p->send_cnt.assign(G, 0);
        for (int q = 0; q < G; q++) {
            p->send_off[q] = qpos[q];
            p->send_cnt[q] = qpos[q + 1] - qpos[q];
        }
        TRY(dalloc(p, &p->send_idx, (size_t)p->send_total, s));
        TRY(dalloc(p, &p->send_peer, (size_t)p->send_total, s));
        k_compact_send<<<grid, 256, 0, s>>>(tot, p->n_own, p->nb, flags, pos, p->send_idx, p->send_peer);
        cudaFreeAsync(flags, s);
        cudaFreeAsync(pos, s);
    }
    TRY(dalloc(p, &p->sbuf, (size_t)p->send_total * sizeof(int32_t) * n, s));
    TRY(dalloc(p, &p->dpeer, (size_t)3 * G, s));
    // factor buffers over the local id space
    TRY(dalloc(p, &p->pi, (size_t)p->NL * n, s));
    TRY(dalloc(p, &p->pi_w, (size_t)p->NL * n, s));
    TRY(dalloc(p, &p->pi_val, (size_t)p->NL * n, s));
    TRY(dalloc(p, &p->diag, (size_t)p->NL, s));
    TRY(dalloc(p, &p->rounds, 1, s));
    TRY(dalloc(p, &p->live, (size_t)2 * kMaxFlagRounds, s));
    p->ws_bytes = lf_factor_workspace_size(p->NL, n);
    {
        char* w = nullptr;
        TRY(dalloc(p, &w, p->ws_bytes, s));
        p->ws = w;
        Carve c(p->ws, p->ws_bytes);
        factor_ws_carve(c, p->NL, n, &p->fws);
    }
    cudaFreeAsync(bits, s);
    cudaFreeAsync(pc, s);
    cudaFreeAsync(wpre, s);
    cudaFreeAsync(dbounds, s);
    cudaFreeAsync(gb, s);
    TRY(set_cuda_rc(cudaGetLastError(), "setup kernels"));
#undef TRY
    *out = p;
    return LF_OK;
}

int lf_part_destroy(void* part, void* stream) {
    Part* p = (Part*)part;
    if (!p) return LF_OK;
    for (void* a : p->allocs) cudaFreeAsync(a, (cudaStream_t)stream);
    delete p;
    return LF_OK;
}

int lf_part_info(void* part, int64_t* info, int cap) {
    Part* p = (Part*)part;
    if (!p || !info) return set_error(LF_EINVAL, "lf_part_info: NULL");
    const int64_t v[8] = {p->lo, p->hi, p->nb, p->na, p->NL, p->send_total, p->nnz, p->G};
    for (int i = 0; i < cap && i < 8; i++) info[i] = v[i];
    return LF_OK;
}

int lf_part_factor(void** parts, int nparts, void* comm, const lf_factor_opts_t* opts, void* stream) {
    g_err_clear();
    Comm* c = (Comm*)comm;
    if (!parts || nparts < 1 || !c) return set_error(LF_EINVAL, "lf_part_factor: bad arguments");
    lf_factor_opts_t o;
    if (opts) o = *opts; else lf_factor_opts_default(&o);
    if (o.until_maximal || o.M < 0 || o.M > kMaxFlagRounds || o.m < 1)
        return set_error(LF_EINVAL, "lf_part_factor: needs 0 <= M <= 1024, no until_maximal");
    cudaStream_t s = (cudaStream_t)stream;
    if (c->kind == 0) {
        if (nparts != 1) return set_error(LF_EINVAL, "lf_part_factor: NCCL runs one partition per process");
        Part* p = (Part*)parts[0];
        if (p->G != c->nranks || p->rank != c->rank) return set_error(LF_EINVAL, "lf_part_factor: comm/partition mismatch");
        p->comm = c;
        return run_factor(p, &o, s);
    }
    // loopback: all G partitions in this process, lockstep threads on one stream
    if (nparts != ((Part*)parts[0])->G) return set_error(LF_EINVAL, "lf_part_factor: loopback needs all partitions");
    c->parts.assign(nparts, nullptr);
    for (int i = 0; i < nparts; i++) {
        Part* p = (Part*)parts[i];
        c->parts[p->rank] = p;
        p->comm = c;
    }
    c->bar.n = nparts;
    c->bar.aborted = false;
    int dev = 0;
    cudaGetDevice(&dev);
    std::vector<int> rcs(nparts, 0);
    std::vector<std::string> errs(nparts);
    std::vector<std::thread> th;
    for (int i = 0; i < nparts; i++) {
        th.emplace_back([&, i] {
            cudaSetDevice(dev);
            int rc = run_factor(c->parts[i], &o, s);
            if (rc) {
                errs[i] = lf_last_error();
                c->bar.abort();
            }
            rcs[i] = rc;
        });
    }
    for (auto& t : th) t.join();
    for (int i = 0; i < nparts; i++)
        if (rcs[i]) return set_error(rcs[i], errs[i].c_str());
    return LF_OK;
}

int lf_part_export(void* part, int32_t* pi, float* pi_w, float* pi_val, float* diag, int32_t* rounds,
                   int64_t* live, void* stream) {
    Part* p = (Part*)part;
    if (!p) return set_error(LF_EINVAL, "lf_part_export: NULL");
    cudaStream_t s = (cudaStream_t)stream;
    if (p->n_own > 0) {
        k_export<<<persistent_grid((const void*)k_export, 256), 256, 0, s>>>(p->n_own, p->n, p->nb, p->pi, p->pi_w,
                                                                           p->pi_val, p->diag, p->l2g, pi, pi_w,
                                                                           pi_val, diag);
        LF_CUDA(cudaGetLastError());
    }
    if (rounds) LF_CUDA(cudaMemcpyAsync(rounds, p->rounds, sizeof(int32_t), cudaMemcpyDeviceToDevice, s));
    if (live) LF_CUDA(cudaMemcpyAsync(live, p->live, sizeof(int64_t) * 2 * p->M, cudaMemcpyDeviceToDevice, s));
    return LF_OK;
}


int lf_part_linear_forest(void** parts, int nparts, void* comm, void* stream) {
    g_err_clear();
    Comm* c = (Comm*)comm;
    if (!parts || nparts < 1 || !c) return set_error(LF_EINVAL, "lf_part_linear_forest: bad arguments");
    if (c->kind == 1 && nparts != ((Part*)parts[0])->G)
        return set_error(LF_EINVAL, "lf_part_linear_forest: loopback needs all partitions");
    cudaStream_t s = (cudaStream_t)stream;
    return for_parts(parts, nparts, c, [&](Part* p) { return run_forest(p, s); });
}

int lf_part_tridiag(void** parts, int nparts, void* comm, float* const* a, float* const* b, float* const* cc,
                    void* stream) {
    g_err_clear();
    Comm* c = (Comm*)comm;
    if (!parts || nparts < 1 || !c || !a || !b || !cc) return set_error(LF_EINVAL, "lf_part_tridiag: bad arguments");
    cudaStream_t s = (cudaStream_t)stream;
    // outputs are given per partition in the order of `parts`
    std::vector<Part*> order(nparts);
    for (int i = 0; i < nparts; i++) order[i] = (Part*)parts[i];
    return for_parts(parts, nparts, c, [&](Part* p) {
        int i = 0;
        while (order[i] != p) i++;
        return run_tridiag(p, a[i], b[i], cc[i], s);
    });
}

int lf_part_forest_export(void* part, int32_t* forest, int32_t* path_id, int32_t* pos, int32_t* iperm,
                          int64_t* n_cycles, void* stream) {
    Part* p = (Part*)part;
    if (!p || !p->lf_ready) return set_error(LF_EINVAL, "lf_part_forest_export: no linear forest yet");
    cudaStream_t s = (cudaStream_t)stream;
    const size_t n = (size_t)p->n_own;
    if (forest) LF_CUDA(cudaMemcpyAsync(forest, p->forest, sizeof(int32_t) * 2 * n, cudaMemcpyDeviceToDevice, s));
    if (path_id) LF_CUDA(cudaMemcpyAsync(path_id, p->path_id, sizeof(int32_t) * n, cudaMemcpyDeviceToDevice, s));
    if (pos) LF_CUDA(cudaMemcpyAsync(pos, p->pos, sizeof(int32_t) * n, cudaMemcpyDeviceToDevice, s));
    if (iperm) LF_CUDA(cudaMemcpyAsync(iperm, p->iperm, sizeof(int32_t) * n, cudaMemcpyDeviceToDevice, s));
    if (n_cycles) LF_CUDA(cudaMemcpyAsync(n_cycles, p->n_cycles, sizeof(int64_t), cudaMemcpyDeviceToDevice, s));
    return LF_OK;
}

}  // extern "C"
