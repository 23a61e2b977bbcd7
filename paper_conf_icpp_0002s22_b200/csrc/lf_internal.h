// lf_internal.h -- host-side internals shared by the translation units of liblf.so.
#pragma once

#include <cuda_runtime.h>

#include <cstddef>
#include <cstdint>

#include "../../include/lf.h"

namespace lf {

constexpr int kMaxFlagRounds = 1024;  // maximality flags kept on the device (ring)

// error state (thread-local message, lf_api.cu)
int set_error(int code, const char* msg);
int set_cuda_error(cudaError_t e, const char* where);
inline int set_cuda_rc(cudaError_t e, const char* where) { return e == cudaSuccess ? LF_OK : set_cuda_error(e, where); }
void g_err_clear();

#define LF_CUDA(call)                                                     \
    do {                                                                  \
        cudaError_t e_ = (call);                                          \
        if (e_ != cudaSuccess) return ::lf::set_cuda_error(e_, #call);    \
    } while (0)

// optional per-kernel event timing (lf_profile_enable / lf_profile_collect)
int prof_begin(const char* name, int k, cudaStream_t s);
void prof_end(cudaStream_t s, int idx);
struct ProfScope {
    cudaStream_t s;
    int idx;
    ProfScope(const char* name, int k, cudaStream_t st) : s(st), idx(prof_begin(name, k, st)) {}
    ~ProfScope() { prof_end(s, idx); }
};
#define LF_PROF(name, k, s) ::lf::ProfScope lf_prof_scope_(name, k, s)

// Programmatic dependent launch (PDL): a kernel launched this way may be scheduled while
// its stream predecessor (a kernel) is still finishing; it calls pdl_wait() before it
// touches anything the predecessor writes.  Disabled by the environment variable
// LF_NO_PDL (then an ordinary launch).
bool pdl_enabled();
template <typename... KArgs, typename... Args>
inline cudaError_t launch_pdl(void (*kernel)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t s,
                              Args&&... args) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.dynamicSmemBytes = smem;
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = pdl_enabled() ? 1 : 0;
    return cudaLaunchKernelEx(&cfg, kernel, static_cast<Args&&>(args)...);
}

// grid of a persistent kernel: resident blocks per SM x SM count (cached per kernel)
int persistent_grid(const void* kernel, int block, size_t smem = 0);
int sm_count();

// 256-byte aligned bump allocator over a caller workspace
struct Carve {
    char* base;
    size_t cap;
    size_t off = 0;
    Carve(void* b, size_t c) : base((char*)b), cap(c) {}
    template <class T>
    T* take(size_t n) {
        off = (off + 255) & ~(size_t)255;
        T* p = (T*)(base ? base + off : nullptr);
        off += n * sizeof(T);
        return p;
    }
    bool ok() const { return off <= cap; }
};

struct FactorWs {
    uint8_t* state;     // [N]
    int32_t* prop_j;    // [N*n]
    float* prop_v;      // [N*n]
    int32_t* wl[2];     // [N] each
    int32_t* counts;    // [4]
    int* flags;         // [kMaxFlagRounds]
    int32_t* long_rows; // [N] rows deferred to the warp-per-row pass of a round
    int32_t* long_count;// [kMaxFlagRounds]
    unsigned long long* live_part;  // [kMaxFlagRounds][2][64] live-row counter slots
};
size_t factor_ws_carve(Carve& c, int64_t N, int n, FactorWs* w);

// partitioned run of the factor (one contiguous row range of a larger graph, ghost
// vertices filled by a halo exchange between rounds); nullptr = a whole graph
struct PartCtx {
    int64_t row_base;   // local id of the first own row (number of ghosts below the range)
    int64_t gid_off;    // global id of own local vertex v is v + gid_off
    int64_t NL;         // local vertices (ghosts below + own + ghosts above)
    const int32_t* l2g; // [NL] global id of each local vertex
    void* ctx;
    int (*pre_propose)(void* ctx, int k, cudaStream_t s);  // ghost state (degree, charge)
    int (*pre_mutual)(void* ctx, int k, cudaStream_t s);   // ghost proposals
    int (*pre_finalize)(void* ctx, cudaStream_t s);        // global flags / counters
};

int factor_dispatch(const lf_csr_t* A, int n, const lf_factor_opts_t* o, int32_t* pi, float* pi_w,
                    float* pi_val, float* diag, int32_t* rounds_dev, int64_t* live,
                    const FactorWs& w, cudaStream_t s, const PartCtx* part = nullptr);

struct ForestWs {
    int2* rq1[2];          // reduced graph, cycle pass: stride pointers (ping-pong)
    ulonglong2* rk1[2];    //   min edge keys
    int2* rq2[2];          // reduced graph, rank pass: stride pointers
    int2* rr2[2];          //   distances
    short2* loc1;          // [N] local results of the cycle pass
    uint64_t* kst;         // [N] weakest key of a local cycle
    int2* loc2;            // [N] local results of the rank pass
    uint64_t* cyc_k;       // [list1 pos] weakest edge key of the global cycle through a boundary vertex
    int2* end2;            // [list pos] path ends per direction of a boundary vertex
    int2* dist2;           // [list2 pos] distances to them
    int32_t* bidx1;        // [N] list1 position of a boundary vertex
    int32_t* bidx2;        // [N] list2 position of a boundary vertex
    int32_t* list1;        // boundary vertices, cycle pass
    int32_t* list2;        // boundary vertices, rank pass
    int32_t* len;          // [N] path length at the path-ID vertex, else 0
    int32_t* off;          // [N] exclusive scan of len
    int* ctl;              // [256] per-step counters, list sizes
    void* scan_tmp;        // CUB temp storage
    size_t scan_tmp_bytes;
    ulonglong2* kraw;      // [list1 pos] per-direction min keys after the cycle pass
    ulonglong2* ekb;       // [list1 pos] slot keys of boundary vertices
    uint8_t* pdir;         // [N] forest slot toward the path-ID end (predecessor slot)
    int32_t* tsum;         // [chunks + 2] path-length sums per offset chunk -> exclusive prefix
    int2* cq;              // [list position] reduced-graph records of the boundary list being
    ulonglong2* cq_k;      //   scanned: stride pointers (vertex ids), keys or distances
    int2* cq_r;            // [list position] single-pass forest: initial window lengths,
    int2* cq_dk;           //   initial DK (2 * distance to the minimum's near endpoint + bit),
    int2* dk2;             //   final DK per direction
    int2* rdk[2];          //   grid-path ping-pong DK
    // global ruling set (lf_forest.cu k_grs_*): packed per-vertex records, visit bitmap,
    // records of splitter-free cycles
    int4* grs_rec;         // [N] 16-byte per-vertex records (lf_forest.cu grs_load)
    int4* grs_meet;        // [2N] meet records per (vertex, slot)
    uint64_t* grs_meetk;
    int4* grs_mstop;       // [2N] per walk
    uint32_t* grs_bits;    // [N/32 + 1] splitter or visited by a walk
    int4* grs_cyc;         // [N/3 + 1] (lowest vertex, DK, L, 0) of a cycle without splitters
    uint64_t* grs_cyck;    // [N/3 + 1] its weakest key
    int4* grs_desc;        // [2N] walk descriptors (32 bytes per splitter / splitter-free cycle)
};
size_t forest_ws_carve(Carve& c, int64_t N, ForestWs* w, bool with_grs = true);

// Partitioned linear forest: this rank's rows [lo, hi) of the factor;
// paths and cycles that cross ranks are resolved through an exchanged list of "exit"
// records (boundary vertices with a cross-rank forest link).  Buffers sized by the
// global N are indexed by global vertex id; `exit_cap` bounds any rank's exit records.
struct ForestPartCtx {
    int64_t lo, hi;
    int G, rank;
    const int32_t* ghost_list;   // sorted global ids of ghost vertices
    int64_t n_ghost, ghost_below;
    const int2* ghost_nb;        // [local id] factor slots (global ids) of ghosts
    int64_t exit_cap;
    // global buffers
    int2* gq[2];
    ulonglong2* gk[2];
    int2* gr[2];
    uint64_t* gcyc;              // [glist pos] exit-graph results (compact)
    int2* gend;
    int2* gdist;
    int32_t* gbidx;              // [N] glist position of an exit vertex
    int32_t* glist;              // [G * exit_cap]
    int2* gcq;                   // [G * exit_cap] exit-graph records at glist positions
    ulonglong2* gcq_k;
    int* gctl;                   // [256]
    void* rec_send;              // [exit_cap] records
    void* rec_all;               // [G * exit_cap] records
    int2* pub_send;              // [exit_cap] (path id, global offset)
    int2* pub_all;               // [G * exit_cap]
    int32_t* offG;               // [N] global offsets of cross-rank path ids
    int64_t* tot;                // [G + 2] per-rank path-length totals, base, cycles
    void* ctx;
    int (*allgather)(void* ctx, const void* send, void* recv, size_t bytes_per_rank, cudaStream_t s);
    int (*allreduce_i64)(void* ctx, int64_t* buf, int count, cudaStream_t s);
};
size_t exit_record_bytes();

int forest_part_run(int64_t N, const int32_t* pi2, const float* pi2_w, int32_t* forest, int32_t* path_id,
                    int32_t* pos, int32_t* iperm, int64_t* n_cycles, const ForestWs& w,
                    const ForestPartCtx& pc, cudaStream_t s);

// optional fused tridiagonal copy at the end of forest_run (all NULL: none)
struct TriOut {
    const float* pi2_val;
    const float* diag;
    float *a, *b, *c;
};
int forest_run(int64_t N, const int32_t* pi2, const float* pi2_w, int32_t* forest, int32_t* path_id,
               int32_t* pos, int32_t* perm, int32_t* iperm, int64_t* n_cycles, const ForestWs& w,
               cudaStream_t s, const TriOut* tri = nullptr);

int forest_stats(const ForestWs& w, int32_t* out, int cap);

int tridiag_run(int64_t N, const int32_t* forest, const int32_t* iperm, const int32_t* pi2,
                const float* pi2_val, const float* diag, float* a, float* b, float* c,
                cudaStream_t s);

size_t trisolve_ws_bytes(int64_t N);
int trisolve_run(int64_t N, const float* a, const float* b, const float* c, const float* x,
                 float* y, void* ws, cudaStream_t s);

// diagnostic timeline (LF_TIMELINE builds): [2 i] first start, [2 i + 1] last exit (ns)
int timeline_factor(unsigned long long* out, int reset);
int timeline_forest(unsigned long long* out, int reset);
}  // namespace lf
