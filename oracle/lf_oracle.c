/*
 * lf_oracle.c -- plain, slow, single-threaded CPU oracle for the hot path of
 * Klein & Strzodka, "Highly Parallel Linear Forest Extraction from a Weighted Graph
 * on GPUs", ICPP'22.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  It shares no code,
 * header, table or helper with the CUDA path (paper_conf_icpp_0002s22_b200/csrc).
 *
 * Every function follows the paper's algorithm step by step, in its order and
 * notation, with the readings of SURVEY.md §8(c) (listed in DESIGN.md §3) where the
 * paper is silent or garbled.  No blocking, fusion, worklists or reordering.
 *
 * Conventions:
 *   A is CSR: int64 rowptr[N+1], int32 col[Z], float val[Z]; symmetric.
 *   edge weight |w({v,j})| = |a_vj| for j != v, a_vj != 0      (A' = |A|-diag)
 *   pi[v*n + s], s < n: the confirmed neighbours of v, sorted by key descending
 *   (|w| desc, then lower vertex index first: reading c1/c8), -1 padding last.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>

#define LFO_OK 0
#define LFO_EINVAL -1
#define LFO_ENOMEM -2

/* ------------------------------------------------------------------------- */
/* charge(v, k): "a part of the MD5 algorithm" (Alg. 2 L8-L12).  */
/* Reading c2: MD5 round 1 (RFC 1321 steps 1..16, function F) over the 12-byte  */
/* message (v, k, seed) with standard MD5 padding; h = a + 0x67452301;           */
/* charge is '+' iff h < p * 2^32.                                               */
/* ------------------------------------------------------------------------- */
static uint32_t rotl32(uint32_t x, int s) { return (x << s) | (x >> (32 - s)); }

void lfo_md5_round1_state(uint32_t v, uint32_t k, uint32_t seed, uint32_t out[4])
{
    /* RFC 1321 sine table T[1..16] and round-1 shifts. */
    static const uint32_t T[16] = {
        0xd76aa478u, 0xe8c7b756u, 0x242070dbu, 0xc1bdceeeu,
        0xf57c0fafu, 0x4787c62au, 0xa8304613u, 0xfd469501u,
        0x698098d8u, 0x8b44f7afu, 0xffff5bb1u, 0x895cd7beu,
        0x6b901122u, 0xfd987193u, 0xa679438eu, 0x49b40821u};
    static const int S[4] = {7, 12, 17, 22};
    uint32_t X[16];
    memset(X, 0, sizeof(X));
    X[0] = v;
    X[1] = k;
    X[2] = seed;
    X[3] = 0x80u;       /* padding bit after the 12-byte message */
    X[14] = 96u;        /* message length in bits */
    uint32_t a = 0x67452301u, b = 0xefcdab89u, c = 0x98badcfeu, d = 0x10325476u;
    for (int i = 0; i < 16; i++) {
        uint32_t F = (b & c) | (~b & d);
        uint32_t tmp = d;
        d = c;
        c = b;
        b = b + rotl32(a + F + T[i] + X[i], S[i % 4]);
        a = tmp;
    }
    out[0] = a; out[1] = b; out[2] = c; out[3] = d;
}

uint32_t lfo_charge_hash(uint32_t v, uint32_t k, uint32_t seed)
{
    uint32_t st[4];
    lfo_md5_round1_state(v, k, seed, st);
    return st[0] + 0x67452301u;
}

/* returns 1 for '+', 0 for '-' */
int lfo_charge(uint32_t v, uint32_t k, uint32_t seed, float p)
{
    double thr = (double)p * 4294967296.0;
    return (double)lfo_charge_hash(v, k, seed) < thr ? 1 : 0;
}

/* ------------------------------------------------------------------------- */
/* helpers                                                                    */
/* ------------------------------------------------------------------------- */

/* w1 "stronger" than w2 in the proposal order: |w| desc, ties -> lower index (c1). */
static int stronger(float w1, int32_t j1, float w2, int32_t j2)
{
    if (w1 != w2) return w1 > w2;
    return j1 < j2;
}

static int in_set(const int32_t* s, int cnt, int32_t x)
{
    for (int i = 0; i < cnt; i++)
        if (s[i] == x) return 1;
    return 0;
}

static int set_size(const int32_t* s, int n)
{
    int c = 0;
    for (int i = 0; i < n; i++)
        if (s[i] >= 0) c++;
    return c;
}

/* |a_vw| of the edge {v,w} looked up in row v (0 if absent). */
static float edge_weight(const int64_t* rowptr, const int32_t* col, const float* val,
                         int32_t v, int32_t w)
{
    for (int64_t e = rowptr[v]; e < rowptr[v + 1]; e++)
        if (col[e] == w) return fabsf(val[e]);
    return 0.0f;
}

/* sort the (index, weight) slots of one vertex by proposal order, -1 last (c8) */
static void canon_slots(int32_t* s, float* w, int n)
{
    for (int i = 0; i < n; i++)
        for (int j = i + 1; j < n; j++) {
            int swap;
            if (s[i] < 0) swap = s[j] >= 0;
            else if (s[j] < 0) swap = 0;
            else swap = stronger(w[j], s[j], w[i], s[i]);
            if (swap) {
                int32_t ts = s[i]; s[i] = s[j]; s[j] = ts;
                float tw = w[i]; w[i] = w[j]; w[j] = tw;
            }
        }
}

/* ------------------------------------------------------------------------- */
/* Algorithm 2: parallel [0,n]-factor (PAPER.md:L93-L128, L134, L179-L181,     */
/* L199), executed sequentially with explicit copies for every "in parallel"   */
/* loop.                                                                       */
/*                                                                             */
/* charge_override: NULL, or [M*N] bytes (1 '+', 0 '-') used instead of the    */
/* hash (test hook for the Table 1 worked example).                            */
/* live_rows/live_nnz: NULL or [M]: rows with |pi(v)|<n and a non-empty        */
/* charge-free eligible set at round start, and their stored nnz (byte model,  */
/* SURVEY.md §8(d)).                                                           */
/* ------------------------------------------------------------------------- */
int lfo_factor(int64_t N, const int64_t* rowptr, const int32_t* col, const float* val,
               int n, int M, int m, int k_m, float p, uint32_t seed, int until_maximal,
               const uint8_t* charge_override,
               int32_t* pi, float* pi_w, int32_t* rounds_out,
               int64_t* live_rows, int64_t* live_nnz, int max_rounds_recorded)
{
    if (n < 1 || n > 4 || N < 0 || M < 0 || m < 1) return LFO_EINVAL;
    if (until_maximal && (k_m < 0 || k_m >= m)) return LFO_EINVAL;  /* no uncharged round */
    int32_t* pi_prev = (int32_t*)malloc(sizeof(int32_t) * (size_t)(N * n + 1));  /* pi'   */
    int32_t* prop = (int32_t*)malloc(sizeof(int32_t) * (size_t)(N * n + 1));     /* pi after L19-21 */
    float* prop_w = (float*)malloc(sizeof(float) * (size_t)(N * n + 1));
    uint8_t* q = (uint8_t*)malloc((size_t)N + 1);                                 /* charges */
    if (!pi_prev || !prop || !prop_w || !q) {
        free(pi_prev); free(prop); free(prop_w); free(q);
        return LFO_ENOMEM;
    }
    /* L4-L6: pi(v) <- empty */
    for (int64_t i = 0; i < N * n; i++) { pi[i] = -1; pi_w[i] = 0.0f; }
    int rounds = M;
    for (int64_t k = 0; until_maximal || k < M; k++) {
        int charging = (k % m) != k_m;                    /* L16 condition */
        /* L8-L12: charges for this iteration (only used when charging) */
        if (charging)
            for (int64_t v = 0; v < N; v++)
                q[v] = charge_override ? charge_override[k * N + v]
                                       : (uint8_t)lfo_charge((uint32_t)v, (uint32_t)k, seed, p);
        /* L13: pi' <- pi */
        memcpy(pi_prev, pi, sizeof(int32_t) * (size_t)(N * n));
        /* byte-model counters: live rows at round start */
        if (live_rows && k < max_rounds_recorded) {
            int64_t lr = 0, ln = 0;
            for (int64_t v = 0; v < N; v++) {
                if (set_size(&pi_prev[v * n], n) >= n) continue;
                int live = 0;
                for (int64_t e = rowptr[v]; e < rowptr[v + 1]; e++) {
                    int32_t j = col[e];
                    if (j == v || val[e] == 0.0f) continue;
                    if (set_size(&pi_prev[(int64_t)j * n], n) >= n) continue;
                    if (in_set(&pi_prev[v * n], n, j)) continue;
                    live = 1;
                }
                if (live) { lr++; ln += rowptr[v + 1] - rowptr[v]; }
            }
            live_rows[k] = lr;
            live_nnz[k] = ln;
        }
        /* L14-L22: edge proposition, for v in V "in parallel" (reads pi', q; writes prop) */
        int64_t added = 0;
        for (int64_t v = 0; v < N; v++) {
            int32_t* pv = &prop[v * n];
            float* pw = &prop_w[v * n];
            for (int s = 0; s < n; s++) { pv[s] = pi_prev[v * n + s]; pw[s] = pi_w[v * n + s]; }
            int cnt = set_size(pv, n);
            /* L19-L21: while |pi(v)| < n and Theta = W \ pi(v) non-empty: add max_target */
            while (cnt < n) {
                int32_t best = -1;
                float bw = 0.0f;
                for (int64_t e = rowptr[v]; e < rowptr[v + 1]; e++) {
                    int32_t j = col[e];
                    float w = fabsf(val[e]);
                    if (j == v || w == 0.0f) continue;                       /* A' = |A| - diag */
                    if (set_size(&pi_prev[(int64_t)j * n], n) == n) continue; /* L15 */
                    if (charging && q[j] == q[v]) continue;                   /* L17 */
                    if (in_set(pv, cnt, j)) continue;                          /* L19: W \ pi(v) */
                    if (best < 0 || stronger(w, j, bw, best)) { best = j; bw = w; }
                }
                if (best < 0) break;
                pv[cnt] = best;   /* L20 */
                pw[cnt] = bw;
                cnt++;
                added++;
            }
        }
        /* L23-L25: maximal? (nothing was added in a round without charging) */
        if (added == 0 && (k % m) == k_m) {
            rounds = (int)(k + 1);
            break;
        }
        /* L26-L28: pi(v) <- { w in pi(v) | v in pi(w) }, reading the proposals */
        for (int64_t v = 0; v < N; v++) {
            int32_t keep[4];
            float keep_w[4];
            int c = 0;
            for (int s = 0; s < n; s++) {
                int32_t w = prop[v * n + s];
                if (w < 0) continue;
                if (in_set(&prop[(int64_t)w * n], n, (int32_t)v)) { keep[c] = w; keep_w[c] = prop_w[v * n + s]; c++; }
            }
            for (int s = 0; s < n; s++) {
                pi[v * n + s] = s < c ? keep[s] : -1;
                pi_w[v * n + s] = s < c ? keep_w[s] : 0.0f;
            }
            canon_slots(&pi[v * n], &pi_w[v * n], n);
        }
    }
    if (rounds_out) *rounds_out = rounds;
    free(pi_prev); free(prop); free(prop_w); free(q);
    return LFO_OK;
}

/* ------------------------------------------------------------------------- */
/* Algorithm 1: sequential greedy [0,n]-factor.        */
/* "in order of decreasing |w|"; equal weights in the consistent edge order     */
/* (|w| desc, min(u,v) asc, max(u,v) asc) -- reading c1.                        */
/* ------------------------------------------------------------------------- */
typedef struct { float w; int32_t u, v; } lfo_edge_t;

static int edge_cmp(const void* a, const void* b)
{
    const lfo_edge_t* x = (const lfo_edge_t*)a;
    const lfo_edge_t* y = (const lfo_edge_t*)b;
    if (x->w != y->w) return x->w > y->w ? -1 : 1;
    if (x->u != y->u) return x->u < y->u ? -1 : 1;
    if (x->v != y->v) return x->v < y->v ? -1 : 1;
    return 0;
}

int lfo_greedy(int64_t N, const int64_t* rowptr, const int32_t* col, const float* val,
               int n, int32_t* pi, float* pi_w)
{
    if (n < 1 || n > 4) return LFO_EINVAL;
    int64_t E = 0;
    for (int64_t v = 0; v < N; v++)
        for (int64_t e = rowptr[v]; e < rowptr[v + 1]; e++)
            if (col[e] > v && val[e] != 0.0f) E++;
    lfo_edge_t* ed = (lfo_edge_t*)malloc(sizeof(lfo_edge_t) * (size_t)(E + 1));
    if (!ed) return LFO_ENOMEM;
    E = 0;
    for (int64_t v = 0; v < N; v++)
        for (int64_t e = rowptr[v]; e < rowptr[v + 1]; e++)
            if (col[e] > v && val[e] != 0.0f) { ed[E].w = fabsf(val[e]); ed[E].u = (int32_t)v; ed[E].v = col[e]; E++; }
    qsort(ed, (size_t)E, sizeof(lfo_edge_t), edge_cmp);
    for (int64_t i = 0; i < N * n; i++) { pi[i] = -1; pi_w[i] = 0.0f; }
    for (int64_t i = 0; i < E; i++) {
        int32_t u = ed[i].u, v = ed[i].v;
        int du = set_size(&pi[(int64_t)u * n], n), dv = set_size(&pi[(int64_t)v * n], n);
        if (du < n && dv < n && u != v) {               /* Alg. 1 L5 */
            pi[(int64_t)u * n + du] = v; pi_w[(int64_t)u * n + du] = ed[i].w;   /* L6 */
            pi[(int64_t)v * n + dv] = u; pi_w[(int64_t)v * n + dv] = ed[i].w;   /* L7 */
        }
    }
    for (int64_t v = 0; v < N; v++) canon_slots(&pi[v * n], &pi_w[v * n], n);
    free(ed);
    return LFO_OK;
}

/* ------------------------------------------------------------------------- */
/* Section 3.3: from a [0,2]-factor to a linear forest,   */
/* done here by plain sequential component walks (the paper's sequential CPU   */
/* version, L388/L421), not by the bidirectional scan.                        */
/*   step (1) break every cycle at its weakest edge: minimum |w|, ties ->      */
/*            lexicographically larger (min,max) vertex pair (reading c9)      */
/*   step (2) path ID l(v) = minimum end ID, p(v) = 1-based position counted   */
/*            from that end (L223; readings c11, c12, c16)                      */
/*   step (3) perm = vertex IDs sorted by (l, p); perm[new] = old (c14)         */
/* ------------------------------------------------------------------------- */

/* 1 if edge (w1,a1,b1) is weaker than (w2,a2,b2); a<b are the endpoint IDs */
static int weaker(float w1, int32_t a1, int32_t b1, float w2, int32_t a2, int32_t b2)
{
    if (w1 != w2) return w1 < w2;
    if (a1 != a2) return a1 > a2;
    return b1 > b2;
}

static int32_t other_nb(const int32_t* f, int32_t v, int32_t from)
{
    /* the forest neighbour of v that is not `from` (or -1) */
    int32_t a = f[2 * (int64_t)v], b = f[2 * (int64_t)v + 1];
    if (a >= 0 && a != from) return a;
    if (b >= 0 && b != from) return b;
    return -1;
}

typedef struct { int32_t l, p, v; } lfo_key_t;

static int key_cmp(const void* a, const void* b)
{
    const lfo_key_t* x = (const lfo_key_t*)a;
    const lfo_key_t* y = (const lfo_key_t*)b;
    if (x->l != y->l) return x->l < y->l ? -1 : 1;
    if (x->p != y->p) return x->p < y->p ? -1 : 1;
    return 0;
}

int lfo_linear_forest(int64_t N, const int32_t* pi2, const float* pi2_w,
                      int32_t* forest, int32_t* path_id, int32_t* pos,
                      int32_t* perm, int32_t* iperm, int64_t* n_cycles_out)
{
    /* validate: a symmetric [0,2]-factor */
    for (int64_t v = 0; v < N; v++)
        for (int s = 0; s < 2; s++) {
            int32_t w = pi2[2 * v + s];
            if (w < -1 || w >= N || w == v) return LFO_EINVAL;
            if (w >= 0 && !(pi2[2 * (int64_t)w] == v || pi2[2 * (int64_t)w + 1] == v)) return LFO_EINVAL;
        }
    for (int64_t v = 0; v < N; v++)
        if (pi2[2 * v] >= 0 && pi2[2 * v] == pi2[2 * v + 1]) return LFO_EINVAL;
    memcpy(forest, pi2, sizeof(int32_t) * (size_t)(2 * N));
    uint8_t* seen = (uint8_t*)calloc((size_t)N + 1, 1);
    if (!seen) return LFO_ENOMEM;
    int64_t ncyc = 0;
    /* step (1a): every component that has a vertex with fewer than two neighbours is a
       path; walk it from that end and mark it.  What stays unmarked lies on cycles. */
    for (int64_t s0 = 0; s0 < N; s0++) {
        int deg = (forest[2 * s0] >= 0) + (forest[2 * s0 + 1] >= 0);
        if (deg > 1 || seen[s0]) continue;
        int32_t prev = -1, cur = (int32_t)s0;
        while (cur >= 0) { seen[cur] = 1; int32_t nx = other_nb(forest, cur, prev); prev = cur; cur = nx; }
    }
    /* step (1b): walk each cycle once, find its weakest edge, remove it */
    for (int64_t s0 = 0; s0 < N; s0++) {
        if (seen[s0]) continue;
        ncyc++;
        float bw = pi2_w[2 * s0];
        int32_t first = forest[2 * s0];
        int32_t ba = (int32_t)s0 < first ? (int32_t)s0 : first;
        int32_t bb = (int32_t)s0 < first ? first : (int32_t)s0;
        int32_t prev = (int32_t)s0, cur = first;
        seen[s0] = 1;
        while (cur != (int32_t)s0) {
            seen[cur] = 1;
            int32_t nxt = other_nb(forest, cur, prev);
            /* weight of edge {cur, nxt}, read from cur's slots */
            float w = forest[2 * (int64_t)cur] == nxt ? pi2_w[2 * (int64_t)cur] : pi2_w[2 * (int64_t)cur + 1];
            int32_t a = cur < nxt ? cur : nxt, b = cur < nxt ? nxt : cur;
            if (weaker(w, a, b, bw, ba, bb)) { bw = w; ba = a; bb = b; }
            prev = cur;
            cur = nxt;
        }
        /* remove {ba,bb} from both endpoints; keep slot order, -1 last */
        int32_t ends[2] = {ba, bb};
        for (int e = 0; e < 2; e++) {
            int32_t x = ends[e], y = ends[1 - e];
            int32_t* f = &forest[2 * (int64_t)x];
            if (f[0] == y) { f[0] = f[1]; f[1] = -1; }
            else if (f[1] == y) { f[1] = -1; }
        }
    }
    /* step (2): walk every path from each end */
    for (int64_t v = 0; v < N; v++) { path_id[v] = -1; pos[v] = 0; }
    for (int64_t s0 = 0; s0 < N; s0++) {
        int deg = (forest[2 * s0] >= 0) + (forest[2 * s0 + 1] >= 0);
        if (deg > 1 || path_id[s0] >= 0) continue;
        /* s0 is a path end: find the other end */
        int32_t prev = -1, cur = (int32_t)s0, len = 1;
        while (1) {
            int32_t nxt = other_nb(forest, cur, prev);
            if (nxt < 0) break;
            prev = cur; cur = nxt; len++;
        }
        int32_t e0 = (int32_t)s0, e1 = cur;
        int32_t l = e0 < e1 ? e0 : e1;
        /* positions from end l */
        prev = -1; cur = l;
        for (int32_t i = 1; i <= len; i++) {
            path_id[cur] = l;
            pos[cur] = i;
            int32_t nxt = other_nb(forest, cur, prev);
            prev = cur; cur = nxt;
        }
    }
    for (int64_t v = 0; v < N; v++)
        if (path_id[v] < 0) { free(seen); return LFO_EINVAL; } /* an unbroken cycle: cannot happen */
    /* step (3): sort vertex IDs by (l, p) */
    lfo_key_t* keys = (lfo_key_t*)malloc(sizeof(lfo_key_t) * (size_t)(N + 1));
    if (!keys) { free(seen); return LFO_ENOMEM; }
    for (int64_t v = 0; v < N; v++) { keys[v].l = path_id[v]; keys[v].p = pos[v]; keys[v].v = (int32_t)v; }
    qsort(keys, (size_t)N, sizeof(lfo_key_t), key_cmp);
    for (int64_t r = 0; r < N; r++) { perm[r] = keys[r].v; iperm[keys[r].v] = (int32_t)r; }
    if (n_cycles_out) *n_cycles_out = ncyc;
    free(keys);
    free(seen);
    return LFO_OK;
}

/* ------------------------------------------------------------------------- */
/* Step (4): extract the tridiagonal coefficients of Q^T A Q restricted to the  */
/* diagonal and the linear-forest edges (reading c15):     */
/*   b[r] = a_{v v}, a[r] = a_{v, perm[r-1]}, c[r] = a_{v, perm[r+1]} when that  */
/*   pair is a forest edge, else 0;  v = perm[r].  Values copied from A.         */
/* ------------------------------------------------------------------------- */
static float entry(const int64_t* rowptr, const int32_t* col, const float* val, int32_t v, int32_t w)
{
    for (int64_t e = rowptr[v]; e < rowptr[v + 1]; e++)
        if (col[e] == w) return val[e];
    return 0.0f;
}

int lfo_tridiag(int64_t N, const int64_t* rowptr, const int32_t* col, const float* val,
                const int32_t* forest, const int32_t* perm,
                float* a, float* b, float* c)
{
    for (int64_t r = 0; r < N; r++) {
        int32_t v = perm[r];
        const int32_t* f = &forest[2 * (int64_t)v];
        b[r] = entry(rowptr, col, val, v, v);
        a[r] = 0.0f;
        c[r] = 0.0f;
        if (r > 0) {
            int32_t u = perm[r - 1];
            if (f[0] == u || f[1] == u) a[r] = entry(rowptr, col, val, v, u);
        }
        if (r + 1 < N) {
            int32_t u = perm[r + 1];
            if (f[0] == u || f[1] == u) c[r] = entry(rowptr, col, val, v, u);
        }
    }
    return LFO_OK;
}

/* weight of the factor, Eq. (3), in fp64 (a metric) */
double lfo_factor_weight(int64_t N, const int32_t* pi, int n, const int64_t* rowptr,
                         const int32_t* col, const float* val)
{
    double s = 0.0;
    for (int64_t v = 0; v < N; v++)
        for (int i = 0; i < n; i++) {
            int32_t w = pi[v * n + i];
            if (w > v) s += (double)edge_weight(rowptr, col, val, (int32_t)v, w);
        }
    return s;
}
