"""Independent pure-Python checkers used to pin the oracle (small inputs only).

Nothing here calls the oracle or the CUDA path.  Each function is a *different*
route to a result the paper fixes, so that agreement with the oracle is evidence:
  - bidirectional_scan_alg3: the paper's Algorithm 3, literally,
    with ceil(log2 N) steps (reading c10), versus the oracle's sequential walks;
  - brute_force_factor: exhaustive maximum-weight [0,n]-factor (tiny graphs);
  - md5_finish: MD5 rounds 2-4 of RFC 1321, so that round 1 (the charge) can be
    checked against hashlib.
"""
from __future__ import annotations

import itertools
import math

import numpy as np


def edges_of(A):
    """Undirected off-diagonal edges (u<v, |w|) of a CSR matrix."""
    out = []
    for v in range(A.N):
        for e in range(A.rowptr[v], A.rowptr[v + 1]):
            j = int(A.col[e])
            if j > v and A.val[e] != 0:
                out.append((v, j, abs(float(A.val[e]))))
    return out


def brute_force_factor(N, edges, n):
    """Maximum total |w| over all edge subsets with every degree <= n."""
    best = 0.0
    best_set = ()
    E = len(edges)
    assert E <= 20
    for mask in range(1 << E):
        deg = [0] * N
        ok = True
        wsum = 0.0
        for i in range(E):
            if mask >> i & 1:
                u, v, w = edges[i]
                deg[u] += 1
                deg[v] += 1
                if deg[u] > n or deg[v] > n:
                    ok = False
                    break
                wsum += w
        if ok and wsum > best:
            best, best_set = wsum, tuple(i for i in range(E) if mask >> i & 1)
    return best, best_set


def bidirectional_scan_alg3(forest):
    """Algorithm 3 on an acyclic [0,2]-factor.

    forest: int array [N,2] of neighbours (-1 = none).  Returns (l, p) with the path
    ID defined as the *minimum* end ID (text L223, reading c11) and 1-based positions.
    """
    N = forest.shape[0]
    # L1-L4: r(v) <- (1,1); q(v) <- make_tuple(pi(v)): neighbours, padded with the
    # path-end marker -(v+1) (L245)
    q = np.empty((N, 2), dtype=np.int64)
    r = np.ones((N, 2), dtype=np.int64)
    for v in range(N):
        for i in range(2):
            q[v, i] = forest[v, i] if forest[v, i] >= 0 else -(v + 1)
    steps = max(1, math.ceil(math.log2(N))) if N > 1 else 1
    for _ in range(steps):  # launched ceil(log2 N) times instead of testing L5 (L243)
        qp, rp = q.copy(), r.copy()  # L6-L7 (ping-pong, L249)
        for v in range(N):
            w = [qp[v, 0], qp[v, 1]]
            rr = [rp[v, 0], rp[v, 1]]
            for i in range(2):
                if w[i] >= 0:  # not is_path_end(w_i)
                    wi = w[i]
                    vv = qp[wi]
                    tt = rp[wi]
                    for j in range(2):
                        if vv[j] != v:  # L16
                            rr[i] = rr[i] + tt[j]  # L17
                            w[i] = vv[j]  # L18
            q[v] = w
            r[v] = rr
    l = np.empty(N, dtype=np.int64)
    p = np.empty(N, dtype=np.int64)
    for v in range(N):
        assert q[v, 0] < 0 and q[v, 1] < 0, "cycle left in forest"
        ends = [-(q[v, 0] + 1), -(q[v, 1] + 1)]
        i = 0 if ends[0] < ends[1] else 1  # min end ID (L223)
        if ends[0] == ends[1]:
            i = 0 if r[v, 0] <= r[v, 1] else 1  # singleton: both markers equal
        l[v] = ends[i]
        p[v] = r[v, i]
    return l, p


def bidirectional_min_scan_cycles(pi2, pi2_w):
    """Step (1) with the bidirectional min-scan.

    Returns the set of removed edges (min,max): for every vertex still holding two
    positive stride pointers after ceil(log2 N) steps (a cycle, L245), the weakest
    edge key seen in both directions.  Key = (|w|, -min, -max) minimised (reading c9).
    """
    N = pi2.shape[0]
    q = np.empty((N, 2), dtype=np.int64)
    mk = [[None, None] for _ in range(N)]
    for v in range(N):
        for i in range(2):
            w = int(pi2[v, i])
            q[v, i] = w if w >= 0 else -(v + 1)
            if w >= 0:
                a, b = min(v, w), max(v, w)
                mk[v][i] = (float(pi2_w[v, i]), -a, -b)
            else:
                mk[v][i] = (math.inf, 0, 0)
    steps = max(1, math.ceil(math.log2(N))) if N > 1 else 1
    for _ in range(steps):
        qp = q.copy()
        mp = [list(x) for x in mk]
        for v in range(N):
            for i in range(2):
                wi = qp[v, i]
                if wi >= 0:
                    for j in range(2):
                        if qp[wi, j] != v:
                            mk[v][i] = min(mp[v][i], mp[wi][j])
                            q[v, i] = qp[wi, j]
    removed = set()
    for v in range(N):
        if q[v, 0] >= 0 and q[v, 1] >= 0:
            k = min(mk[v][0], mk[v][1])
            removed.add((-k[1], -k[2]))
    return removed


# --- MD5 rounds 2..4 (RFC 1321) to finish a round-1 state -------------------

_K = [int(abs(math.sin(i + 1)) * 2 ** 32) & 0xFFFFFFFF for i in range(64)]
_S = [7, 12, 17, 22] * 4 + [5, 9, 14, 20] * 4 + [4, 11, 16, 23] * 4 + [6, 10, 15, 21] * 4
_IV = (0x67452301, 0xEFCDAB89, 0x98BADCFE, 0x10325476)


def _rotl(x, s):
    x &= 0xFFFFFFFF
    return ((x << s) | (x >> (32 - s))) & 0xFFFFFFFF


def md5_finish(state_after_round1, X):
    """Run MD5 steps 17..64 on (a,b,c,d) and return the 16-byte digest."""
    a, b, c, d = (int(x) for x in state_after_round1)
    for i in range(16, 64):
        if i < 32:
            F = (b & d) | (c & ~d & 0xFFFFFFFF)
            g = (5 * i + 1) % 16
        elif i < 48:
            F = b ^ c ^ d
            g = (3 * i + 5) % 16
        else:
            F = c ^ (b | (~d & 0xFFFFFFFF))
            g = (7 * i) % 16
        a, d, c, b = d, c, b, (b + _rotl(a + F + _K[i] + X[g], _S[i])) & 0xFFFFFFFF
    out = [(x + y) & 0xFFFFFFFF for x, y in zip(_IV, (a, b, c, d))]
    return b"".join(int(x).to_bytes(4, "little") for x in out)


def random_02_factor(N, rng, n_cycles=3, ties=False):
    """A random [0,2]-factor made of disjoint cycles and paths (N x 2 slots, weights)."""
    perm = rng.permutation(N)
    pi = -np.ones((N, 2), dtype=np.int32)
    pw = np.zeros((N, 2), dtype=np.float32)
    # cut the permutation into pieces; the first n_cycles pieces of length>=3 are cycles
    cuts = sorted(set(rng.integers(1, N, size=max(1, N // 4)).tolist())) if N > 1 else []
    pieces = [perm[a:b] for a, b in zip([0] + cuts, cuts + [N]) if b > a]
    made = 0
    for pc in pieces:
        L = len(pc)
        links = [(pc[i], pc[i + 1]) for i in range(L - 1)]
        if L >= 3 and made < n_cycles:
            links.append((pc[-1], pc[0]))
            made += 1
        for u, v in links:
            w = np.float32(rng.integers(1, 4) / 4.0) if ties else np.float32(rng.random() + 1e-3)
            for x, y in ((u, v), (v, u)):
                s = 0 if pi[x, 0] < 0 else 1
                pi[x, s] = y
                pw[x, s] = w
    # canonical slot order: |w| desc, lower index first (c8)
    for v in range(N):
        sl = [(pw[v, i], pi[v, i]) for i in range(2) if pi[v, i] >= 0]
        sl.sort(key=lambda t: (-t[0], t[1]))
        for i in range(2):
            pi[v, i], pw[v, i] = (sl[i][1], sl[i][0]) if i < len(sl) else (-1, 0.0)
    return pi, pw


def all_subsets(iterable):
    s = list(iterable)
    return itertools.chain.from_iterable(itertools.combinations(s, r) for r in range(len(s) + 1))
