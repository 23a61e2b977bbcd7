"""CPU oracle (TEST INFRASTRUCTURE ONLY) -- ctypes binding of oracle/lf_oracle.c.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference
legs may import this package.  The product path (paper_conf_icpp_0002s22_b200) never
imports it, and it never imports the product path.  See lf_oracle.c for the paper
passages each function follows and DESIGN.md §3 for the readings it takes.

Parity status: every function is pinned by tests in tests/test_oracle_*.py against
values the paper prints (Table 1, Tables 4/5 ANISO rows), a library routine (hashlib
MD5 for the charge), a second algorithm from the paper (Alg. 1 vs Alg. 2 with m=1,
M=inf), closed forms, brute force on tiny graphs and invariants; except the charged
rounds' exact bits, whose hash the paper does not specify ("parity unpinned" against
the paper for those bits; pinned statistically and through the MD5 library check).
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "lf_oracle.c")
_LIB = os.path.join(_HERE, "liblf_oracle.so")
_lib = None


def build(force=False):
    """Compile the oracle (plain C, -O2, single thread, no intrinsics)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c99", "-Wall", "-shared", "-fPIC",
                               "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


def lib():
    global _lib
    if _lib is None:
        build()
        L = C.CDLL(_LIB)
        P = C.c_void_p
        L.lfo_md5_round1_state.argtypes = [C.c_uint32, C.c_uint32, C.c_uint32, P]
        L.lfo_charge_hash.argtypes = [C.c_uint32, C.c_uint32, C.c_uint32]
        L.lfo_charge_hash.restype = C.c_uint32
        L.lfo_charge.argtypes = [C.c_uint32, C.c_uint32, C.c_uint32, C.c_float]
        L.lfo_factor.argtypes = [C.c_int64, P, P, P, C.c_int, C.c_int, C.c_int, C.c_int,
                                 C.c_float, C.c_uint32, C.c_int, P, P, P, P, P, P, C.c_int]
        L.lfo_greedy.argtypes = [C.c_int64, P, P, P, C.c_int, P, P]
        L.lfo_linear_forest.argtypes = [C.c_int64, P, P, P, P, P, P, P, P]
        L.lfo_tridiag.argtypes = [C.c_int64, P, P, P, P, P, P, P, P]
        L.lfo_factor_weight.argtypes = [C.c_int64, P, C.c_int, P, P, P]
        L.lfo_factor_weight.restype = C.c_double
        _lib = L
    return _lib


def _p(a):
    return None if a is None else a.ctypes.data_as(C.c_void_p)


def _csr(A):
    rp = np.ascontiguousarray(A.rowptr, dtype=np.int64)
    col = np.ascontiguousarray(A.col, dtype=np.int32)
    val = np.ascontiguousarray(A.val, dtype=np.float32)
    return rp, col, val


def md5_round1_state(v, k, seed=0):
    out = np.zeros(4, dtype=np.uint32)
    lib().lfo_md5_round1_state(v, k, seed, _p(out))
    return out


def charge_hash(v, k, seed=0):
    return int(lib().lfo_charge_hash(v, k, seed))


def charge(v, k, seed=0, p=0.5):
    return int(lib().lfo_charge(v, k, seed, p))


def factor(A, n, M=5, m=5, k_m=0, p=0.5, seed=0, until_maximal=False,
           charge_override=None, counters=False):
    """Algorithm 2 -> (pi[N,n] int32, pi_w[N,n] float32, rounds, live_rows, live_nnz)."""
    rp, col, val = _csr(A)
    N = A.N
    pi = np.empty(N * n, dtype=np.int32)
    pw = np.empty(N * n, dtype=np.float32)
    rounds = np.zeros(1, dtype=np.int32)
    co = None
    if charge_override is not None:
        co = np.ascontiguousarray(charge_override, dtype=np.uint8).reshape(-1)
        assert co.size >= M * N
    R = M if not until_maximal else 0
    lr = np.zeros(max(R, 1), dtype=np.int64) if counters else None
    ln = np.zeros(max(R, 1), dtype=np.int64) if counters else None
    rc = lib().lfo_factor(N, _p(rp), _p(col), _p(val), n, M, m, k_m, p, seed,
                          int(bool(until_maximal)), _p(co), _p(pi), _p(pw), _p(rounds),
                          _p(lr), _p(ln), R if counters else 0)
    if rc != 0:
        raise ValueError(f"lfo_factor failed ({rc})")
    return pi.reshape(N, n), pw.reshape(N, n), int(rounds[0]), lr, ln


def greedy(A, n):
    """Algorithm 1 -> (pi[N,n], pi_w[N,n])."""
    rp, col, val = _csr(A)
    N = A.N
    pi = np.empty(N * n, dtype=np.int32)
    pw = np.empty(N * n, dtype=np.float32)
    rc = lib().lfo_greedy(N, _p(rp), _p(col), _p(val), n, _p(pi), _p(pw))
    if rc != 0:
        raise ValueError(f"lfo_greedy failed ({rc})")
    return pi.reshape(N, n), pw.reshape(N, n)


def linear_forest(pi2, pi2_w):
    """Section 3.3 steps (1)-(3) -> dict(forest, path_id, pos, perm, iperm, n_cycles)."""
    pi2 = np.ascontiguousarray(pi2, dtype=np.int32).reshape(-1)
    pw = np.ascontiguousarray(pi2_w, dtype=np.float32).reshape(-1)
    N = pi2.size // 2
    forest = np.empty(2 * N, dtype=np.int32)
    pid = np.empty(N, dtype=np.int32)
    pos = np.empty(N, dtype=np.int32)
    perm = np.empty(N, dtype=np.int32)
    iperm = np.empty(N, dtype=np.int32)
    ncyc = np.zeros(1, dtype=np.int64)
    rc = lib().lfo_linear_forest(N, _p(pi2), _p(pw), _p(forest), _p(pid), _p(pos),
                                 _p(perm), _p(iperm), _p(ncyc))
    if rc != 0:
        raise ValueError(f"lfo_linear_forest failed ({rc})")
    return dict(forest=forest.reshape(N, 2), path_id=pid, pos=pos, perm=perm, iperm=iperm,
                n_cycles=int(ncyc[0]))


def tridiag(A, forest, perm):
    """Step (4) -> (a, b, c) float32 [N]."""
    rp, col, val = _csr(A)
    N = A.N
    f = np.ascontiguousarray(forest, dtype=np.int32).reshape(-1)
    pm = np.ascontiguousarray(perm, dtype=np.int32)
    a = np.empty(N, dtype=np.float32)
    b = np.empty(N, dtype=np.float32)
    c = np.empty(N, dtype=np.float32)
    lib().lfo_tridiag(N, _p(rp), _p(col), _p(val), _p(f), _p(pm), _p(a), _p(b), _p(c))
    return a, b, c


def factor_weight(A, pi):
    """omega_pi, Eq. (3), fp64."""
    rp, col, val = _csr(A)
    pi = np.ascontiguousarray(pi, dtype=np.int32)
    n = pi.shape[1] if pi.ndim == 2 else 1
    return float(lib().lfo_factor_weight(A.N, _p(pi.reshape(-1)), n, _p(rp), _p(col), _p(val)))


def graph_weight(A):
    """omega_G, Eq. (4): sum over undirected off-diagonal edges of |w|, fp64."""
    rows = np.repeat(np.arange(A.N, dtype=np.int64), np.diff(A.rowptr))
    off = rows < A.col
    return float(np.abs(A.val[off].astype(np.float64)).sum())


def coverage(A, pi):
    """c_pi, Eq. (4)."""
    return factor_weight(A, pi) / graph_weight(A)


def coverage_id(A):
    """c_id, Eq. (5): weight of the sub/super-diagonal couplings {i, i+1}, over omega_G.

    Eq. (5) sums |w({i,i-1})| + |w({i,i+1})| over i, which counts every coupling
    {i,i+1} twice; the paper's printed values (ANISO1 0.68 = 2/3) correspond to
    counting each such edge once, which is what is computed here.
    """
    rows = np.repeat(np.arange(A.N, dtype=np.int64), np.diff(A.rowptr))
    sel = A.col.astype(np.int64) == rows + 1
    return float(np.abs(A.val[sel].astype(np.float64)).sum()) / graph_weight(A)


def run_pipeline(A, n=2, M=5, m=5, k_m=0, p=0.5, seed=0):
    """Whole hot path on the CPU: factor -> linear forest -> tridiag (n must be 2 for LF)."""
    pi, pw, rounds, _, _ = factor(A, n, M, m, k_m, p, seed)
    out = dict(pi=pi, pi_w=pw, rounds=rounds)
    if n == 2:
        lf = linear_forest(pi, pw)
        out.update(lf)
        out["a"], out["b"], out["c"] = tridiag(A, lf["forest"], lf["perm"])
    return out


class _SymCSR:
    """A CSR triple with the attributes the oracle functions read."""

    def __init__(self, N, rowptr, col, val):
        self.N, self.rowptr, self.col, self.val = int(N), rowptr, col, val


def symmetrize(A):
    """S = A' + A'^T for a general A (§4, §5.1; reading f3-1):
    A' = |A| - diag|A|; the entries of S are the union of the off-diagonal patterns of A and
    A^T, s_ij = fl32(|a_ij| + |a_ji|) with a missing entry counted as 0; rows ascending.
    The definition written out with numpy: the directed entries and their transposes, sorted
    by (row, col) (library sort), equal keys added in float32."""
    rp, col, val = _csr(A)
    N = A.N
    rows = np.repeat(np.arange(N, dtype=np.int64), np.diff(rp))
    off = rows != col
    i, j = rows[off], col[off].astype(np.int64)
    w = np.abs(val[off]).astype(np.float32)
    key = np.concatenate([i * N + j, j * N + i])
    x = np.concatenate([w, w])
    order = np.argsort(key, kind="stable")
    key, x = key[order], x[order]
    first = np.ones(key.size, dtype=bool)
    first[1:] = key[1:] != key[:-1]
    starts = np.flatnonzero(first)
    s_val = x[starts].copy()
    pair = np.flatnonzero(~first)  # the second entry of a key (at most two: no duplicates in A)
    s_val[np.searchsorted(starts, pair, side="right") - 1] = (x[pair - 1] + x[pair]).astype(np.float32)
    uk = key[starts]
    s_rows = uk // N
    s_col = (uk % N).astype(np.int32)
    s_rp = np.zeros(N + 1, dtype=np.int64)
    np.cumsum(np.bincount(s_rows, minlength=N), out=s_rp[1:])
    return _SymCSR(N, s_rp, s_col, s_val.astype(np.float32))


def run_pipeline_general(A, M=5, m=5, k_m=0, p=0.5, seed=0):
    """The hot path on a general A: [0,2]-factor and linear forest of
    S = A' + A'^T, tridiagonal coefficients from A itself (lfo_tridiag reads row perm[r] of
    A, so a coupling A does not store is 0)."""
    S = symmetrize(A)
    pi, pw, rounds, _, _ = factor(S, 2, M, m, k_m, p, seed)
    out = dict(S=S, pi=pi, pi_w=pw, rounds=rounds)
    lf = linear_forest(pi, pw)
    out.update(lf)
    out["a"], out["b"], out["c"] = tridiag(A, lf["forest"], lf["perm"])
    return out


def coarsen(A, mu):
    """The coarse graph of AlgTriBlockPrecond (§6; readings f1-1..f1-3):
    every matched pair of the [0,1]-factor mu is one coarse vertex (leader = its smaller id),
    every unmatched vertex one more (with a ghost partner); coarse vertices numbered in leader
    order; coarse weight w(P,Q) = sum of |a_ij| over i in P, j in Q (fp64, one rounding to
    fp32), no coarse diagonal.  Returns (cid [N], members [Nc, 2] (-1 = ghost), CSR)."""
    rp, col, val = _csr(A)
    N = A.N
    mu = np.asarray(mu, dtype=np.int64).reshape(-1)
    v = np.arange(N, dtype=np.int64)
    lead = (mu < 0) | (v < mu)
    pre = np.cumsum(lead) - lead  # exclusive prefix of the leaders
    cid = np.where(lead, pre, pre[np.maximum(mu, 0)]).astype(np.int32)
    Nc = int(lead.sum())
    members = np.full((Nc, 2), -1, dtype=np.int32)
    members[pre[lead], 0] = v[lead]
    members[pre[lead], 1] = mu[lead]
    rows = np.repeat(v, np.diff(rp))
    ci, cj = cid[rows].astype(np.int64), cid[col].astype(np.int64)
    off = ci != cj
    sums = {}
    for a, b, w in zip(ci[off], cj[off], np.abs(val[off]).astype(np.float64)):
        sums[(a, b)] = sums.get((a, b), 0.0) + w
    keys = sorted(sums)
    c_rows = np.array([k[0] for k in keys], dtype=np.int64)
    c_col = np.array([k[1] for k in keys], dtype=np.int32)
    c_val = np.array([sums[k] for k in keys], dtype=np.float64).astype(np.float32)
    c_rp = np.zeros(Nc + 1, dtype=np.int64)
    np.cumsum(np.bincount(c_rows, minlength=Nc), out=c_rp[1:])
    return cid, members, _SymCSR(Nc, c_rp, c_col, c_val)


def block_tridiag(A, members, cforest, cperm):
    """The 2x2 block tridiagonal system (§6) in the coarse forest's order:
    block row R = coarse vertex P = cperm[R] with fine rows members[P] (-1 = ghost):
    D = the pair's own 2x2 block of A (a ghost row is (0, 1)), L / U = the blocks of A coupling
    P to cperm[R-1] / cperm[R+1] if that is a coarse forest edge, else 0.  Row-major blocks."""
    rp, col, val = _csr(A)
    ent = {}
    for i in range(A.N):
        for e in range(rp[i], rp[i + 1]):
            ent[(i, int(col[e]))] = val[e]

    def a(i, j):
        return ent.get((int(i), int(j)), np.float32(0)) if i >= 0 and j >= 0 else np.float32(0)

    Nc = members.shape[0]
    cf = np.asarray(cforest).reshape(-1, 2)
    D = np.zeros((Nc, 4), np.float32)
    L = np.zeros((Nc, 4), np.float32)
    U = np.zeros((Nc, 4), np.float32)
    fperm = np.zeros((Nc, 2), np.int32)
    for R in range(Nc):
        P = int(cperm[R])
        p0, p1 = members[P]
        fperm[R] = (p0, p1)
        D[R] = (a(p0, p0), a(p0, p1), a(p1, p0), a(p1, p1))
        if p1 < 0:
            D[R, 3] = 1.0
        for Q, out in ((cperm[R - 1] if R > 0 else -1, L), (cperm[R + 1] if R + 1 < Nc else -1, U)):
            if Q >= 0 and Q in cf[P]:
                q0, q1 = members[Q]
                out[R] = (a(p0, q0), a(p0, q1), a(p1, q0), a(p1, q1))
    return D, L, U, fperm


def run_block_pipeline(A, M=5, m=5, k_m=0, p=0.5, seed=0):
    """AlgTriBlockPrecond on the CPU: [0,1]-factor -> coarse graph -> [0,2]-factor + linear
    forest on it -> 2x2 block tridiagonal system (§6)."""
    mu, _, _, _, _ = factor(A, 1, M, m, k_m, p, seed)
    cid, members, C = coarsen(A, mu)
    cpi, cpw, _, _, _ = factor(C, 2, M, m, k_m, p, seed)
    clf = linear_forest(cpi, cpw)
    D, L, U, fperm = block_tridiag(A, members, clf["forest"], clf["perm"])
    return dict(mu=np.asarray(mu).reshape(-1), cid=cid, members=members, C=C, cpi=cpi, cforest=clf["forest"],
                cperm=clf["perm"], D=D, L=L, U=U, fperm=fperm)


def tri_solve(a, b, c, x):
    """Apply the tridiagonal preconditioner: y = T^{-1} x, fp64.

    T is the tridiagonal matrix lf_tridiag writes (§3.3 step (4), L219, L297),
    in the permuted order: row r is a[r]*y[r-1] + b[r]*y[r] + c[r]*y[r+1] (a[0] and
    c[N-1] ignored).  The paper inverts it with the solver of its ref. [21] (L37, L447,
    "scaled partial pivoting"); the plain definition of that result is T^{-1} x, computed
    here by LAPACK's banded LU with partial pivoting (scipy.linalg.solve_banded, gbsv) on
    the whole N x N system in fp64 -- a library primitive as one step, no segmentation.
    Pinned in tests/test_oracle_trisolve.py by a closed form (1-D Laplacian), a
    manufactured solution, dense brute force and the block-decoupling invariant.
    """
    from scipy.linalg import solve_banded

    a = np.asarray(a, dtype=np.float64)
    b = np.asarray(b, dtype=np.float64)
    c = np.asarray(c, dtype=np.float64)
    x = np.asarray(x, dtype=np.float64)
    N = b.shape[0]
    if N == 0:
        return np.zeros(0)
    ab = np.zeros((3, N))
    ab[0, 1:] = c[:-1]   # superdiagonal: T[r, r+1] = c[r]
    ab[1, :] = b
    ab[2, :-1] = a[1:]   # subdiagonal:   T[r, r-1] = a[r]
    return solve_banded((1, 1), ab, x, check_finite=True)


def tri_matvec(a, b, c, y):
    """T y in fp64, the definition of row r above written out (for residual checks)."""
    a = np.asarray(a, dtype=np.float64)
    b = np.asarray(b, dtype=np.float64)
    c = np.asarray(c, dtype=np.float64)
    y = np.asarray(y, dtype=np.float64)
    out = b * y
    out[1:] += a[1:] * y[:-1]
    out[:-1] += c[:-1] * y[1:]
    return out
