"""Graph/matrix generators (see package docstring). numpy only, seeded, deterministic.

Recipes: SURVEY.md §8(d) "Concrete synthetic inputs" and Appendix A.3 (ANISO stencils,
PAPER.md:L303-L311). Every generator returns a symmetric CSR matrix A whose
off-diagonal magnitudes |a_uv| are the edge weights |w({u,v})| of the paper's graph
("each matrix entry a_ij corresponds to the weight of the edge").
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np

GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_DROP_SALT = np.uint64(0xD1B54A32D192ED03)
_JIT_SALT = np.uint64(0xA0761D6478BD642F)


@dataclass
class CSR:
    """Symmetric sparse matrix, CSR, diagonal included."""

    N: int
    rowptr: np.ndarray  # int64 [N+1]
    col: np.ndarray  # int32 [Z]
    val: np.ndarray  # float32 [Z]
    name: str = ""
    meta: dict = field(default_factory=dict)

    @property
    def nnz(self) -> int:
        return int(self.rowptr[-1])

    @property
    def n_edges(self) -> int:
        """Undirected off-diagonal edges with nonzero weight (E in SURVEY.md §8)."""
        if "E_exact" in self.meta:  # closed form of a streamed generator (no O(nnz) temporaries)
            return int(self.meta["E_exact"])
        rows = np.repeat(np.arange(self.N, dtype=np.int64), np.diff(self.rowptr))
        off = (rows != self.col) & (self.val != 0)
        return int(off.sum()) // 2

    def dense(self) -> np.ndarray:
        A = np.zeros((self.N, self.N), dtype=np.float64)
        rows = np.repeat(np.arange(self.N), np.diff(self.rowptr))
        A[rows, self.col] = self.val
        return A


def splitmix64(x):
    """SplitMix64 finaliser on uint64 (wrap-around arithmetic)."""
    z = np.asarray(x, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = z + GOLDEN
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        return z ^ (z >> np.uint64(31))


def edge_hash_u(s, t, N, seed, salt=np.uint64(0)):
    """u in [0,1) on a 24-bit grid for the undirected edge {s,t}."""
    s = np.asarray(s, dtype=np.uint64)
    t = np.asarray(t, dtype=np.uint64)
    lo = np.minimum(s, t)
    hi = np.maximum(s, t)
    with np.errstate(over="ignore"):
        x = np.uint64(seed) ^ salt ^ ((lo * np.uint64(N) + hi) * GOLDEN)
    h = splitmix64(x) >> np.uint64(40)
    return h.astype(np.float64) * (2.0 ** -24)


def csr_from_edges(N, s, t, w_abs, diag="rowsum", sign=-1.0, name="", meta=None,
                   shuffle_cols_seed=None):
    """Symmetric CSR from undirected edges {s,t} with |a_st| = w_abs.

    a_st = a_ts = sign * w_abs. Diagonal: "rowsum" -> sum_j |a_vj| + 1 (fp64 sum,
    rounded to fp32), a float -> that constant, None -> no diagonal entries stored.
    shuffle_cols_seed permutes columns inside each row (inputs need not be sorted).
    """
    s = np.asarray(s, dtype=np.int64)
    t = np.asarray(t, dtype=np.int64)
    w = np.asarray(w_abs, dtype=np.float32)
    assert s.shape == t.shape == w.shape
    assert np.all(s != t), "self loops are not edges"
    off_val = (np.float32(sign) * w).astype(np.float32)
    rows = [s, t]
    cols = [t, s]
    vals = [off_val, off_val]
    if diag is not None:
        v = np.arange(N, dtype=np.int64)
        if isinstance(diag, str) and diag == "rowsum":
            aw = np.abs(w.astype(np.float64))
            acc = np.bincount(s, weights=aw, minlength=N) + np.bincount(t, weights=aw, minlength=N)
            d = (acc + 1.0).astype(np.float32)
        else:
            d = np.full(N, np.float32(diag), dtype=np.float32)
        rows.append(v)
        cols.append(v)
        vals.append(d)
    r = np.concatenate(rows)
    c = np.concatenate(cols)
    x = np.concatenate(vals)
    key = r * np.int64(N) + c
    if shuffle_cols_seed is None:
        order = np.argsort(key, kind="stable")
    else:
        rng = np.random.default_rng(shuffle_cols_seed)
        order = np.lexsort((rng.random(r.shape[0]), r))
    ks = key[order]
    if ks.size > 1 and shuffle_cols_seed is None:
        assert not np.any(ks[1:] == ks[:-1]), "duplicate (i,j)"
    r = r[order]
    col = c[order].astype(np.int32)
    val = x[order]
    counts = np.bincount(r, minlength=N).astype(np.int64)
    rowptr = np.zeros(N + 1, dtype=np.int64)
    np.cumsum(counts, out=rowptr[1:])
    m = dict(meta or {})
    m.setdefault("E", int(s.shape[0]))
    return CSR(N=int(N), rowptr=rowptr, col=col, val=val, name=name, meta=m)


# ---------------------------------------------------------------------------
# structured grids
# ---------------------------------------------------------------------------

def _grid_edges_2d(nx, ny, offsets):
    """Forward offsets (dx,dy) on an nx x ny grid, id = x + nx*y."""
    ss, tt, kk = [], [], []
    y, x = np.meshgrid(np.arange(ny, dtype=np.int64), np.arange(nx, dtype=np.int64),
                       indexing="ij")
    for i, (dx, dy) in enumerate(offsets):
        ok = (x + dx >= 0) & (x + dx < nx) & (y + dy >= 0) & (y + dy < ny)
        src = (x + nx * y)[ok]
        ss.append(src)
        tt.append(src + dx + nx * dy)
        kk.append(np.full(src.shape, i, dtype=np.int64))
    return np.concatenate(ss), np.concatenate(tt), np.concatenate(kk)


def grid2d_5pt(nx=64, ny=None, seed=1, ties=False, diag="rowsum", shuffle_cols_seed=None):
    """C1: 2D 5-point Laplacian graph on nx*ny, seeded weights w = 1-u in (0,1].

    ties=True draws w from {1,2,3,4}/4 instead (tie-heavy test variant, §8(d)).
    """
    ny = nx if ny is None else ny
    N = nx * ny
    s, t, _ = _grid_edges_2d(nx, ny, [(1, 0), (0, 1)])
    u = edge_hash_u(s, t, N, seed)
    if ties:
        w = (np.floor(u * 4.0) + 1.0) / 4.0
    else:
        w = 1.0 - u
    return csr_from_edges(N, s, t, w, diag=diag, name=f"grid2d_5pt_{nx}x{ny}",
                          meta={"seed": seed, "ties": ties}, shuffle_cols_seed=shuffle_cols_seed)


# ANISO stencils: rows = dy +1,0,-1
# (printed top row couples to the +nx neighbour), cols = dx -1,0,+1.
ANISO = {
    1: [[-0.2, -0.1, -0.2], [-1.0, 3.0, -1.0], [-0.2, -0.1, -0.2]],
    2: [[-0.1, -0.2, -1.0], [-0.2, 3.0, -0.2], [-1.0, -0.2, -0.1]],
}


def aniso2d(nx=2500, kind=1):
    """ANISO1/ANISO2: 2D 9-point stencil on an nx x nx grid."""
    S = ANISO[kind]
    N = nx * nx
    fwd = [(1, 0), (-1, 1), (0, 1), (1, 1)]  # (dx, dy) with the partner (-dx,-dy)

    def coef(dx, dy):
        return S[1 - dy][dx + 1]

    for dx, dy in fwd:
        assert coef(dx, dy) == coef(-dx, -dy), "stencil not symmetric"
    s, t, k = _grid_edges_2d(nx, nx, fwd)
    w = np.array([abs(coef(dx, dy)) for dx, dy in fwd], dtype=np.float32)[k]
    return csr_from_edges(N, s, t, w, diag=np.float32(S[1][1]), name=f"aniso{kind}_{nx}",
                          meta={"kind": kind, "nx": nx})


def _grid3d_edges(nx, ny, nz, offsets, z_lo=0, z_hi=None):
    """Forward 3D offsets (dx,dy,dz) on nx*ny*nz, natural id = x + nx*(y + ny*z).

    Only sources with z in [z_lo, z_hi) are emitted (slab generation)."""
    z_hi = nz if z_hi is None else z_hi
    zz, yy, xx = np.meshgrid(np.arange(z_lo, z_hi, dtype=np.int64),
                             np.arange(ny, dtype=np.int64),
                             np.arange(nx, dtype=np.int64), indexing="ij")
    ss, tt, kk = [], [], []
    vid = xx + nx * (yy + ny * zz)
    for i, (dx, dy, dz) in enumerate(offsets):
        ok = ((xx + dx >= 0) & (xx + dx < nx) & (yy + dy >= 0) & (yy + dy < ny)
              & (zz + dz >= 0) & (zz + dz < nz))
        src = vid[ok]
        ss.append(src)
        tt.append(src + dx + nx * (dy + ny * dz))
        kk.append(np.full(src.shape, i, dtype=np.int64))
    return np.concatenate(ss), np.concatenate(tt), np.concatenate(kk)


def grid3d_7pt_aniso(n=128, seed=2, eps=(1.0, 0.1, 0.01)):
    """C2: 3D 7-point anisotropic Laplacian graph, |w| = eps_d * (1 + 0.25u)."""
    N = n ** 3
    s, t, k = _grid3d_edges(n, n, n, [(1, 0, 0), (0, 1, 0), (0, 0, 1)])
    u = edge_hash_u(s, t, N, seed)
    w = np.asarray(eps, dtype=np.float64)[k] * (1.0 + 0.25 * u)
    return csr_from_edges(N, s, t, w, name=f"grid3d_7pt_aniso_{n}",
                          meta={"seed": seed, "n": n})


def grid3d_7pt_aniso_rows(n, nz, z_lo, z_hi, seed=2, eps=(1.0, 0.1, 0.01)):
    """Rows of the planes [z_lo, z_hi) of the n x n x nz 7-point anisotropic graph (the C2
    recipe on a taller grid), with GLOBAL column ids: rowptr (rebased), col, val, lo, hi.

    Equal to rows [lo, hi) of grid3d_7pt_aniso on the same grid (tests check this); used
    to give every rank of a multi-GPU run its own slab without building the whole graph."""
    N = n * n * nz
    plane = n * n
    lo, hi = z_lo * plane, z_hi * plane
    v = np.arange(lo, hi, dtype=np.int64)
    x, y, z = v % n, (v // n) % n, v // plane
    offs = [(-plane, z > 0, 2), (-n, y > 0, 1), (-1, x > 0, 0), (0, None, None), (1, x < n - 1, 0),
            (n, y < n - 1, 1), (plane, z < nz - 1, 2)]
    cols, vals, masks = [], [], []
    wsum = np.zeros(v.shape[0], dtype=np.float64)
    for d, m, ax in offs:
        if d == 0:
            continue
        j = v + d
        u = edge_hash_u(v, j, N, seed)
        w = (np.asarray(eps, dtype=np.float64)[ax] * (1.0 + 0.25 * u)).astype(np.float32)
        wsum += np.where(m, np.abs(w.astype(np.float64)), 0.0)
    diag = (wsum + 1.0).astype(np.float32)
    for d, m, ax in offs:
        j = v + d
        if d == 0:
            cols.append(j)
            vals.append(diag)
            masks.append(np.ones(v.shape[0], dtype=bool))
            continue
        u = edge_hash_u(v, j, N, seed)
        w = (np.asarray(eps, dtype=np.float64)[ax] * (1.0 + 0.25 * u)).astype(np.float32)
        cols.append(j)
        vals.append(-w)
        masks.append(m)
    C = np.stack(cols, 1)
    V = np.stack(vals, 1)
    Mk = np.stack(masks, 1)
    counts = Mk.sum(1).astype(np.int64)
    rowptr = np.zeros(v.shape[0] + 1, dtype=np.int64)
    np.cumsum(counts, out=rowptr[1:])
    return rowptr, C[Mk].astype(np.int32), V[Mk].astype(np.float32), lo, hi


def _fwd27():
    out = []
    for dz in (-1, 0, 1):
        for dy in (-1, 0, 1):
            for dx in (-1, 0, 1):
                if (dz, dy, dx) > (0, 0, 0):
                    out.append((dx, dy, dz))
    return out


def grid3d_27pt(n=512, seed=5):
    """C5 (and small replicas): 3D 27-point graph, natural order, w = 1 - u."""
    N = n ** 3
    s, t, _ = _grid3d_edges(n, n, n, _fwd27())
    w = 1.0 - edge_hash_u(s, t, N, seed)
    return csr_from_edges(N, s, t, w, name=f"grid3d_27pt_{n}", meta={"seed": seed, "n": n})


def grid3d_27pt_slab_edges(n, z_lo, z_hi, seed=5):
    """Edges of the 27-pt graph whose smaller endpoint lies in planes [z_lo, z_hi)."""
    N = n ** 3
    s, t, _ = _grid3d_edges(n, n, n, _fwd27(), z_lo, z_hi)
    w = (1.0 - edge_hash_u(s, t, N, seed)).astype(np.float32)
    return s, t, w


# the 27 stencil offsets (dx, dy, dz) in ascending column order of a natural-order row
_OFF27 = [(dx, dy, dz) for dz in (-1, 0, 1) for dy in (-1, 0, 1) for dx in (-1, 0, 1)]


def grid27_nnz(n, z_lo=0, z_hi=None, nz=None):
    """Stored entries (diagonal included) of the planes [z_lo, z_hi) of the n x n x nz
    27-point graph: every row stores cx*cy*cz entries, c = 3 minus the missing sides."""
    nz = n if nz is None else nz
    z_hi = nz if z_hi is None else z_hi
    s = 3 * n - 2 if n > 1 else 1
    cz = sum(3 - (z == 0) - (z == nz - 1) if nz > 1 else 1 for z in range(z_lo, z_hi))
    return s * s * cz


def grid3d_27pt_rows(n, z_lo, z_hi, seed=5, nz=None):
    """Rows of the planes [z_lo, z_hi) of the n x n x nz 27-point graph (the C5 recipe:
    natural order, w = 1 - u), with GLOBAL column ids: rowptr (rebased), col, val, lo, hi.

    Row by row, the same matrix as grid3d_27pt (tests/test_gen.py checks it at small n):
    columns ascend because the offsets are visited in (dz, dy, dx) order, and the diagonal
    is the exact fp64 sum of the row's |w| plus 1 (every w is a multiple of 2^-24, so the
    sum is exact in any order) rounded to fp32.  Needs only O(rows) memory, so the 512^3
    graph (3.6e9 entries) can be built slab by slab (grid3d_27pt_big)."""
    nz = n if nz is None else nz
    N = n * n * nz
    plane = n * n
    lo, hi = z_lo * plane, z_hi * plane
    v = np.arange(lo, hi, dtype=np.int64)
    x, y, z = v % n, (v // n) % n, v // plane
    C = np.empty((v.shape[0], 27), dtype=np.int64)
    W = np.zeros((v.shape[0], 27), dtype=np.float32)
    Mk = np.empty((v.shape[0], 27), dtype=bool)
    for i, (dx, dy, dz) in enumerate(_OFF27):
        m = ((x + dx >= 0) & (x + dx < n) & (y + dy >= 0) & (y + dy < n)
             & (z + dz >= 0) & (z + dz < nz))
        j = v + dx + n * (dy + n * dz)
        C[:, i] = j
        Mk[:, i] = m
        if (dx, dy, dz) != (0, 0, 0):
            jj = np.where(m, j, v + 1)  # any valid id; masked out below
            W[:, i] = np.where(m, (1.0 - edge_hash_u(v, jj, N, seed)), 0.0).astype(np.float32)
    diag = (np.abs(W.astype(np.float64)).sum(1) + 1.0).astype(np.float32)
    V = -W
    V[:, 13] = diag  # offset (0, 0, 0)
    counts = Mk.sum(1).astype(np.int64)
    rowptr = np.zeros(v.shape[0] + 1, dtype=np.int64)
    np.cumsum(counts, out=rowptr[1:])
    return rowptr, C[Mk].astype(np.int32), V[Mk].astype(np.float32), lo, hi


def grid3d_27pt_big(n=512, seed=5, planes_per_chunk=2):
    """The whole n^3 27-point graph (C5) built slab by slab into preallocated arrays
    (30 GB at n = 512, no temporaries of that size).  Same matrix as grid3d_27pt."""
    N = n ** 3
    Z = grid27_nnz(n)
    rowptr = np.empty(N + 1, dtype=np.int64)
    col = np.empty(Z, dtype=np.int32)
    val = np.empty(Z, dtype=np.float32)
    rowptr[0] = 0
    e = 0
    for z0 in range(0, n, planes_per_chunk):
        z1 = min(n, z0 + planes_per_chunk)
        rp, c, w, lo, hi = grid3d_27pt_rows(n, z0, z1, seed)
        rowptr[lo + 1:hi + 1] = rp[1:] + e
        col[e:e + c.shape[0]] = c
        val[e:e + c.shape[0]] = w
        e += c.shape[0]
    assert e == Z
    E = (Z - N) // 2
    return CSR(N=N, rowptr=rowptr, col=col, val=val, name=f"grid3d_27pt_{n}",
               meta={"seed": seed, "n": n, "E": E, "E_exact": E})


def fem27_bricks(n=100, seed=3, dropout=0.02, brick=5, jitter=0.3):
    """C3: jittered 27-pt lattice, 2% dropout, brick-ordered labels ("FEM-like").

    |w| = (0.5 + (1-u)) / l^2 with l^2 the squared distance of the jittered points.
    """
    N = n ** 3
    s, t, _ = _grid3d_edges(n, n, n, _fwd27())
    # seeded dropout of 2% of the lattice edges
    d = edge_hash_u(s, t, N, seed, salt=_DROP_SALT)
    keep = d >= dropout
    s, t = s[keep], t[keep]
    # per-vertex jitter in [-jitter, jitter) per coordinate
    vid = np.arange(N, dtype=np.uint64)
    jit = []
    for c in range(3):
        with np.errstate(over="ignore"):
            h = splitmix64(np.uint64(seed) ^ _JIT_SALT ^ ((vid * np.uint64(3) + np.uint64(c)) * GOLDEN))
        jit.append(((h >> np.uint64(40)).astype(np.float64) * 2.0 ** -24 * 2.0 - 1.0) * jitter)

    def pos(v):
        x = v % n
        y = (v // n) % n
        z = v // (n * n)
        return (x + jit[0][v], y + jit[1][v], z + jit[2][v])

    ps, pt = pos(s), pos(t)
    l2 = sum((a - b) ** 2 for a, b in zip(ps, pt))
    u = edge_hash_u(s, t, N, seed)
    w = (0.5 + (1.0 - u)) / l2
    # brick relabelling: bricks in seeded random order, natural order inside a brick
    nb = n // brick
    assert nb * brick == n
    rng = np.random.default_rng(seed)
    brick_rank = np.empty(nb ** 3, dtype=np.int64)
    brick_rank[rng.permutation(nb ** 3)] = np.arange(nb ** 3, dtype=np.int64)
    v = np.arange(N, dtype=np.int64)
    x, y, z = v % n, (v // n) % n, v // (n * n)
    b = (x // brick) + nb * ((y // brick) + nb * (z // brick))
    loc = (x % brick) + brick * ((y % brick) + brick * (z % brick))
    label = brick_rank[b] * brick ** 3 + loc
    return csr_from_edges(N, label[s], label[t], w, name=f"fem27_bricks_{n}",
                          meta={"seed": seed, "n": n, "dropout": dropout})


def chung_lu(N=5_000_000, gamma=2.3, dbar=8.0, dmax=50_000, seed=4):
    """C4: Chung-Lu power-law graph with seeded random labels, w = 1 - u."""
    rng = np.random.default_rng(seed)
    i = np.arange(N, dtype=np.float64)
    wt = (i + 1.0) ** (-1.0 / (gamma - 1.0))
    wt *= dbar * N / wt.sum()
    wt = np.minimum(wt, dmax)
    cdf = np.cumsum(wt)
    cdf /= cdf[-1]
    m = int(round(N * dbar / 2))
    # iid endpoint pairs: sorted queries make searchsorted cache-friendly; pairing the
    # sorted a-draws with a random permutation of the sorted b-draws keeps pairs iid.
    a = np.searchsorted(cdf, np.sort(rng.random(m)), side="right")
    b = np.searchsorted(cdf, np.sort(rng.random(m)), side="right")[rng.permutation(m)]
    a = np.minimum(a, N - 1)
    b = np.minimum(b, N - 1)
    ok = a != b
    a, b = a[ok], b[ok]
    lo, hi = np.minimum(a, b).astype(np.int64), np.maximum(a, b).astype(np.int64)
    key = np.sort(lo * np.int64(N) + hi)
    key = key[np.concatenate(([True], key[1:] != key[:-1]))]
    lo, hi = key // N, key % N
    relabel = rng.permutation(N).astype(np.int64)
    s, t = relabel[lo], relabel[hi]
    w = 1.0 - edge_hash_u(s, t, N, seed)
    return csr_from_edges(N, s, t, w, name=f"chung_lu_{N}",
                          meta={"seed": seed, "gamma": gamma, "dbar": dbar})


def random_graph(N, E, seed=0, ties=False, diag="rowsum", shuffle_cols_seed=None):
    """Small random simple graph for property tests (E distinct edges, seeded)."""
    rng = np.random.default_rng(seed)
    maxE = N * (N - 1) // 2
    E = min(E, maxE)
    if E == 0:
        s = t = np.zeros(0, dtype=np.int64)
    else:
        keys = set()
        while len(keys) < E:
            a = rng.integers(0, N, size=2 * (E - len(keys)) + 8)
            b = rng.integers(0, N, size=a.shape[0])
            for x, y in zip(a.tolist(), b.tolist()):
                if x != y:
                    keys.add((min(x, y), max(x, y)))
                    if len(keys) == E:
                        break
        ks = sorted(keys)
        s = np.array([k[0] for k in ks], dtype=np.int64)
        t = np.array([k[1] for k in ks], dtype=np.int64)
    u = edge_hash_u(s, t, N, seed)
    w = (np.floor(u * 4.0) + 1.0) / 4.0 if ties else 1.0 - u
    return csr_from_edges(N, s, t, w, diag=diag, name=f"random_{N}_{E}_{seed}",
                          meta={"seed": seed, "ties": ties}, shuffle_cols_seed=shuffle_cols_seed)


def directed_hash_u(i, j, N, seed):
    """u in [0,1) on a 24-bit grid for the ORDERED pair (i, j) (input generation only)."""
    i = np.asarray(i, dtype=np.uint64)
    j = np.asarray(j, dtype=np.uint64)
    with np.errstate(over="ignore"):
        x = np.uint64(seed) ^ np.uint64(0xA5A5A5A5) ^ ((i * np.uint64(N) + j) * GOLDEN)
    return (splitmix64(x) >> np.uint64(40)).astype(np.float64) * (2.0 ** -24)


def nonsymmetric(base, seed=7, drop=0.15, zeros=0.02, ties=False):
    """A general (non-symmetric) matrix on the pattern of `base` (PAPER.md
    L231, L315): every off-diagonal directed entry (i,j) of base is dropped with probability
    `drop`, stored as an explicit zero with probability `zeros`, else gets its own value
    a_ij = -(0.5 + u_ij) from a hash of the ORDERED pair (so a_ij != a_ji); `ties` rounds
    the values to multiples of 1/4 (many equal |a_ij| + |a_ji|).  The diagonal of base is
    kept.  Columns stay ascending within rows."""
    N = base.N
    rows = np.repeat(np.arange(N, dtype=np.int64), np.diff(base.rowptr))
    col = base.col.astype(np.int64)
    off = rows != col
    u = directed_hash_u(rows, col, N, seed)
    r2 = directed_hash_u(col, rows, N, seed + 1)  # an independent draw for the drop / zero tests
    keep = ~off | (r2 >= drop)
    val = np.where(off, -(0.5 + u), base.val.astype(np.float64))
    if ties:
        val = np.where(off, -np.round((0.5 + u) * 4.0) / 4.0, val)
    val = np.where(off & (r2 >= drop) & (r2 < drop + zeros), 0.0, val).astype(np.float32)
    rows, col, val = rows[keep], col[keep].astype(np.int32), val[keep]
    counts = np.bincount(rows, minlength=N).astype(np.int64)
    rowptr = np.zeros(N + 1, dtype=np.int64)
    np.cumsum(counts, out=rowptr[1:])
    return CSR(N=int(N), rowptr=rowptr, col=col, val=val, name=f"nonsym_{base.name}",
               meta={"seed": seed, "drop": drop, "zeros": zeros, "base": base.name})


CONFIG_NAMES = ("C1", "C2", "C3", "C4", "C5")


def config(name, scale=None):
    """BASELINE.json configs. `scale` shrinks for tests."""
    if name == "C1":
        return grid2d_5pt(64 if scale is None else scale, seed=1)
    if name == "C2":
        return grid3d_7pt_aniso(128 if scale is None else scale, seed=2)
    if name == "C3":
        return fem27_bricks(100 if scale is None else scale, seed=3)
    if name == "C4":
        return chung_lu(5_000_000 if scale is None else scale, seed=4)
    if name == "C5":
        return grid3d_27pt(512 if scale is None else scale, seed=5)
    raise KeyError(name)
