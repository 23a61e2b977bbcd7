"""CUDA path (through the C ABI) vs the CPU oracle, element by element, bit-exact.

Parity bar (DESIGN.md §3 reading c18): factor edges, |w|, signed values, diagonal, live-row counters,
round count, forest, path IDs, positions, perm/iperm and a/b/c are integer or copied fp32
data, so every comparison is exact equality (no tolerance).
"""
import os

import numpy as np
import pytest

import lfgen

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def torch_cuda():
    import torch

    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_icpp_0002s22_b200 import _build

    _build.build()
    return torch


@pytest.fixture(scope="module")
def lfm(torch_cuda):
    from paper_conf_icpp_0002s22_b200 import lf

    lf.load()
    return lf


def dev(torch, A):
    return (torch.from_numpy(A.rowptr).cuda(), torch.from_numpy(A.col).cuda(),
            torch.from_numpy(A.val).cuda())


def _slot_values(A, pi):
    """signed a_{v,pi[v,s]} looked up in the CSR (0 for padding) -- test-side check."""
    N, n = pi.shape
    out = np.zeros((N, n), np.float32)
    rows = np.repeat(np.arange(N, dtype=np.int64), np.diff(A.rowptr))
    key = rows * N + A.col
    order = np.argsort(key)
    ks = key[order]
    for s in range(n):
        w = pi[:, s].astype(np.int64)
        ok = w >= 0
        q = np.arange(N, dtype=np.int64)[ok] * N + w[ok]
        idx = np.searchsorted(ks, q)
        out[ok, s] = A.val[order[idx]]
    return out


def _diag(A):
    rows = np.repeat(np.arange(A.N, dtype=np.int64), np.diff(A.rowptr))
    d = np.zeros(A.N, np.float32)
    sel = rows == A.col
    d[rows[sel]] = A.val[sel]
    return d


def check_factor(torch, lfm, oracle_mod, A, n, **kw):
    rp, col, val = dev(torch, A)
    M = kw.get("M", 5)
    until = kw.get("until_maximal", False)
    out = lfm.factor(rp, col, val, n, live=not until, **kw)
    torch.cuda.synchronize()
    pi_o, pw_o, rounds_o, lr, ln = oracle_mod.factor(A, n, counters=not until, **kw)
    pi = out["pi"].cpu().numpy()
    pw = out["pi_w"].cpu().numpy()
    assert np.array_equal(pi, pi_o), f"pi mismatch at {np.argwhere((pi != pi_o).any(1))[:5].ravel()}"
    assert np.array_equal(pw.view(np.uint32), pw_o.view(np.uint32))
    assert np.array_equal(out["pi_val"].cpu().numpy().view(np.uint32),
                          _slot_values(A, pi_o).view(np.uint32))
    assert np.array_equal(out["diag"].cpu().numpy().view(np.uint32), _diag(A).view(np.uint32))
    assert int(out["rounds"].item()) == rounds_o
    if not until and M > 0:
        live = out["live"].cpu().numpy()
        assert np.array_equal(live[:M], lr), (live[:M], lr)
        assert np.array_equal(live[M:2 * M], ln)
    return out, (pi_o, pw_o)


def check_forest(torch, lfm, oracle_mod, A, fac, ref):
    lf_out = lfm.linear_forest(fac["pi"], fac["pi_w"])
    a, b, c = lfm.tridiag(lf_out["forest"], lf_out["iperm"], fac["pi"], fac["pi_val"], fac["diag"])
    torch.cuda.synchronize()
    o = oracle_mod.linear_forest(*ref)
    for k in ("forest", "path_id", "pos", "perm", "iperm"):
        got = lf_out[k].cpu().numpy()
        assert np.array_equal(got, o[k]), f"{k} mismatch: first at {np.argwhere(got != o[k])[:3].ravel()}"
    assert int(lf_out["n_cycles"].item()) == o["n_cycles"]
    ta, tb, tc = oracle_mod.tridiag(A, o["forest"], o["perm"])
    for g, e in ((a, ta), (b, tb), (c, tc)):
        assert np.array_equal(g.cpu().numpy().view(np.uint32), e.view(np.uint32))
    # the fused call (what the pipeline / bench run) gives the same outputs
    fu = lfm.linear_forest_tridiag(fac["pi"], fac["pi_w"], fac["pi_val"], fac["diag"])
    torch.cuda.synchronize()
    for k in ("forest", "path_id", "pos", "perm", "iperm"):
        got = fu[k].cpu().numpy()
        assert np.array_equal(got, o[k]), f"fused {k} mismatch: first at {np.argwhere(got != o[k])[:3].ravel()}"
    assert int(fu["n_cycles"].item()) == o["n_cycles"]
    for g, e in ((fu["a"], ta), (fu["b"], tb), (fu["c"], tc)):
        assert np.array_equal(g.cpu().numpy().view(np.uint32), e.view(np.uint32)), "fused tridiag mismatch"
    return lf_out


SMALL = [
    ("c1", lambda: lfgen.config("C1")),
    ("grid_ties", lambda: lfgen.grid2d_5pt(40, seed=3, ties=True)),
    ("grid_shuffled_cols", lambda: lfgen.grid2d_5pt(33, 17, seed=4, shuffle_cols_seed=9)),
    ("aniso1_64", lambda: lfgen.aniso2d(64, 1)),
    ("aniso2_50", lambda: lfgen.aniso2d(50, 2)),
    ("c2_small", lambda: lfgen.grid3d_7pt_aniso(24)),
    ("c3_small", lambda: lfgen.fem27_bricks(20)),
    ("c4_small", lambda: lfgen.chung_lu(20000)),
    ("c5_small", lambda: lfgen.grid3d_27pt(16)),
    ("random_ties_nodiag", lambda: lfgen.random_graph(3000, 9000, seed=5, ties=True, diag=None)),
]


@pytest.mark.parametrize("name,make", SMALL, ids=[s[0] for s in SMALL])
@pytest.mark.parametrize("n", [1, 2, 3, 4])
def test_factor_small(torch_cuda, lfm, oracle_mod, name, make, n):
    A = make()
    check_factor(torch_cuda, lfm, oracle_mod, A, n)


def with_zeros(A, seed=7, frac=0.15):
    """A copy of A with ~frac of its edges stored as explicit +0.0 and ~frac as -0.0 (both
    triangles): zero entries are not edges (PAPER.md:L31 w(e) != 0; A' = |A| - diag, L231)."""
    import copy

    B = copy.deepcopy(A)
    rows = np.repeat(np.arange(B.N, dtype=np.int64), np.diff(B.rowptr))
    col = B.col.astype(np.int64)
    off = rows != col
    u = lfgen.edge_hash_u(rows, col, B.N, seed)  # symmetric in (row, col)
    B.val[off & (u < frac)] = np.float32(0.0)
    B.val[off & (u >= frac) & (u < 2 * frac)] = np.float32(-0.0)
    B.name = A.name + "_zeros"
    return B


SMALL_ZEROS = [
    ("c1_zeros", lambda: with_zeros(lfgen.config("C1"))),
    ("c5_small_zeros", lambda: with_zeros(lfgen.grid3d_27pt(12), frac=0.3)),
    ("random_zeros_shuffled", lambda: with_zeros(lfgen.random_graph(2000, 7000, seed=2, shuffle_cols_seed=4))),
]
FOREST_MODES = ["tile", "grs"]  # DESIGN.md §5.4 tile path / §5.5 global ruling set


@pytest.mark.parametrize("forest", FOREST_MODES)
@pytest.mark.parametrize("name,make", SMALL + SMALL_ZEROS, ids=[s[0] for s in SMALL + SMALL_ZEROS])
def test_pipeline_small(torch_cuda, lfm, oracle_mod, monkeypatch, name, make, forest):
    monkeypatch.setenv("LF_FOREST", forest)
    A = make()
    fac, ref = check_factor(torch_cuda, lfm, oracle_mod, A, 2)
    check_forest(torch_cuda, lfm, oracle_mod, A, fac, ref)


@pytest.mark.parametrize("name,make", SMALL_ZEROS, ids=[s[0] for s in SMALL_ZEROS])
@pytest.mark.parametrize("n", [1, 3, 4])
def test_factor_explicit_zeros(torch_cuda, lfm, oracle_mod, name, make, n):
    A = make()
    assert (A.val == 0).sum() > 0 and np.signbit(A.val[A.val == 0]).any()
    check_factor(torch_cuda, lfm, oracle_mod, A, n)


@pytest.mark.parametrize("m,k_m,M,seed", [(5, 1, 5, 0), (1, 0, 7, 0), (3, 2, 9, 17), (2, 1, 6, 123)])
def test_factor_charge_schedules(torch_cuda, lfm, oracle_mod, m, k_m, M, seed):
    """Charged first rounds (k_m != 0) and other schedules, several seeds (L316-L320)."""
    for A in (lfgen.grid2d_5pt(48, seed=2), lfgen.fem27_bricks(10)):
        for n in (1, 2, 4):
            check_factor(torch_cuda, lfm, oracle_mod, A, n, M=M, m=m, k_m=k_m, seed=seed)


def test_factor_until_maximal(torch_cuda, lfm, oracle_mod):
    """M_max mode (L23-L25): ANISO config (1) closed form nx/2+2 and config (3)."""
    A = lfgen.aniso2d(60, 1)
    out, _ = check_factor(torch_cuda, lfm, oracle_mod, A, 2, M=0, m=1, k_m=0, until_maximal=True)
    assert int(out["rounds"].item()) == 32
    check_factor(torch_cuda, lfm, oracle_mod, lfgen.aniso2d(40, 2), 2, M=0, m=5, k_m=1,
                 until_maximal=True)


@pytest.mark.parametrize("forest", FOREST_MODES)
def test_edge_cases(torch_cuda, lfm, oracle_mod, monkeypatch, forest):
    """Empty graph, single vertex, edgeless graph, M=0, a single path, a single cycle."""
    monkeypatch.setenv("LF_FOREST", forest)
    torch = torch_cuda
    cases = [
        lfgen.csr_from_edges(1, np.zeros(0, int), np.zeros(0, int), np.zeros(0)),
        lfgen.csr_from_edges(7, np.zeros(0, int), np.zeros(0, int), np.zeros(0)),
        lfgen.csr_from_edges(2, np.array([0]), np.array([1]), np.array([0.5])),
        lfgen.csr_from_edges(5, np.arange(4), np.arange(1, 5), np.array([0.1, 0.2, 0.3, 0.4])),
        # a 6-cycle with equal weights: ties decide the weakest edge (reading c9)
        lfgen.csr_from_edges(6, np.arange(6), (np.arange(6) + 1) % 6, np.full(6, 0.25)),
        lfgen.csr_from_edges(300, np.arange(300), (np.arange(300) + 1) % 300,
                             np.linspace(1, 2, 300)),
    ]
    for A in cases:
        fac, ref = check_factor(torch, lfm, oracle_mod, A, 2)
        check_forest(torch, lfm, oracle_mod, A, fac, ref)
    A = lfgen.grid2d_5pt(8)
    check_factor(torch, lfm, oracle_mod, A, 2, M=0)


@pytest.mark.parametrize("forest", FOREST_MODES)
def test_long_paths_and_cycles(torch_cuda, lfm, oracle_mod, monkeypatch, forest):
    """A 2-factor that is one huge cycle and one long path: ranking across 2^17 steps."""
    monkeypatch.setenv("LF_FOREST", forest)
    N = 1 << 17
    s = np.arange(N - 1)
    t = s + 1
    w = 1.0 - lfgen.edge_hash_u(s, t, N, 3)
    # a path 0..N/2-1, a cycle N/2..N-1
    keep = s != N // 2 - 1
    s2 = np.concatenate([s[keep], [N - 1]])
    t2 = np.concatenate([t[keep], [N // 2]])
    w2 = np.concatenate([w[keep], [0.5]])
    A = lfgen.csr_from_edges(N, s2, t2, w2)
    fac, ref = check_factor(torch_cuda, lfm, oracle_mod, A, 2, M=3)
    check_forest(torch_cuda, lfm, oracle_mod, A, fac, ref)


@pytest.mark.parametrize("forest", FOREST_MODES)
def test_random_graph_sweep(torch_cuda, lfm, oracle_mod, monkeypatch, forest):
    monkeypatch.setenv("LF_FOREST", forest)
    for seed in range(6):
        A = lfgen.random_graph(2000 + 300 * seed, 5000 + 2000 * seed, seed=seed, ties=seed % 2 == 0,
                               shuffle_cols_seed=seed if seed % 3 == 0 else None)
        fac, ref = check_factor(torch_cuda, lfm, oracle_mod, A, 2, seed=seed)
        check_forest(torch_cuda, lfm, oracle_mod, A, fac, ref)


# ---------------------------------------------------------------------------
# BASELINE.json configs at full size (the launch configuration bench.py times)
# ---------------------------------------------------------------------------

@pytest.mark.parametrize("n", [1, 2, 3, 4])
def test_c2_full_size(torch_cuda, lfm, oracle_mod, n):
    A = _cached("C2")
    fac, ref = check_factor(torch_cuda, lfm, oracle_mod, A, n)
    if n == 2:
        check_forest(torch_cuda, lfm, oracle_mod, A, fac, ref)


def test_factor_unaligned_inputs(torch_cuda, lfm, oracle_mod):
    """CSR arrays that are offset views (col/val 4-byte, rowptr 8-byte aligned, not 16):
    the round-0 stream must fall back from bulk copies to per-thread staging."""
    torch = torch_cuda
    A = _cached("C1")
    pad = lambda x: torch.cat([torch.zeros(1, dtype=x.dtype), x]).cuda()[1:]
    rp, col, val = pad(torch.from_numpy(A.rowptr)), pad(torch.from_numpy(A.col)), pad(torch.from_numpy(A.val))
    assert col.data_ptr() % 16 != 0 and rp.data_ptr() % 16 != 0
    out = lfm.factor(rp, col, val, 2, live=True)
    torch.cuda.synchronize()
    pi_o, pw_o, rounds_o, lr, ln = oracle_mod.factor(A, 2, counters=True)
    assert np.array_equal(out["pi"].cpu().numpy(), pi_o)
    assert np.array_equal(out["pi_w"].cpu().numpy().view(np.uint32), pw_o.view(np.uint32))
    assert np.array_equal(out["live"].cpu().numpy()[:5], lr)


@pytest.mark.parametrize("cfg", ["C2", "C3"])
def test_repeated_runs_cached_and_uncached_rounds(torch_cuda, lfm, oracle_mod, monkeypatch, cfg):
    """Rounds 1..M-1 in both modes (shared-memory cached / global worklists),
    five back-to-back runs each on one workspace without a host sync in between: every run
    equals the oracle-checked first one (catches races that a single run can miss)."""
    torch = torch_cuda
    A = _cached(cfg)
    ref, _ = check_factor(torch, lfm, oracle_mod, A, 2)
    rp, col, val = dev(torch, A)
    ws = lfm.Workspace()
    for mode in ("cached", "uncached"):
        if mode == "uncached":
            monkeypatch.setenv("LF_NO_CACHED_ROUNDS", "1")
        else:
            monkeypatch.delenv("LF_NO_CACHED_ROUNDS", raising=False)
        outs = [lfm.factor(rp, col, val, 2, live=True, ws=ws) for _ in range(5)]
        torch.cuda.synchronize()
        for i, out in enumerate(outs):
            for k in ("pi", "pi_w", "pi_val", "live", "rounds"):
                assert torch.equal(out[k], ref[k]), f"{mode} run {i}: {k} differs"
    monkeypatch.delenv("LF_NO_CACHED_ROUNDS", raising=False)


@pytest.mark.parametrize("forest", FOREST_MODES)
@pytest.mark.parametrize("cfg", ["C1", "C2", "C3", "C4"])
def test_config_full_size(torch_cuda, lfm, oracle_mod, monkeypatch, cfg, forest):
    monkeypatch.setenv("LF_FOREST", forest)
    A = _cached(cfg)
    fac, ref = check_factor(torch_cuda, lfm, oracle_mod, A, 2)
    check_forest(torch_cuda, lfm, oracle_mod, A, fac, ref)


def test_pipeline_host_matches(torch_cuda, lfm, oracle_mod):
    """lf_pipeline_host (HOST buffers, the e2e entry) gives the oracle's perm and a/b/c."""
    torch = torch_cuda
    A = _cached("C1")
    rp = torch.from_numpy(A.rowptr).pin_memory()
    col = torch.from_numpy(A.col).pin_memory()
    val = torch.from_numpy(A.val).pin_memory()
    perm, pid, pos, a, b, c = lfm.pipeline_host(rp, col, val)
    o = oracle_mod.run_pipeline(A)
    assert np.array_equal(perm.numpy(), o["perm"])
    assert np.array_equal(pid.numpy(), o["path_id"])
    assert np.array_equal(pos.numpy(), o["pos"])
    for g, e in ((a, o["a"]), (b, o["b"]), (c, o["c"])):
        assert np.array_equal(g.numpy().view(np.uint32), e.view(np.uint32))


def test_native_library_loaded(torch_cuda, lfm):
    lfm.load()
    maps = open("/proc/self/maps").read()
    assert "liblf.so" in maps


_CACHE = {}


def _cached(name):
    if name not in _CACHE:
        _CACHE[name] = lfgen.config(name)
    return _CACHE[name]


def canonical_factor(N, s, t, w):
    """A [0,2]-factor (max degree 2) from undirected edges, in lf_factor's canonical slot
    form: slots sorted by (|w| desc, id asc), -1 padding last (reading c8)."""
    pi = -np.ones((N, 2), np.int32)
    pw = np.zeros((N, 2), np.float32)
    nbrs = [[] for _ in range(N)]
    for a, b, x in zip(s.tolist(), t.tolist(), np.asarray(w, np.float32).tolist()):
        nbrs[a].append((-x, b))
        nbrs[b].append((-x, a))
    for v, L in enumerate(nbrs):
        assert len(L) <= 2
        for i, (nx, u) in enumerate(sorted(L)):
            pi[v, i] = u
            pw[v, i] = -nx
    return pi, pw


@pytest.mark.parametrize("forest", FOREST_MODES)
@pytest.mark.parametrize("ties", [False, True])
def test_forest_cycles_and_paths_of_all_lengths(torch_cuda, lfm, oracle_mod, monkeypatch, forest, ties):
    """Cycles of every length 3..300 and paths of length 1..300 under a random relabelling,
    given directly as a [0,2]-factor: in GRS mode most short cycles hold no splitter (they
    are walked by their lowest-priority vertex) and long ones several; tie-heavy weights
    exercise reading c9."""
    torch = torch_cuda
    monkeypatch.setenv("LF_FOREST", forest)
    rng = np.random.default_rng(11 + ties)
    segs, N = [], 0
    for L in list(range(3, 301)) + [1000, 4099]:
        segs.append(("c", N, L))
        N += L
    for L in list(range(1, 301)) + [2000]:
        segs.append(("p", N, L))
        N += L
    N += 37  # isolated vertices
    lab = rng.permutation(N)
    s, t = [], []
    for kind, b, L in segs:
        ids = np.arange(b, b + L)
        if kind == "c":
            s += ids.tolist(); t += np.roll(ids, -1).tolist()
        else:
            s += ids[:-1].tolist(); t += ids[1:].tolist()
    s, t = lab[np.array(s)], lab[np.array(t)]
    w = (np.floor(rng.random(s.shape[0]) * 3) + 1) / 4 if ties else 1.0 - lfgen.edge_hash_u(s, t, N, 5)
    pi, pw = canonical_factor(N, s, t, w)
    o = oracle_mod.linear_forest(pi, pw)
    out = lfm.linear_forest(torch.from_numpy(pi).cuda(), torch.from_numpy(pw).cuda())
    torch.cuda.synchronize()
    for k in ("forest", "path_id", "pos", "perm", "iperm"):
        got = out[k].cpu().numpy()
        assert np.array_equal(got, o[k]), f"{k} mismatch: first at {np.argwhere(got != o[k])[:3].ravel()}"
    assert int(out["n_cycles"].item()) == o["n_cycles"] == 300
