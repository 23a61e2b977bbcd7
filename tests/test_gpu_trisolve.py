"""lf_tri_solve (applying the tridiagonal preconditioner, PAPER.md
L37, L447, ref. [21]) through the C ABI vs oracle.tri_solve (fp64 banded LU).

Tolerance (readings f2-3 and f2-5): the kernel computes in fp32 (L301), the oracle in fp64, so
results agree up to rounding, not bit for bit.  Two bars, both derived from fp32
Gaussian elimination with partial pivoting on a tridiagonal system (growth factor <= 2):
  backward error  per independent block B (split where a[r] = c[r-1] = 0):
                  ||x - T y||_B / (||T||_B ||y||_B + ||x||_B) <= 16 eps32 (inf-norms; any
                  nonsingular T: each U entry takes <= 2 roundings and the pivoting keeps
                  the growth small -- componentwise error is NOT bounded by |T||y| under
                  pivoting, so the normwise form is the one that holds)
  forward error   ||y - y_oracle||_inf <= 1e-4 ||y_oracle||_inf  (diagonally dominant
                  T, as every linear-forest T of the graphs here is: cond_inf <= ~1e2)
A diagonal T (every row its own segment) is one reciprocal (MUFU + Newton, <= 1 ulp) and
one product per row (<= 0.5 ulp): within 3 ulp of the fp32 quotient (reading f2-5).
Inputs a, b, c always come from the oracle pipeline or the test, never from the GPU.
"""
import numpy as np
import pytest

import lfgen

pytestmark = pytest.mark.gpu

EPS32 = float(np.finfo(np.float32).eps)


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


def gpu_solve(torch, lfm, a, b, c, x):
    t = [torch.from_numpy(np.ascontiguousarray(v, dtype=np.float32)).cuda() for v in (a, b, c, x)]
    y = lfm.tri_solve(*t)
    torch.cuda.synchronize()
    return y.cpu().numpy()


def check(oracle_mod, a, b, c, x, y, forward=True):
    a, b, c, x = (np.asarray(v, np.float32) for v in (a, b, c, x))
    assert np.all(np.isfinite(y))
    r = np.abs(x.astype(np.float64) - oracle_mod.tri_matvec(a, b, c, y))
    # normwise backward error of every independent block (split where a[r] = c[r-1] = 0)
    N = b.shape[0]
    st = np.flatnonzero(np.r_[True, (a[1:] == 0) & (c[:-1] == 0)])
    rowT = np.abs(a).astype(np.float64) + np.abs(b) + np.abs(c)
    rowT[0] -= abs(float(a[0]))
    rowT[N - 1] -= abs(float(c[N - 1]))
    den = (np.maximum.reduceat(rowT, st) * np.maximum.reduceat(np.abs(y.astype(np.float64)), st)
           + np.maximum.reduceat(np.abs(x.astype(np.float64)), st))
    be = np.max(np.maximum.reduceat(r, st) / np.maximum(den, 1e-300))
    assert be <= 16 * EPS32, f"backward error {be:.3e} (block normwise)"
    if forward:
        yo = oracle_mod.tri_solve(a, b, c, x)
        fe = np.max(np.abs(y - yo)) / max(np.max(np.abs(yo)), 1e-300)
        assert fe <= 1e-4, f"forward error {fe:.3e}"


def pipeline_tri(oracle_mod, A):
    o = oracle_mod.run_pipeline(A)
    return o["a"], o["b"], o["c"]


@pytest.mark.parametrize("name,make", [
    ("c1", lambda: lfgen.config("C1")),
    ("aniso1_64", lambda: lfgen.aniso2d(64, 1)),
    ("c2_small", lambda: lfgen.grid3d_7pt_aniso(24)),
    ("c3_small", lambda: lfgen.fem27_bricks(20)),
    ("c4_small", lambda: lfgen.chung_lu(20000)),
    ("random_ties", lambda: lfgen.random_graph(3000, 9000, seed=5, ties=True)),
], ids=lambda v: v if isinstance(v, str) else "")
def test_linear_forest_systems(torch_cuda, lfm, oracle_mod, name, make):
    """T from the oracle's [0,2]-factor + linear forest + tridiag of the graph; x random
    and the paper's manufactured right-hand side T sin(16 pi i / N) (L437)."""
    A = make()
    a, b, c = pipeline_tri(oracle_mod, A)
    N = A.N
    rng = np.random.default_rng(11)
    xs = [rng.standard_normal(N).astype(np.float32)]
    xt = np.sin(16 * np.pi * np.arange(N) / N)
    xs.append(oracle_mod.tri_matvec(a, b, c, xt).astype(np.float32))
    dominant = bool(np.all(np.abs(b) > np.abs(a) + np.abs(c)))
    for x in xs:
        y = gpu_solve(torch_cuda, lfm, a, b, c, x)
        check(oracle_mod, a, b, c, x, y, forward=dominant)


def test_random_segments_pivoting(torch_cuda, lfm, oracle_mod):
    """Non-dominant random rows (pivot interchanges on about half the steps), ragged
    segment lengths 1..400 split by a[r] = c[r-1] = 0, tiny diagonals."""
    rng = np.random.default_rng(3)
    N = 150_000
    a = rng.uniform(-1, 1, N).astype(np.float32)
    b = rng.uniform(-1, 1, N).astype(np.float32)
    c = rng.uniform(-1, 1, N).astype(np.float32)
    b[rng.random(N) < 0.1] *= 1e-4
    cuts = np.cumsum(rng.integers(1, 401, N // 50))
    cuts = cuts[cuts < N]
    a[cuts] = 0.0
    c[cuts - 1] = 0.0
    x = rng.standard_normal(N).astype(np.float32)
    y = gpu_solve(torch_cuda, lfm, a, b, c, x)
    check(oracle_mod, a, b, c, x, y, forward=False)


def test_one_long_segment(torch_cuda, lfm, oracle_mod):
    """A single path of 300k rows (one thread walks it): dominant 1-D operator."""
    N = 300_000
    rng = np.random.default_rng(4)
    a = -rng.uniform(0.5, 1, N).astype(np.float32)
    c = -rng.uniform(0.5, 1, N).astype(np.float32)
    b = (np.abs(a) + np.abs(c) + rng.uniform(0.1, 1, N)).astype(np.float32)
    x = rng.standard_normal(N).astype(np.float32)
    y = gpu_solve(torch_cuda, lfm, a, b, c, x)
    check(oracle_mod, a, b, c, x, y)


def test_diagonal_bit_exact_and_edges(torch_cuda, lfm, oracle_mod):
    torch = torch_cuda
    rng = np.random.default_rng(8)
    for N in (1, 2, 31, 32, 33, 4097):
        b = rng.uniform(0.5, 2, N).astype(np.float32) * rng.choice([-1, 1], N)
        z = np.zeros(N, np.float32)
        x = rng.standard_normal(N).astype(np.float32)
        y = gpu_solve(torch, lfm, z, b, z, x)
        yo = oracle_mod.tri_solve(z, b, z, x)
        # x * rcp(b), rcp = MUFU approximation + one Newton step (~1 ulp), then one
        # rounding of the product -> within 3 ulp of the fp32-rounded quotient
        assert np.all(np.abs(y - yo) <= 3 * np.spacing(np.abs(yo.astype(np.float32))))
    # N = 1 with garbage in the ignored a[0], c[N-1]
    y = gpu_solve(torch, lfm, np.array([5.0]), np.array([2.0]), np.array([7.0]), np.array([3.0]))
    assert abs(y[0] - 1.5) <= 3 * np.spacing(np.float32(1.5))
    # N = 0 is a no-op; y aliasing x is rejected
    e = torch.empty(0, device="cuda")
    lfm.tri_solve(e, e, e, e)
    v = torch.ones(4, device="cuda")
    with pytest.raises(lfm.LFError):
        lfm.tri_solve(v, v, v, v, out=v)


def test_c2_full_size(torch_cuda, lfm, oracle_mod):
    """The bench workload (C2, N = 2^21): T from the oracle pipeline, x random."""
    A = lfgen.config("C2")
    a, b, c = pipeline_tri(oracle_mod, A)
    x = np.random.default_rng(2).standard_normal(A.N).astype(np.float32)
    y = gpu_solve(torch_cuda, lfm, a, b, c, x)
    check(oracle_mod, a, b, c, x, y)


@pytest.mark.parametrize("N", [1, 31, 32, 33, 2047, 2048, 2049, 100_003])
def test_dominant_ragged_couplings(torch_cuda, lfm, oracle_mod, N):
    """Diagonally dominant T (the partition path): two-sided cuts at random rows and at
    multiples of the 32-row chunk, one-sided zero couplings (a[r] = 0 with c[r-1] != 0),
    ragged N around the chunk and block sizes."""
    rng = np.random.default_rng(N)
    a = -rng.uniform(0.1, 1, N).astype(np.float32)
    c = -rng.uniform(0.1, 1, N).astype(np.float32)
    b = (np.abs(a) + np.abs(c) + rng.uniform(0.01, 0.5, N)).astype(np.float32)
    cut = np.flatnonzero((rng.random(N) < 0.02) | (np.arange(N) % 32 == 0) & (rng.random(N) < 0.5))
    cut = cut[cut > 0]
    a[cut] = 0.0
    c[cut - 1] = 0.0
    a[rng.random(N) < 0.01] = 0.0
    c[rng.random(N) < 0.01] = 0.0
    x = rng.standard_normal(N).astype(np.float32)
    y = gpu_solve(torch_cuda, lfm, a, b, c, x)
    check(oracle_mod, a, b, c, x, y)


def test_unaligned_inputs(torch_cuda, lfm, oracle_mod):
    """a, b, c, x as 4-byte-offset views (the staging falls back from 16-byte loads to
    4-byte copies): same bar as aligned inputs."""
    torch = torch_cuda
    N = 50_001
    rng = np.random.default_rng(21)
    a = -rng.uniform(0.1, 1, N).astype(np.float32)
    c = -rng.uniform(0.1, 1, N).astype(np.float32)
    b = (np.abs(a) + np.abs(c) + rng.uniform(0.01, 0.5, N)).astype(np.float32)
    cut = np.flatnonzero(rng.random(N) < 0.01)
    cut = cut[cut > 0]
    a[cut] = 0.0
    c[cut - 1] = 0.0
    x = rng.standard_normal(N).astype(np.float32)
    views = []
    for v in (a, b, c, x):
        buf = torch.empty(N + 1, device="cuda")
        buf[1:] = torch.from_numpy(v).cuda()
        views.append(buf[1:])
    y = lfm.tri_solve(*views)
    torch.cuda.synchronize()
    check(oracle_mod, a, b, c, x, y.cpu().numpy())


def test_pivoting_path_forward_error_per_block(torch_cuda, lfm, oracle_mod):
    """The scaled-partial-pivoting path (k_seg_solve: taken because T is not diagonally
    dominant) against oracle.tri_solve element by element: well-conditioned, non-dominant
    blocks of 2..12 rows (|b| < |a| + |c| in most rows, pivot interchanges), each block's
    forward error within 64 kappa_inf(B) eps32 of the fp64 solution (DESIGN.md reading
    f2-5: fp32 elimination with growth <= 2 on a tridiagonal block)."""
    rng = np.random.default_rng(17)
    blocks, kap = [], []
    while sum(len(b_[1]) for b_ in blocks) < 60_000:
        L = int(rng.integers(2, 13))
        a = rng.uniform(-1, 1, L).astype(np.float32)
        c = rng.uniform(-1, 1, L).astype(np.float32)
        b = (rng.uniform(-0.3, 0.3, L)).astype(np.float32)
        a[0] = 0.0
        c[-1] = 0.0
        D = np.diag(b.astype(np.float64)) + np.diag(a[1:].astype(np.float64), -1) + np.diag(c[:-1].astype(np.float64), 1)
        k = np.linalg.cond(D, np.inf)
        if not np.isfinite(k) or k > 1e3:
            continue
        blocks.append((a, b, c))
        kap.append(k)
    a = np.concatenate([x[0] for x in blocks])
    b = np.concatenate([x[1] for x in blocks])
    c = np.concatenate([x[2] for x in blocks])
    assert np.mean(np.abs(b) < np.abs(a) + np.abs(c)) > 0.5  # mostly non-dominant rows
    x = rng.standard_normal(b.shape[0]).astype(np.float32)
    y = gpu_solve(torch_cuda, lfm, a, b, c, x)
    yo = oracle_mod.tri_solve(a, b, c, x)
    s = 0
    for (ab, bb, cb), k in zip(blocks, kap):
        e = s + bb.shape[0]
        err = np.max(np.abs(y[s:e] - yo[s:e])) / max(np.max(np.abs(yo[s:e])), 1e-30)
        assert err <= 64 * k * EPS32, (s, err, k)
        s = e
