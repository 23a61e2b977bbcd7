"""Input validation through the C ABI (include/lf.h lf_validate_csr / lf_validate_factor):
every precondition violation of PAPER.md's undirected weighted graph (L31, L231, L315) is
reported as LF_EINPUT; valid inputs (sorted or not, explicit zeros, sign-asymmetric values
with equal |a|) pass.  And lf_linear_forest on a malformed factor terminates (bounded walks)."""
import copy

import numpy as np
import pytest

import lfgen

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def lfm():
    import torch

    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_icpp_0002s22_b200 import _build, lf

    _build.build()
    lf.load()
    return lf


def dev(A):
    import torch

    return (torch.from_numpy(np.ascontiguousarray(A.rowptr)).cuda(), torch.from_numpy(np.ascontiguousarray(A.col)).cuda(),
            torch.from_numpy(np.ascontiguousarray(A.val)).cuda())


def expect(lfm, A, msg):
    if msg is None:
        lfm.validate(*dev(A))
        return
    with pytest.raises(lfm.LFError) as e:
        lfm.validate(*dev(A))
    assert "LF_EINPUT" in str(e.value) and msg in str(e.value), str(e.value)


def raw(N, rows, cols, vals):
    rows, cols = np.asarray(rows, np.int64), np.asarray(cols, np.int32)
    rp = np.zeros(N + 1, np.int64)
    np.add.at(rp, rows + 1, 1)
    return lfgen.CSR(N=N, rowptr=np.cumsum(rp), col=cols, val=np.asarray(vals, np.float32))


@pytest.mark.parametrize("make", [lambda: lfgen.config("C1"), lambda: lfgen.chung_lu(20000),
                                  lambda: lfgen.random_graph(500, 2000, seed=3, shuffle_cols_seed=5),
                                  lambda: lfgen.grid3d_27pt(10)],
                         ids=["c1", "c4_small", "shuffled_rows", "c5_small"])
def test_valid_inputs_pass(lfm, make):
    expect(lfm, make(), None)


def test_zero_entries_and_signs(lfm):
    A = lfgen.config("C1")
    B = copy.deepcopy(A)
    rows = np.repeat(np.arange(B.N), np.diff(B.rowptr))
    off = np.flatnonzero(rows != B.col)

    def partner(e):
        i, j = rows[e], B.col[e]
        return B.rowptr[j] + int(np.flatnonzero(B.col[B.rowptr[j]:B.rowptr[j + 1]] == i)[0])

    B.val[off[0]] = 0.0           # explicit zeros (both triangles): not edges (L31)
    B.val[partner(off[0])] = -0.0
    expect(lfm, B, None)
    B2 = copy.deepcopy(B)         # an edge whose partner entry is a stored zero: asymmetric
    B2.val[partner(off[0])] = A.val[off[0]]
    expect(lfm, B2, "values not symmetric")
    C = copy.deepcopy(A)          # a_ij = -a_ji: the same |w|, the same undirected edge
    i, j = rows[off[5]], C.col[off[5]]
    C.val[off[5]] = -C.val[off[5]]
    expect(lfm, C, None)


def test_rejections(lfm):
    A = lfgen.config("C1")
    rows = np.repeat(np.arange(A.N), np.diff(A.rowptr))
    off = np.flatnonzero(rows != A.col)
    # |a_ij| != |a_ji|
    B = copy.deepcopy(A)
    B.val[off[3]] *= np.float32(1.5)
    expect(lfm, B, "values not symmetric")
    # (i,j) without (j,i): drop one off-diagonal entry
    e = off[7]
    keep = np.ones(A.nnz, bool)
    keep[e] = False
    C = raw(A.N, rows[keep], A.col[keep], A.val[keep])
    expect(lfm, C, "pattern not symmetric")
    # duplicate (i,j), sorted and unsorted rows
    D = raw(3, [0, 0, 0, 1, 1, 2], [0, 1, 1, 0, 1, 2], [2, -1, -1, -1, 2, 1])
    expect(lfm, D, "duplicate")
    E = raw(3, [0, 0, 0, 1, 1, 2], [1, 0, 1, 0, 1, 2], [-1, 2, -1, -1, 2, 1])
    expect(lfm, E, "duplicate")
    # rowptr, column range, NaN
    F = copy.deepcopy(A)
    F.rowptr = F.rowptr.copy()
    F.rowptr[5], F.rowptr[6] = F.rowptr[6], F.rowptr[5]
    expect(lfm, F, "rowptr")
    G = copy.deepcopy(A)
    G.col = G.col.copy()
    G.col[10] = A.N + 3
    expect(lfm, G, "out of range")
    H = copy.deepcopy(A)
    H.val[12] = np.nan
    expect(lfm, H, "NaN")


def test_validate_factor(lfm):
    import torch

    A = lfgen.config("C1")
    fac = lfm.factor(*dev(A), 2)
    lfm.validate_factor(fac["pi"])
    bad = []
    p = fac["pi"].cpu().numpy()
    v = int(np.flatnonzero(p[:, 1] >= 0)[0])
    x = p.copy(); w = x[v, 0]; x[w][x[w] == v] = -1; x[w] = np.sort(x[w])[::-1]; bad.append((x, "symmetric"))
    x = p.copy(); x[v, 0] = v; bad.append((x, "slot"))
    x = p.copy(); x[v, 1] = x[v, 0]; bad.append((x, "slot"))
    x = p.copy(); x[v, 0] = A.N; bad.append((x, "slot"))
    x = p.copy(); u = int(np.flatnonzero(p[:, 1] < 0)[0]); x[u] = [-1, x[u, 0] if x[u, 0] >= 0 else 5]; bad.append((x, ""))
    for x, msg in bad:
        with pytest.raises(lfm.LFError) as e:
            lfm.validate_factor(torch.from_numpy(np.ascontiguousarray(x)).cuda())
        assert "LF_EINPUT" in str(e.value) and msg in str(e.value)


@pytest.mark.timeout(120)
@pytest.mark.parametrize("forest", ["tile", "grs"])
def test_linear_forest_malformed_terminates(lfm, monkeypatch, forest):
    """A non-symmetric 'factor' (one-way links forming loops): the call returns and its
    walks stop (no hang, no fault); lf_forest_stats flags what a bound caught."""
    import torch

    monkeypatch.setenv("LF_FOREST", forest)
    N = 4096
    rng = np.random.default_rng(1)
    pi = np.stack([(np.arange(N) + 1) % N, rng.permutation(N)], 1).astype(np.int32)
    pi[pi[:, 1] == np.arange(N), 1] = -1
    pw = rng.random((N, 2)).astype(np.float32)
    pw[pi < 0] = 0
    ws = lfm.Workspace()
    out = lfm.linear_forest(torch.from_numpy(pi).cuda(), torch.from_numpy(pw).cuda(), ws=ws)
    torch.cuda.synchronize()
    st = lfm.forest_stats(N, ws)
    assert "malformed_input" in st
    assert out["perm"].numel() == N
