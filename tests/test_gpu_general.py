"""General (non-symmetric) inputs on the CUDA path vs the oracle (
PAPER.md §4, §5.1), bit-exact: S = A' + A'^T (lf_symmetrize), the factor and the
linear forest of S, the coefficients of the original A (lf_orig_coeffs + the fused
permutation/tridiagonal copy), both forest organisations."""
import numpy as np
import pytest

import lfgen

pytestmark = pytest.mark.gpu

FOREST_MODES = ["tile", "grs"]


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

    return (torch.from_numpy(A.rowptr).cuda(), torch.from_numpy(A.col).cuda(), torch.from_numpy(A.val).cuda())


def _shuffled_rows(A, seed):
    rng = np.random.default_rng(seed)
    col, val = A.col.copy(), A.val.copy()
    for i in range(A.N):
        s, e = A.rowptr[i], A.rowptr[i + 1]
        p = rng.permutation(e - s)
        col[s:e], val[s:e] = col[s:e][p], val[s:e][p]
    return lfgen.CSR(N=A.N, rowptr=A.rowptr, col=col, val=val, name=A.name + "_shuf", meta={})


CASES = {
    "c1": lambda: lfgen.nonsymmetric(lfgen.grid2d_5pt(64, seed=1), seed=11),
    "c1_ties": lambda: lfgen.nonsymmetric(lfgen.grid2d_5pt(48, seed=1), seed=12, ties=True, zeros=0.1),
    "g27": lambda: lfgen.nonsymmetric(lfgen.grid3d_27pt(24, seed=5), seed=13, drop=0.3),
    "c4": lambda: lfgen.nonsymmetric(lfgen.chung_lu(20000, seed=4), seed=14),
    "g3": lambda: lfgen.nonsymmetric(lfgen.config("C3"), seed=7),  # bench.py's G3 input
    "rand_shuf": lambda: _shuffled_rows(lfgen.nonsymmetric(lfgen.random_graph(3000, 9000, seed=3), seed=15), 7),
}


@pytest.mark.parametrize("case", sorted(CASES))
def test_symmetrize_bit_exact(lfm, case):
    import oracle

    A = CASES[case]()
    S = oracle.symmetrize(A)
    rp, col, val = lfm.symmetrize(*dev(A))
    assert np.array_equal(rp.cpu().numpy(), S.rowptr)
    assert np.array_equal(col.cpu().numpy(), S.col)
    assert np.array_equal(val.cpu().numpy().view(np.uint32), S.val.view(np.uint32))


@pytest.mark.parametrize("forest", FOREST_MODES)
@pytest.mark.parametrize("case", sorted(CASES))
def test_general_pipeline_bit_exact(lfm, case, forest, monkeypatch):
    import oracle

    monkeypatch.setenv("LF_FOREST", forest)
    A = CASES[case]()
    o = oracle.run_pipeline_general(A)
    _, fac, lf = lfm.general_pipeline(*dev(A))
    assert np.array_equal(fac["pi"].cpu().numpy(), o["pi"])
    assert np.array_equal(fac["pi_w"].cpu().numpy(), o["pi_w"])
    for k in ("forest", "path_id", "pos", "perm", "iperm"):
        assert np.array_equal(lf[k].cpu().numpy().reshape(o[k].shape), o[k]), k
    for k in ("a", "b", "c"):
        assert np.array_equal(lf[k].cpu().numpy().view(np.uint32), o[k].view(np.uint32)), k


def test_orig_coeffs_equal_captured_values_on_symmetric_input(lfm):
    A = lfgen.config("C1")
    rp, col, val = dev(A)
    fac = lfm.factor(rp, col, val, 2)
    pv, dg = lfm.orig_coeffs(rp, col, val, fac["pi"])
    assert np.array_equal(pv.cpu().numpy().view(np.uint32), fac["pi_val"].cpu().numpy().view(np.uint32))
    assert np.array_equal(dg.cpu().numpy().view(np.uint32), fac["diag"].cpu().numpy().view(np.uint32))


def test_symmetrize_empty_and_diagonal_only(lfm):
    import torch

    # no entries at all
    rp = torch.zeros(5, dtype=torch.int64, device="cuda")
    col = torch.zeros(0, dtype=torch.int32, device="cuda")
    val = torch.zeros(0, dtype=torch.float32, device="cuda")
    s_rp, s_col, s_val = lfm.symmetrize(rp, col, val)
    assert s_rp.cpu().tolist() == [0] * 5 and s_col.numel() == 0
    # only a diagonal: S is empty
    rp = torch.arange(5, dtype=torch.int64, device="cuda")
    col = torch.arange(4, dtype=torch.int32, device="cuda")
    val = torch.full((4,), 3.0, device="cuda")
    s_rp, s_col, s_val = lfm.symmetrize(rp, col, val)
    assert s_rp.cpu().tolist() == [0] * 5 and s_col.numel() == 0
