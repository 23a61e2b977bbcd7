"""AlgTriBlockPrecond construction on the CUDA path vs the oracle (
PAPER.md §6), bit-exact: the [0,1]-factor, the coarse graph (lf_coarsen), its
[0,2]-factor and linear forest, the 2x2 blocks and the fine order (lf_block_tridiag)."""
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

    return (torch.from_numpy(A.rowptr).cuda(), torch.from_numpy(A.col).cuda(), torch.from_numpy(A.val).cuda())


CASES = {
    "c1": lambda: lfgen.config("C1"),
    "aniso1": lambda: lfgen.aniso2d(64, 1),
    "g27": lambda: lfgen.grid3d_27pt(20, seed=5),
    "c2s": lambda: lfgen.config("C2", scale=32),
    "c4s": lambda: lfgen.chung_lu(30000, seed=4),
    "c3": lambda: lfgen.config("C3"),  # bench.py's B3 input
}


@pytest.mark.parametrize("m", [1, 5])
@pytest.mark.parametrize("case", sorted(CASES))
def test_block_pipeline_bit_exact(lfm, case, m):
    import oracle

    A = CASES[case]()
    o = oracle.run_block_pipeline(A, m=m)
    g = lfm.block_pipeline(*dev(A), m=m)
    assert np.array_equal(g["mu"].cpu().numpy().reshape(-1), o["mu"])
    assert np.array_equal(g["cid"].cpu().numpy(), o["cid"])
    assert np.array_equal(g["members"].cpu().numpy(), o["members"])
    c_rp, c_col, c_val = (x.cpu().numpy() for x in g["coarse"])
    assert np.array_equal(c_rp, o["C"].rowptr)
    assert np.array_equal(c_col, o["C"].col)
    assert np.array_equal(c_val.view(np.uint32), o["C"].val.view(np.uint32))
    assert np.array_equal(g["cpi"].cpu().numpy(), o["cpi"])
    assert np.array_equal(g["cforest"].cpu().numpy().reshape(-1), o["cforest"].reshape(-1))
    assert np.array_equal(g["cperm"].cpu().numpy(), o["cperm"])
    assert np.array_equal(g["fperm"].cpu().numpy(), o["fperm"])
    for k in ("D", "L", "U"):
        assert np.array_equal(g[k].cpu().numpy().view(np.uint32), o[k].view(np.uint32)), k


def test_block_no_match(lfm):
    """A diagonal-only matrix: no edge, every vertex a coarse vertex with a ghost."""
    import torch

    N = 10
    rp = torch.arange(N + 1, dtype=torch.int64, device="cuda")
    col = torch.arange(N, dtype=torch.int32, device="cuda")
    val = torch.full((N,), 2.0, device="cuda")
    g = lfm.block_pipeline(rp, col, val)
    assert g["members"].shape[0] == N
    assert (g["fperm"][:, 1] == -1).all()
    assert torch.equal(g["D"].cpu(), torch.tensor([[2.0, 0.0, 0.0, 1.0]] * N))
    assert (g["L"] == 0).all() and (g["U"] == 0).all()
