"""Small cases for compute-sanitizer runs (memcheck / racecheck / synccheck / initcheck):
the single-GPU pipeline in both forest modes (tile path, global ruling set) and both round
modes (cached, rows), factors n = 1..4, the row-partitioned path through the loopback
exchange (G = 3), general inputs (f3), the block preconditioner (f1) and lf_tri_solve -- every
result still compared with the oracle."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import lfgen  # noqa: E402
import oracle  # noqa: E402
from paper_conf_icpp_0002s22_b200 import dist, lf  # noqa: E402

lf.load()
oracle.build()


def dev(A):
    return tuple(torch.from_numpy(x).cuda() for x in (A.rowptr, A.col, A.val))


def check_pipeline(A, tag):
    P = lf.Pipeline(*dev(A)).run()
    torch.cuda.synchronize()
    o = oracle.run_pipeline(A)
    assert np.array_equal(P.fac["pi"].cpu().numpy(), o["pi"]), tag
    for k in ("forest", "path_id", "pos", "perm", "iperm"):
        assert np.array_equal(P.lf[k].cpu().numpy(), o[k]), (tag, k)
    for g, e in zip(P.tri, (o["a"], o["b"], o["c"])):
        assert np.array_equal(g.cpu().numpy().view(np.uint32), e.view(np.uint32)), tag
    return P


graphs = [("C1", lfgen.config("C1")), ("C2-32", lfgen.grid3d_7pt_aniso(32)), ("C5-16", lfgen.grid3d_27pt(16)),
          ("C3-15", lfgen.fem27_bricks(15)), ("C4-20k", lfgen.chung_lu(20000))]
for forest in ("tile", "grs"):
    for rounds in ("cached", "rows"):
        os.environ["LF_FOREST"] = forest
        if rounds == "rows":
            os.environ["LF_NO_CACHED_ROUNDS"] = "1"
        else:
            os.environ.pop("LF_NO_CACHED_ROUNDS", None)
        for name, A in graphs:
            check_pipeline(A, f"{name}/{forest}/{rounds}")
            print("ok pipeline", name, forest, rounds, flush=True)
os.environ.pop("LF_FOREST", None)
os.environ.pop("LF_NO_CACHED_ROUNDS", None)
A = lfgen.config("C1")
for n in (1, 3, 4):
    out = lf.factor(*dev(A), n)
    torch.cuda.synchronize()
    assert np.array_equal(out["pi"].cpu().numpy(), oracle.factor(A, n)[0])
print("ok factor n=1,3,4", flush=True)
for name, A in graphs[:2]:
    G = 3
    bounds = dist.plan_bounds(A.rowptr, G)
    comm = dist.Comm.loopback(G)
    parts = [dist.Partition(*(torch.from_numpy(x).cuda() for x in dist.row_slice(A, int(bounds[r]), int(bounds[r + 1]))),
                            bounds, r, n=2) for r in range(G)]
    dist.factor(parts, comm)
    dist.linear_forest(parts, comm)
    dist.tridiag(parts, comm)
    fe = [p.forest_export() for p in parts]
    torch.cuda.synchronize()
    o = oracle.run_pipeline(A)
    assert np.array_equal(np.concatenate([f["path_id"].cpu().numpy() for f in fe]), o["path_id"])
    for p in parts:
        p.close()
    comm.close()
    print("ok partitioned loopback", name, flush=True)
for name, base in graphs[:3]:  # general inputs in both forest modes
    A = lfgen.nonsymmetric(base, seed=5)
    o = oracle.run_pipeline_general(A)
    for forest in ("tile", "grs"):
        os.environ["LF_FOREST"] = forest
        _, fac, lfo = lf.general_pipeline(*dev(A))
        torch.cuda.synchronize()
        assert np.array_equal(lfo["perm"].cpu().numpy(), o["perm"]), (name, forest)
        assert np.array_equal(lfo["a"].cpu().numpy().view(np.uint32), o["a"].view(np.uint32)), (name, forest)
    os.environ.pop("LF_FOREST", None)
    print("ok general", name, flush=True)
for name, A in graphs[:3]:  # AlgTriBlockPrecond
    o = oracle.run_block_pipeline(A)
    g = lf.block_pipeline(*dev(A))
    torch.cuda.synchronize()
    assert np.array_equal(g["fperm"].cpu().numpy(), o["fperm"]), name
    for k in ("D", "L", "U"):
        assert np.array_equal(g[k].cpu().numpy().view(np.uint32), o[k].view(np.uint32)), (name, k)
    print("ok block", name, flush=True)
A = lfgen.config("C1")
P = check_pipeline(A, "C1")
x = np.random.default_rng(0).standard_normal(A.N).astype(np.float32)
y = lf.tri_solve(*P.tri, torch.from_numpy(x).cuda()).cpu().numpy()
yo = oracle.tri_solve(*(t.cpu().numpy() for t in P.tri), x)
assert np.max(np.abs(y - yo)) <= 1e-4 * np.max(np.abs(yo))
print("ok tri_solve", flush=True)
print("ALL OK")
