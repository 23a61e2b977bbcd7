"""C5 (BASELINE.json configs[4]: the 512^3 27-point graph, N = 134,217,728 vertices,
3,609,741,304 stored entries > 2^31, E = 1,737,761,788) through the C ABI, bit-exact.

* The device generator (lfgen/csrc/lfgen_gpu.cu, input generation only) equals the numpy
  generator row for row at small sizes, and at full size its sha256 digests equal those
  of lfgen.grid3d_27pt_big recorded in tests/golden/c5_512_n2.json.
* The whole hot path (lf_factor n=2 M=5 + lf_linear_forest_tridiag, the launch
  configuration bench.py times) and the row-partitioned path (loopback, G = 2 and 4) on
  that graph reproduce the oracle's outputs: sha256 of pi, |w|, forest, path_id, pos,
  perm, iperm, a, b, c, plus the round count, the live-row counters and the cycle count,
  all written by scripts/make_c5_goldens.py, which calls only lfgen/ and oracle/.
* The same digests at 64^3 (tests/golden/c5_64_n2.json) exercise the machinery cheaply.
"""
import hashlib
import json
import os

import numpy as np
import pytest

import lfgen

pytestmark = pytest.mark.gpu
GOLD = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")
CHUNK = 1 << 26  # elements per device->host hashing chunk


@pytest.fixture(scope="module")
def torch_cuda():
    import torch

    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_icpp_0002s22_b200 import _build

    _build.build()
    import lfgen.gpu

    lfgen.gpu.build()
    return torch


def dsha(t):
    """sha256 of a device tensor's bytes (copied to the host in chunks)."""
    h = hashlib.sha256()
    flat = t.reshape(-1)
    for i in range(0, flat.numel(), CHUNK):
        h.update(flat[i:i + CHUNK].cpu().numpy().tobytes())
    return h.hexdigest()


def dsha_parts(ts):
    h = hashlib.sha256()
    for t in ts:
        flat = t.reshape(-1)
        for i in range(0, flat.numel(), CHUNK):
            h.update(flat[i:i + CHUNK].cpu().numpy().tobytes())
    return h.hexdigest()


def golden(n):
    p = os.path.join(GOLD, f"c5_{n}_n2.json")
    if not os.path.exists(p):
        pytest.fail(f"missing {p} (scripts/make_c5_goldens.py --n {n})")
    return json.load(open(p))


@pytest.mark.parametrize("n,nz,z0,z1", [(2, 2, 0, 2), (3, 3, 0, 3), (16, 16, 0, 16), (20, 13, 3, 9),
                                        (7, 5, 4, 5), (9, 9, 2, 2)])
def test_device_generator_equals_numpy(torch_cuda, n, nz, z0, z1):
    import lfgen.gpu

    rp, col, val = lfgen.gpu.grid27_rows(n, z0, z1, seed=5, nz=nz)
    rp_h, col_h, val_h, lo, hi = lfgen.grid3d_27pt_rows(n, z0, z1, seed=5, nz=nz)
    assert np.array_equal(rp.cpu().numpy(), rp_h)
    assert np.array_equal(col.cpu().numpy(), col_h)
    assert np.array_equal(val.cpu().numpy().view(np.uint32), val_h.view(np.uint32))


def _run_single(torch, n):
    import lfgen.gpu
    from paper_conf_icpp_0002s22_b200 import lf

    lf.load()
    rp, col, val = lfgen.gpu.grid27_rows(n, 0, n, seed=5)
    P = lf.Pipeline(rp, col, val).run()
    torch.cuda.synchronize()
    return (rp, col, val), P


def _check_single(torch, n, check_csr):
    g = golden(n)
    (rp, col, val), P = _run_single(torch, n)
    assert rp.numel() - 1 == g["N"] and col.numel() == g["nnz"]
    if check_csr:
        for k, t in (("rowptr", rp), ("col", col), ("val", val)):
            assert dsha(t) == g["sha256"][k], k
    del rp, col, val
    assert int(P.fac["rounds"].item()) == g["rounds"]
    live = P.fac["live"].cpu().numpy()
    assert [int(x) for x in live[:5]] == g["live_rows"]
    assert [int(x) for x in live[5:10]] == g["live_nnz"]
    assert int(P.lf["n_cycles"].item()) == g["n_cycles"]
    idx = torch.as_tensor(np.asarray(g["sample_idx"], dtype=np.int64), device="cuda")
    s = g["sample"]
    # sampled values first (a readable failure), then the digests of every output
    assert P.fac["pi"][idx].cpu().numpy().tolist() == s["pi"]
    assert P.lf["path_id"][idx].cpu().numpy().tolist() == s["path_id"]
    assert P.lf["pos"][idx].cpu().numpy().tolist() == s["pos"]
    assert P.lf["perm"][idx].cpu().numpy().tolist() == s["perm"]
    outs = {"pi": P.fac["pi"], "pi_w": P.fac["pi_w"], "forest": P.lf["forest"], "path_id": P.lf["path_id"],
            "pos": P.lf["pos"], "perm": P.lf["perm"], "iperm": P.lf["iperm"], "a": P.tri[0], "b": P.tri[1],
            "c": P.tri[2]}
    for k, t in outs.items():
        assert dsha(t) == g["sha256"][k], k
    del P
    torch.cuda.empty_cache()


def test_c5_recipe_64_digests(torch_cuda):
    _check_single(torch_cuda, 64, check_csr=True)


def test_c5_full_single_gpu(torch_cuda):
    """C5 at full size, one B200: generator digests + every output digest (nnz > 2^31)."""
    _check_single(torch_cuda, 512, check_csr=True)


def _check_parts(torch, n, G):
    import lfgen.gpu
    from paper_conf_icpp_0002s22_b200 import dist

    g = golden(n)
    bounds = dist.slab_bounds(n, n * n, G)
    comm = dist.Comm.loopback(G)
    parts = []
    for r in range(G):
        z0, z1 = int(bounds[r]) // (n * n), int(bounds[r + 1]) // (n * n)
        rp, col, val = lfgen.gpu.grid27_rows(n, z0, z1, seed=5)
        parts.append(dist.Partition(rp, col, val, bounds, r, n=2))
    dist.factor(parts, comm)
    dist.linear_forest(parts, comm)
    tri = dist.tridiag(parts, comm)
    fac = [p.export(5) for p in parts]
    fe = [p.forest_export() for p in parts]
    torch.cuda.synchronize()
    assert int(fac[0]["rounds"].item()) == g["rounds"]
    live = fac[0]["live"].cpu().numpy()
    assert [int(x) for x in live[:5]] == g["live_rows"]
    assert [int(x) for x in live[5:10]] == g["live_nnz"]
    assert int(fe[0]["n_cycles"].item()) == g["n_cycles"]
    assert dsha_parts([f["pi"] for f in fac]) == g["sha256"]["pi"]
    assert dsha_parts([f["pi_w"] for f in fac]) == g["sha256"]["pi_w"]
    for k in ("forest", "path_id", "pos", "iperm"):
        assert dsha_parts([f[k] for f in fe]) == g["sha256"][k], k
    for i, k in enumerate(("a_owner", "b_owner", "c_owner")):
        assert dsha_parts([t[i] for t in tri]) == g["sha256"][k], k
    for p in parts:
        p.close()
    comm.close()
    del parts, tri, fac, fe
    torch.cuda.empty_cache()


@pytest.mark.parametrize("G", [2, 3])
def test_c5_recipe_64_partitioned(torch_cuda, G):
    _check_parts(torch_cuda, 64, G)


def test_c5_full_partitioned_loopback(torch_cuda):
    """The multi-GPU path's z-slab partition of C5 (4 ranks, loopback exchange on one GPU)."""
    _check_parts(torch_cuda, 512, 4)
