"""Host-side multi-GPU logic on CPU with world_size-2 gloo process groups: row ranges,
halo plan agreement between ranks, NCCL unique-id broadcast."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

import lfgen


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import torch.distributed as dist

    from paper_conf_icpp_0002s22_b200 import dist as lfd

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        res = {}
        A = lfgen.grid3d_7pt_aniso(12)
        b1 = lfd.plan_bounds(A.rowptr, world)
        b2 = lfd.slab_bounds(12, 144, world)
        allb = [None] * world
        dist.all_gather_object(allb, (b1.tolist(), b2.tolist()))
        res["bounds_agree"] = all(x == allb[0] for x in allb)
        lo, hi = int(b2[rank]), int(b2[rank + 1])
        rp, col, _ = lfd.row_slice(A, lo, hi)
        send, recv = lfd.expected_halo((rp, col), lo, hi, b2)
        res["plans_agree"] = lfd.check_plans(send, recv)
        res["halo"] = (send.tolist(), recv.tolist())
        uid = lfd.broadcast_unique_id(make=lambda: bytes(range(128)))
        res["uid_ok"] = uid == bytes(range(128))
        q.put((rank, res))
    finally:
        dist.destroy_process_group()


def test_gloo_two_ranks():
    world = 2
    port = _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = dict(q.get(timeout=240) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for r in range(world):
        assert out[r]["bounds_agree"] and out[r]["plans_agree"] and out[r]["uid_ok"]
    # a 12^3 grid split into two z-slabs: each side sees one 12x12 plane of the other
    assert out[0]["halo"][1][1] == 144 and out[1]["halo"][1][0] == 144


def test_plan_bounds_properties():
    from paper_conf_icpp_0002s22_b200 import dist as lfd

    A = lfgen.chung_lu(5000)
    for G in (1, 2, 3, 8):
        b = lfd.plan_bounds(A.rowptr, G)
        assert b[0] == 0 and b[-1] == A.N and np.all(np.diff(b) >= 0) and len(b) == G + 1
    b = lfd.plan_bounds(lfgen.grid3d_7pt_aniso(8).rowptr, 4, align=64)
    assert np.all(b[1:-1] % 64 == 0)
    assert lfd.slab_bounds(10, 100, 3).tolist() == [0, 300, 600, 1000]
