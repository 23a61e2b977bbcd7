"""Multi-GPU binding: the factor rounds row-partitioned across GPUs.

Argument marshalling around include/lf.h's lf_comm_* / lf_part_* calls plus the host-side
planning that needs no GPU (row ranges, unique-id broadcast, plan checks), which the
gloo tests exercise on CPU.  torch.distributed is used only as the process group that
carries the NCCL unique id; the halo exchange itself runs inside liblf over NCCL.
"""
from __future__ import annotations

import ctypes as C

import numpy as np

from . import lf as _lf


def plan_bounds(rowptr, G, align=1):
    """Contiguous row ranges with balanced stored entries (rowptr: host int64 [N+1]).

    Returns int64 bounds[G+1] (bounds[0] = 0, bounds[G] = N, non-decreasing); with align > 1
    every inner bound is a multiple of `align` (e.g. a z-plane of a grid)."""
    rowptr = np.asarray(rowptr, dtype=np.int64)
    N = rowptr.shape[0] - 1
    Z = int(rowptr[-1])
    b = np.zeros(G + 1, dtype=np.int64)
    for g in range(1, G):
        r = int(np.searchsorted(rowptr, Z * g // G, side="left"))
        if align > 1:
            r = int(round(r / align)) * align
        b[g] = min(max(r, b[g - 1]), N)
    b[G] = N
    return b


def slab_bounds(nz, plane, G):
    """Equal z-slabs of an nx*ny*nz grid with natural ordering: plane = nx*ny."""
    cuts = [(nz * g) // G for g in range(G + 1)]
    return np.asarray([c * plane for c in cuts], dtype=np.int64)


def row_slice(A, lo, hi):
    """Rows [lo, hi) of a host CSR as (rowptr rebased, col (global), val) numpy arrays."""
    a, b = int(A.rowptr[lo]), int(A.rowptr[hi])
    return (A.rowptr[lo:hi + 1] - a).astype(np.int64), A.col[a:b], A.val[a:b]


def expected_halo(A_rows_cols, lo, hi, bounds):
    """Host reference of the exchange plan of one rank: (send counts, recv counts) per peer,
    from its own rows' columns (numpy; used by tests and by check_plans)."""
    rowptr, col = A_rows_cols
    G = len(bounds) - 1
    owner = np.searchsorted(bounds, col, side="right") - 1
    rows = np.repeat(np.arange(hi - lo), np.diff(rowptr))
    send = np.zeros(G, dtype=np.int64)
    recv = np.zeros(G, dtype=np.int64)
    for q in range(G):
        if q == int(np.searchsorted(bounds, lo, side="right") - 1):
            continue
        m = owner == q
        send[q] = np.unique(rows[m]).size
        recv[q] = np.unique(col[m]).size
    return send, recv


def check_plans(send, recv, group=None):
    """All ranks agree on the halo sizes: what r sends to q is what q receives from r."""
    import torch.distributed as dist

    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    obj = [None] * world
    dist.all_gather_object(obj, (list(map(int, send)), list(map(int, recv))), group=group)
    for q in range(world):
        if q != rank and obj[q][0][rank] != int(recv[q]):
            return False
    return True


def broadcast_unique_id(group=None, make=None):
    """Rank 0 creates the 128-byte NCCL id (via liblf unless `make` is given) and every rank
    receives it over the torch process group (any backend)."""
    import torch
    import torch.distributed as dist

    rank = dist.get_rank(group)
    t = torch.zeros(128, dtype=torch.uint8)
    if rank == 0:
        raw = make() if make is not None else _nccl_id()
        t[:] = torch.frombuffer(bytearray(raw), dtype=torch.uint8)
    if dist.get_backend(group) == "nccl":
        t = t.cuda()
    dist.broadcast(t, src=0, group=group)
    return bytes(t.cpu().numpy().tobytes())


def _nccl_id():
    L = _lf.load()
    buf = C.create_string_buffer(128)
    _lf._check(L.lf_comm_nccl_unique_id(buf))
    return buf.raw


class Comm:
    """Exchange backend handle: Comm.nccl(rank, world, id128) or Comm.loopback(G)."""

    def __init__(self, handle, kind):
        self.h = handle
        self.kind = kind

    @classmethod
    def nccl(cls, rank, world, id128):
        L = _lf.load()
        h = C.c_void_p()
        _lf._check(L.lf_comm_create_nccl(C.create_string_buffer(id128, 128), world, rank, C.byref(h)))
        return cls(h, "nccl")

    @classmethod
    def loopback(cls, G):
        L = _lf.load()
        h = C.c_void_p()
        _lf._check(L.lf_comm_create_loopback(G, C.byref(h)))
        return cls(h, "loopback")

    def close(self):
        if self.h:
            _lf.load().lf_comm_destroy(self.h)
            self.h = None


class Partition:
    """One rank's rows [bounds[rank], bounds[rank+1]) on the current device."""

    def __init__(self, rowptr, col, val, bounds, rank, n=2):
        import torch

        self.keep = (rowptr, col, val)  # device tensors must outlive the handle
        self.bounds = np.ascontiguousarray(bounds, dtype=np.int64)
        self.G = len(bounds) - 1
        self.rank = rank
        self.n = n
        self.n_own = int(bounds[rank + 1] - bounds[rank])
        L = _lf.load()
        A = _lf.CSRDesc(self.n_own, col.numel(), rowptr.data_ptr(), col.data_ptr(), val.data_ptr())
        h = C.c_void_p()
        _lf._check(L.lf_part_create(self.G, self.bounds.ctypes.data_as(C.c_void_p), rank, C.byref(A), n,
                                    C.byref(h), _lf._stream()))
        self.h = h
        self.torch = torch

    def info(self):
        out = np.zeros(8, dtype=np.int64)
        _lf._check(_lf.load().lf_part_info(self.h, out.ctypes.data_as(C.c_void_p), 8))
        return dict(zip(("lo", "hi", "ghosts_below", "ghosts_above", "local", "halo_sent", "nnz", "G"),
                        (int(x) for x in out)))

    def export(self, M=5):
        t = self.torch
        dev = "cuda"
        out = dict(pi=t.empty((self.n_own, self.n), dtype=t.int32, device=dev),
                   pi_w=t.empty((self.n_own, self.n), dtype=t.float32, device=dev),
                   pi_val=t.empty((self.n_own, self.n), dtype=t.float32, device=dev),
                   diag=t.empty(self.n_own, dtype=t.float32, device=dev),
                   rounds=t.zeros(1, dtype=t.int32, device=dev),
                   live=t.zeros(2 * max(M, 1), dtype=t.int64, device=dev))
        p = _lf._ptr
        _lf._check(_lf.load().lf_part_export(self.h, p(out["pi"]), p(out["pi_w"]), p(out["pi_val"]),
                                             p(out["diag"]), p(out["rounds"]),
                                             p(out["live"]) if M > 0 else None, _lf._stream()))
        return out

    def forest_export(self):
        t = self.torch
        n = self.n_own
        out = dict(forest=t.empty((n, 2), dtype=t.int32, device="cuda"),
                   path_id=t.empty(n, dtype=t.int32, device="cuda"),
                   pos=t.empty(n, dtype=t.int32, device="cuda"),
                   iperm=t.empty(n, dtype=t.int32, device="cuda"),
                   n_cycles=t.zeros(1, dtype=t.int64, device="cuda"))
        p = _lf._ptr
        _lf._check(_lf.load().lf_part_forest_export(self.h, p(out["forest"]), p(out["path_id"]), p(out["pos"]),
                                                    p(out["iperm"]), p(out["n_cycles"]), _lf._stream()))
        return out

    def close(self):
        if self.h:
            _lf.load().lf_part_destroy(self.h, _lf._stream())
            self.h = None


def factor(parts, comm, *, M=5, m=5, k_m=0, p=0.5, seed=0):
    """lf_part_factor over the partitions of this process (1 for NCCL, all G for loopback)."""
    L = _lf.load()
    arr = (C.c_void_p * len(parts))(*[q.h for q in parts])
    o = _lf.opts(M, m, k_m, p, seed)
    _lf._check(L.lf_part_factor(arr, len(parts), comm.h, C.byref(o), _lf._stream()))


def linear_forest(parts, comm):
    """lf_part_linear_forest over the partitions of this process (after factor, n = 2)."""
    L = _lf.load()
    arr = (C.c_void_p * len(parts))(*[q.h for q in parts])
    _lf._check(L.lf_part_linear_forest(arr, len(parts), comm.h, _lf._stream()))


def tridiag(parts, comm):
    """lf_part_tridiag -> per partition (a, b, c) over its own vertices (row = iperm)."""
    import torch

    L = _lf.load()
    outs = [tuple(torch.empty(q.n_own, dtype=torch.float32, device="cuda") for _ in range(3)) for q in parts]
    arr = (C.c_void_p * len(parts))(*[q.h for q in parts])
    pa = (C.c_void_p * len(parts))(*[o[0].data_ptr() for o in outs])
    pb = (C.c_void_p * len(parts))(*[o[1].data_ptr() for o in outs])
    pc = (C.c_void_p * len(parts))(*[o[2].data_ptr() for o in outs])
    _lf._check(L.lf_part_tridiag(arr, len(parts), comm.h, pa, pb, pc, _lf._stream()))
    return outs
