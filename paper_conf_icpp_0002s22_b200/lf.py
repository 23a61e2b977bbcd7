"""Thin Python binding of liblf.so (include/lf.h): argument marshalling only.

Every step of the path runs in the library's CUDA kernels.  torch tensors serve only as
device memory; the current torch CUDA stream is passed through.  There is no CPU
fallback: if liblf.so is missing or no CUDA device is present, calls raise.
"""
from __future__ import annotations

import ctypes as C
import os
from dataclasses import dataclass

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("LF_LIB_PATH", os.path.join(HERE, "liblf.so"))

LF_OK = 0
ERRORS = {-1: "LF_EINVAL", -2: "LF_ENOMEM", -3: "LF_ECUDA", -4: "LF_ENCCL", -5: "LF_EINPUT"}

# every symbol include/lf.h declares (checked by tests/test_abi.py)
EXPORTS = (
    "lf_factor_opts_default", "lf_factor_workspace_size", "lf_factor",
    "lf_linear_forest_workspace_size", "lf_linear_forest", "lf_tridiag", "lf_linear_forest_tridiag",
    "lf_pipeline_workspace_size", "lf_pipeline_host", "lf_validate_csr", "lf_validate_workspace_size",
    "lf_validate_factor",
    "lf_last_error", "lf_version", "lf_profile_enable", "lf_profile_collect",
    "lf_forest_stats", "lf_comm_nccl_unique_id", "lf_comm_create_nccl", "lf_comm_create_loopback",
    "lf_comm_destroy", "lf_part_create", "lf_part_destroy", "lf_part_info", "lf_part_factor",
    "lf_part_export", "lf_part_linear_forest", "lf_part_forest_export", "lf_part_tridiag",
    "lf_tri_solve_workspace_size", "lf_tri_solve",
    "lf_symmetrize_workspace_size", "lf_symmetrize", "lf_orig_coeffs",
    "lf_coarsen_workspace_size", "lf_coarsen", "lf_block_tridiag",
)


class LFError(RuntimeError):
    pass


class CSRDesc(C.Structure):
    _fields_ = [("n", C.c_int64), ("nnz", C.c_int64), ("rowptr", C.c_void_p),
                ("col", C.c_void_p), ("val", C.c_void_p)]


class FactorOpts(C.Structure):
    _fields_ = [("M", C.c_int32), ("m", C.c_int32), ("k_m", C.c_int32), ("p", C.c_float),
                ("seed", C.c_uint32), ("until_maximal", C.c_int32)]


_lib = None


def load(path: str = LIB_PATH):
    """Load liblf.so (raises if it has not been built)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(path):
        raise LFError(f"{path} not built: run `python -c 'import __graft_entry__ as g; g.build()'`")
    L = C.CDLL(path)
    P, I64, I32 = C.c_void_p, C.c_int64, C.c_int
    L.lf_factor_opts_default.argtypes = [P]
    L.lf_factor_workspace_size.argtypes = [I64, I32]
    L.lf_factor_workspace_size.restype = C.c_size_t
    L.lf_factor.argtypes = [P, I32, P, P, P, P, P, P, P, P, C.c_size_t, P]
    L.lf_linear_forest_workspace_size.argtypes = [I64]
    L.lf_linear_forest_workspace_size.restype = C.c_size_t
    L.lf_linear_forest.argtypes = [I64, P, P, P, P, P, P, P, P, P, C.c_size_t, P]
    L.lf_tridiag.argtypes = [I64, P, P, P, P, P, P, P, P, P]
    L.lf_linear_forest_tridiag.argtypes = [I64, P, P, P, P, P, P, P, P, P, P, P, P, P, P, C.c_size_t, P]
    L.lf_pipeline_workspace_size.argtypes = [I64, I64]
    L.lf_pipeline_workspace_size.restype = C.c_size_t
    L.lf_pipeline_host.argtypes = [P, P, P, P, P, P, P, P, P, C.c_size_t, P]
    L.lf_validate_csr.argtypes = [P, P, C.c_size_t, P]
    L.lf_validate_workspace_size.argtypes = [I64]
    L.lf_validate_workspace_size.restype = C.c_size_t
    L.lf_validate_factor.argtypes = [I64, I32, P, P, C.c_size_t, P]
    L.lf_validate_factor.restype = C.c_int
    L.lf_forest_stats.argtypes = [I64, P, C.c_size_t, P, I32]
    L.lf_comm_nccl_unique_id.argtypes = [P]
    L.lf_comm_create_nccl.argtypes = [P, I32, I32, P]
    L.lf_comm_create_loopback.argtypes = [I32, P]
    L.lf_comm_destroy.argtypes = [P]
    L.lf_part_create.argtypes = [I32, P, I32, P, I32, P, P]
    L.lf_part_destroy.argtypes = [P, P]
    L.lf_part_info.argtypes = [P, P, I32]
    L.lf_part_factor.argtypes = [P, I32, P, P, P]
    L.lf_part_export.argtypes = [P, P, P, P, P, P, P, P]
    L.lf_part_linear_forest.argtypes = [P, I32, P, P]
    L.lf_part_forest_export.argtypes = [P, P, P, P, P, P, P]
    L.lf_part_tridiag.argtypes = [P, I32, P, P, P, P, P]
    L.lf_tri_solve_workspace_size.argtypes = [I64]
    L.lf_tri_solve_workspace_size.restype = C.c_size_t
    L.lf_tri_solve.argtypes = [I64, P, P, P, P, P, P, C.c_size_t, P]
    L.lf_tri_solve.restype = C.c_int
    L.lf_symmetrize_workspace_size.argtypes = [I64, I64]
    L.lf_symmetrize_workspace_size.restype = C.c_size_t
    L.lf_symmetrize.argtypes = [P, P, P, P, P, P, C.c_size_t, P]
    L.lf_symmetrize.restype = C.c_int
    L.lf_orig_coeffs.argtypes = [P, I32, P, P, P, P]
    L.lf_orig_coeffs.restype = C.c_int
    L.lf_coarsen_workspace_size.argtypes = [I64, I64]
    L.lf_coarsen_workspace_size.restype = C.c_size_t
    L.lf_coarsen.argtypes = [P, P, P, P, P, P, P, P, P, C.c_size_t, P]
    L.lf_coarsen.restype = C.c_int
    L.lf_block_tridiag.argtypes = [P, I64, P, P, P, P, P, P, P, P]
    L.lf_block_tridiag.restype = C.c_int
    L.lf_profile_enable.argtypes = [I32]
    L.lf_profile_collect.argtypes = [P, I32, P, I32]
    L.lf_last_error.restype = C.c_char_p
    L.lf_version.restype = C.c_char_p
    for name in ("lf_factor", "lf_linear_forest", "lf_tridiag", "lf_pipeline_host", "lf_validate_csr",
                 "lf_factor_opts_default"):
        getattr(L, name).restype = C.c_int if name != "lf_factor_opts_default" else None
    _lib = L
    return L


def _check(rc):
    if rc != LF_OK:
        msg = load().lf_last_error().decode()
        raise LFError(f"{ERRORS.get(rc, rc)}: {msg}")


def _torch():
    import torch

    if not torch.cuda.is_available():
        raise LFError("liblf needs a CUDA device (no CPU fallback)")
    return torch


def _ptr(t):
    return None if t is None else C.c_void_p(t.data_ptr())


def _stream():
    torch = _torch()
    return C.c_void_p(torch.cuda.current_stream().cuda_stream)


def _csr_desc(rowptr, col, val):
    N = rowptr.numel() - 1
    return CSRDesc(N, col.numel(), rowptr.data_ptr(), col.data_ptr(), val.data_ptr())


def opts(M=5, m=5, k_m=0, p=0.5, seed=0, until_maximal=False) -> FactorOpts:
    return FactorOpts(M, m, k_m, p, seed, 1 if until_maximal else 0)


class Workspace:
    """Grow-only device scratch buffer (torch uint8 tensor)."""

    def __init__(self):
        self.buf = None

    def get(self, nbytes: int):
        torch = _torch()
        if self.buf is None or self.buf.numel() < nbytes:
            self.buf = torch.empty(max(nbytes, 256), dtype=torch.uint8, device="cuda")
        return self.buf


_ws = Workspace()


def factor(rowptr, col, val, n=2, *, M=5, m=5, k_m=0, p=0.5, seed=0, until_maximal=False,
           want_val=True, want_diag=True, live=False, ws=None, out=None):
    """lf_factor on device CSR tensors -> dict(pi[N,n], pi_w, pi_val, diag, rounds, live)."""
    torch = _torch()
    L = load()
    N = rowptr.numel() - 1
    dev = rowptr.device
    if out is None:
        out = dict(
            pi=torch.empty((N, n), dtype=torch.int32, device=dev),
            pi_w=torch.empty((N, n), dtype=torch.float32, device=dev),
            pi_val=torch.empty((N, n), dtype=torch.float32, device=dev) if want_val else None,
            diag=torch.empty(N, dtype=torch.float32, device=dev) if want_diag else None,
            rounds=torch.zeros(1, dtype=torch.int32, device=dev),
            live=torch.zeros(2 * max(M, 1), dtype=torch.int64, device=dev) if live else None,
        )
    A = _csr_desc(rowptr, col, val)
    o = opts(M, m, k_m, p, seed, until_maximal)
    nb = L.lf_factor_workspace_size(N, n)
    buf = (ws or _ws).get(nb)
    _check(L.lf_factor(C.byref(A), n, C.byref(o), _ptr(out["pi"]), _ptr(out["pi_w"]),
                       _ptr(out["pi_val"]), _ptr(out["diag"]), _ptr(out["rounds"]),
                       _ptr(out["live"]), _ptr(buf), nb, _stream()))
    return out


def linear_forest(pi2, pi2_w, *, ws=None, out=None, n_cycles=True):
    """lf_linear_forest -> dict(forest[N,2], path_id, pos, perm, iperm, n_cycles)."""
    torch = _torch()
    L = load()
    N = pi2.shape[0]
    dev = pi2.device
    if out is None:
        out = dict(
            forest=torch.empty((N, 2), dtype=torch.int32, device=dev),
            path_id=torch.empty(N, dtype=torch.int32, device=dev),
            pos=torch.empty(N, dtype=torch.int32, device=dev),
            perm=torch.empty(N, dtype=torch.int32, device=dev),
            iperm=torch.empty(N, dtype=torch.int32, device=dev),
            n_cycles=torch.zeros(1, dtype=torch.int64, device=dev) if n_cycles else None,
        )
    nb = L.lf_linear_forest_workspace_size(N)
    buf = (ws or _ws).get(nb)
    _check(L.lf_linear_forest(N, _ptr(pi2), _ptr(pi2_w), _ptr(out["forest"]), _ptr(out["path_id"]),
                              _ptr(out["pos"]), _ptr(out["perm"]), _ptr(out["iperm"]),
                              _ptr(out["n_cycles"]), _ptr(buf), nb, _stream()))
    return out


def tridiag(forest, iperm, pi2, pi2_val, diag, *, out=None):
    """lf_tridiag -> (a, b, c) device float32 [N]."""
    torch = _torch()
    L = load()
    N = forest.shape[0]
    if out is None:
        out = tuple(torch.empty(N, dtype=torch.float32, device=forest.device) for _ in range(3))
    a, b, c = out
    _check(L.lf_tridiag(N, _ptr(forest), _ptr(iperm), _ptr(pi2), _ptr(pi2_val), _ptr(diag),
                        _ptr(a), _ptr(b), _ptr(c), _stream()))
    return a, b, c


def linear_forest_tridiag(pi2, pi2_w, pi2_val, diag, *, ws=None, out=None, n_cycles=True):
    """lf_linear_forest_tridiag -> dict(forest, path_id, pos, perm, iperm, a, b, c, n_cycles)."""
    torch = _torch()
    L = load()
    N = pi2.shape[0]
    dev = pi2.device
    if out is None:
        out = dict(
            forest=torch.empty((N, 2), dtype=torch.int32, device=dev),
            path_id=torch.empty(N, dtype=torch.int32, device=dev),
            pos=torch.empty(N, dtype=torch.int32, device=dev),
            perm=torch.empty(N, dtype=torch.int32, device=dev),
            iperm=torch.empty(N, dtype=torch.int32, device=dev),
            a=torch.empty(N, dtype=torch.float32, device=dev),
            b=torch.empty(N, dtype=torch.float32, device=dev),
            c=torch.empty(N, dtype=torch.float32, device=dev),
            n_cycles=torch.zeros(1, dtype=torch.int64, device=dev) if n_cycles else None,
        )
    nb = L.lf_linear_forest_workspace_size(N)
    buf = (ws or _ws).get(nb)
    _check(L.lf_linear_forest_tridiag(N, _ptr(pi2), _ptr(pi2_w), _ptr(pi2_val), _ptr(diag),
                                      _ptr(out["forest"]), _ptr(out["path_id"]), _ptr(out["pos"]),
                                      _ptr(out["perm"]), _ptr(out["iperm"]), _ptr(out["a"]),
                                      _ptr(out["b"]), _ptr(out["c"]), _ptr(out["n_cycles"]), _ptr(buf),
                                      nb, _stream()))
    return out


def _check_csr(name, rowptr, col, val):
    """raw pointers cross the ABI: dtype, device, contiguity and lengths are checked here"""
    torch = _torch()
    for nm, t, dt in (("rowptr", rowptr, torch.int64), ("col", col, torch.int32), ("val", val, torch.float32)):
        if not (t.is_cuda and t.dtype == dt and t.is_contiguous() and t.dim() == 1):
            raise LFError(f"{name}: {nm} must be a contiguous 1-D {dt} CUDA tensor")
    if col.numel() != val.numel():
        raise LFError(f"{name}: col and val lengths differ")


def _check_i32(name, nm, t, numel):
    torch = _torch()
    if not (t.is_cuda and t.dtype == torch.int32 and t.is_contiguous() and t.numel() == numel):
        raise LFError(f"{name}: {nm} must be a contiguous int32 CUDA tensor of {numel} elements")


def symmetrize(rowptr, col, val, *, ws=None):
    """lf_symmetrize: S = A' + A'^T of a (possibly non-symmetric) device CSR -> (rowptr, col,
    val) of S, trimmed to its stored entries (one device-to-host read of the count)."""
    torch = _torch()
    L = load()
    _check_csr("symmetrize", rowptr, col, val)
    N = rowptr.numel() - 1
    nnz = col.numel()
    dev = rowptr.device
    s_rp = torch.empty(N + 1, dtype=torch.int64, device=dev)
    s_col = torch.empty(max(2 * nnz, 1), dtype=torch.int32, device=dev)
    s_val = torch.empty(max(2 * nnz, 1), dtype=torch.float32, device=dev)
    s_nnz = torch.zeros(1, dtype=torch.int64, device=dev)
    A = _csr_desc(rowptr, col, val)
    nb = L.lf_symmetrize_workspace_size(N, nnz)
    if nnz and not nb:
        raise LFError("symmetrize: nnz must be < 2^30")
    buf = (ws or _ws).get(nb)
    _check(L.lf_symmetrize(C.byref(A), _ptr(s_rp), _ptr(s_col), _ptr(s_val), _ptr(s_nnz), _ptr(buf), nb,
                           _stream()))
    m = int(s_nnz.item())
    return s_rp, s_col[:m], s_val[:m]


def orig_coeffs(rowptr, col, val, pi, *, out=None):
    """lf_orig_coeffs: (pi_val [N, n], diag [N]) of the ORIGINAL A on the factor slots pi."""
    torch = _torch()
    L = load()
    _check_csr("orig_coeffs", rowptr, col, val)
    N, n = pi.shape
    if rowptr.numel() != N + 1:
        raise LFError("orig_coeffs: pi must have one row per vertex of A")
    _check_i32("orig_coeffs", "pi", pi, N * n)
    if out is None:
        out = (torch.empty((N, n), dtype=torch.float32, device=pi.device),
               torch.empty(N, dtype=torch.float32, device=pi.device))
    A = _csr_desc(rowptr, col, val)
    _check(L.lf_orig_coeffs(C.byref(A), n, _ptr(pi), _ptr(out[0]), _ptr(out[1]), _stream()))
    return out


def general_pipeline(rowptr, col, val, *, M=5, m=5, k_m=0, p=0.5, seed=0, ws=None):
    """The hot path on a general (non-symmetric) A: the [0,2]-factor and
    the linear forest of S = A' + A'^T, the tridiagonal coefficients from A itself."""
    S = symmetrize(rowptr, col, val, ws=ws)
    fac = factor(*S, 2, M=M, m=m, k_m=k_m, p=p, seed=seed, want_val=False, want_diag=False, ws=ws)
    pi_val, diag = orig_coeffs(rowptr, col, val, fac["pi"])
    fac["pi_val"], fac["diag"] = pi_val, diag
    lf = linear_forest_tridiag(fac["pi"], fac["pi_w"], pi_val, diag, ws=ws)
    return S, fac, lf


def coarsen(rowptr, col, val, mu, *, ws=None):
    """lf_coarsen: the coarse graph of the matched pairs of mu ([N] or [N,1]) ->
    (cid [N], members [Nc, 2], (c_rowptr, c_col, c_val)) trimmed (one host read of Nc, nnz)."""
    torch = _torch()
    L = load()
    _check_csr("coarsen", rowptr, col, val)
    N = rowptr.numel() - 1
    nnz = col.numel()
    _check_i32("coarsen", "mu", mu, N)
    dev = rowptr.device
    cid = torch.empty(max(N, 1), dtype=torch.int32, device=dev)
    members = torch.empty((max(N, 1), 2), dtype=torch.int32, device=dev)
    c_rp = torch.empty(N + 1, dtype=torch.int64, device=dev)
    c_col = torch.empty(max(nnz, 1), dtype=torch.int32, device=dev)
    c_val = torch.empty(max(nnz, 1), dtype=torch.float32, device=dev)
    info = torch.zeros(2, dtype=torch.int64, device=dev)
    A = _csr_desc(rowptr, col, val)
    nb = L.lf_coarsen_workspace_size(N, nnz)
    buf = (ws or _ws).get(nb)
    _check(L.lf_coarsen(C.byref(A), _ptr(mu.contiguous()), _ptr(cid), _ptr(members), _ptr(c_rp), _ptr(c_col),
                        _ptr(c_val), _ptr(info), _ptr(buf), nb, _stream()))
    nc, mc = (int(x) for x in info.tolist())
    return cid[:N], members[:nc], (c_rp[:nc + 1], c_col[:mc], c_val[:mc])


def block_tridiag(rowptr, col, val, members, cforest, cperm):
    """lf_block_tridiag -> (D, L, U) [Nc, 4] row-major 2x2 blocks, fperm [Nc, 2] (-1 ghost)."""
    torch = _torch()
    Lb = load()
    _check_csr("block_tridiag", rowptr, col, val)
    nc = members.shape[0]
    _check_i32("block_tridiag", "members", members, 2 * nc)
    _check_i32("block_tridiag", "cforest", cforest, 2 * nc)
    _check_i32("block_tridiag", "cperm", cperm, nc)
    dev = members.device
    D, Lo, U = (torch.empty((max(nc, 1), 4), dtype=torch.float32, device=dev) for _ in range(3))
    fperm = torch.empty((max(nc, 1), 2), dtype=torch.int32, device=dev)
    A = _csr_desc(rowptr, col, val)
    _check(Lb.lf_block_tridiag(C.byref(A), nc, _ptr(members.contiguous()), _ptr(cforest.contiguous()),
                               _ptr(cperm.contiguous()), _ptr(D), _ptr(Lo), _ptr(U), _ptr(fperm), _stream()))
    return D[:nc], Lo[:nc], U[:nc], fperm[:nc]


def block_pipeline(rowptr, col, val, *, M=5, m=5, k_m=0, p=0.5, seed=0, ws=None):
    """AlgTriBlockPrecond (§6): [0,1]-factor, coarse graph of the matched pairs,
    [0,2]-factor + linear forest on it, the 2x2 block tridiagonal system."""
    mu = factor(rowptr, col, val, 1, M=M, m=m, k_m=k_m, p=p, seed=seed, want_val=False, want_diag=False, ws=ws)["pi"]
    cid, members, Cg = coarsen(rowptr, col, val, mu, ws=ws)
    cf = factor(*Cg, 2, M=M, m=m, k_m=k_m, p=p, seed=seed, want_val=False, want_diag=False, ws=ws)
    clf = linear_forest(cf["pi"], cf["pi_w"], ws=ws)
    D, Lo, U, fperm = block_tridiag(rowptr, col, val, members, clf["forest"], clf["perm"])
    return dict(mu=mu, cid=cid, members=members, coarse=Cg, cpi=cf["pi"], cforest=clf["forest"],
                cperm=clf["perm"], D=D, L=Lo, U=U, fperm=fperm)


@dataclass
class Pipeline:
    """Preallocated device buffers for the whole hot path on one graph (n=2)."""

    rowptr: object
    col: object
    val: object
    M: int = 5
    m: int = 5
    k_m: int = 0
    p: float = 0.5
    seed: int = 0

    def __post_init__(self):
        torch = _torch()
        N = self.rowptr.numel() - 1
        self.N = N
        self.ws_f = Workspace()
        self.ws_l = Workspace()
        self.fac = None
        self.lf = None
        self.tri = None

    def run_factor(self):
        self.fac = factor(self.rowptr, self.col, self.val, 2, M=self.M, m=self.m, k_m=self.k_m,
                          p=self.p, seed=self.seed, ws=self.ws_f, out=self.fac, live=True)
        return self.fac

    def run_forest(self):
        """Linear forest + tridiagonal copy (one fused call)."""
        self.lf = linear_forest_tridiag(self.fac["pi"], self.fac["pi_w"], self.fac["pi_val"],
                                        self.fac["diag"], ws=self.ws_l, out=self.lf)
        self.tri = (self.lf["a"], self.lf["b"], self.lf["c"])
        return self.lf

    def run(self):
        self.run_factor()
        self.run_forest()
        return self


def tri_solve(a, b, c, x, *, ws=None, out=None):
    """y = T^{-1} x for the tridiagonal (a, b, c) of lf_tridiag (include/lf.h lf_tri_solve)."""
    torch = _torch()
    L = load()
    N = b.numel()
    y = out if out is not None else torch.empty(N, dtype=torch.float32, device=b.device)
    for nm, t in (("a", a), ("b", b), ("c", c), ("x", x), ("out", y)):
        # raw pointers cross the ABI: a wrong dtype, stride or length would read out of bounds
        if not (t.is_cuda and t.dtype == torch.float32 and t.is_contiguous() and t.numel() == N):
            raise LFError(f"tri_solve: {nm} must be a contiguous float32 CUDA tensor of {N} elements")
    nb = L.lf_tri_solve_workspace_size(N)
    w = (ws or Workspace()).get(nb) if N > 0 else None
    _check(L.lf_tri_solve(N, _ptr(a), _ptr(b), _ptr(c), _ptr(x), _ptr(y), _ptr(w), nb, _stream()))
    return y


def pipeline_host(rowptr_h, col_h, val_h, *, M=5, m=5, k_m=0, p=0.5, seed=0, ws=None, outs=None):
    """lf_pipeline_host with HOST (pinned) torch CPU tensors -> (perm, path_id, pos, a, b, c)."""
    torch = _torch()
    L = load()
    N = rowptr_h.numel() - 1
    if outs is None:
        mk = lambda dt: torch.empty(N, dtype=dt, pin_memory=True)  # noqa: E731
        outs = (mk(torch.int32), mk(torch.int32), mk(torch.int32), mk(torch.float32),
                mk(torch.float32), mk(torch.float32))
    A = _csr_desc(rowptr_h, col_h, val_h)
    o = opts(M, m, k_m, p, seed)
    nb = L.lf_pipeline_workspace_size(N, col_h.numel())
    buf = (ws or _ws).get(nb)
    _check(L.lf_pipeline_host(C.byref(A), C.byref(o), *[_ptr(t) for t in outs], _ptr(buf), nb,
                              _stream()))
    return outs


def validate(rowptr, col, val, ws=None):
    """lf_validate_csr: raises LFError (LF_EINPUT) on a CSR that violates lf_factor's
    preconditions (include/lf.h)."""
    L = load()
    A = _csr_desc(rowptr, col, val)
    nb = L.lf_validate_workspace_size(rowptr.numel() - 1)
    buf = (ws or _ws).get(nb)
    _check(L.lf_validate_csr(C.byref(A), _ptr(buf), nb, _stream()))


def validate_factor(pi, ws=None):
    """lf_validate_factor on a device pi[N, n] (canonical [0,n]-factor form)."""
    L = load()
    N, n = pi.shape
    buf = (ws or _ws).get(256)
    _check(L.lf_validate_factor(N, n, _ptr(pi), _ptr(buf), 256, _stream()))


def profile_enable(on: bool = True):
    load().lf_profile_enable(1 if on else 0)


def profile_collect(cap: int = 4096):
    """-> list of (kernel name, ms) for the launches recorded since profile_enable(True)."""
    L = load()
    stride = 40
    names = C.create_string_buffer(stride * cap)
    ms = (C.c_float * cap)()
    n = L.lf_profile_collect(names, stride, ms, cap)
    out = []
    for i in range(n):
        nm = names.raw[i * stride:(i + 1) * stride].split(b"\0", 1)[0].decode()
        out.append((nm, float(ms[i])))
    return out


FOREST_STATS = ("boundary_cycle_pass", "boundary_rank_pass", "reduced_steps_cycle",
                "reduced_steps_rank", "splitters_cycle_pass", "unvisited", "fallback_tiles",
                "splitters_rank_pass", "max_node_scan_steps", "malformed_input",
                "splitter_free_cycles", "longest_splitter_free_cycle")


def forest_stats(N, ws):
    """Diagnostics of the last linear_forest run that used workspace `ws` (a Workspace)."""
    import numpy as np

    L = load()
    out = np.zeros(32, dtype=np.int32)
    _check(L.lf_forest_stats(N, _ptr(ws.buf), ws.buf.numel(), C.c_void_p(out.ctypes.data), 32))
    d = dict(zip(FOREST_STATS, (int(x) for x in out[:len(FOREST_STATS)])))
    if out[16:].any():  # LF_PHASE_TIMING build: per-phase kcycles summed over tiles
        d["phase_kcycles"] = [int(x) for x in out[16:24]]
        d["redscan_small_us_cum"] = [int(x) for x in out[24:28]]
    return d
