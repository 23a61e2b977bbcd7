"""Device-side input generator (liblfgen_gpu.so, lfgen/csrc/lfgen_gpu.cu): the C5 27-point
graph written straight into HBM, slab by slab.  Input generation only (no method
arithmetic); equal to lfgen.grid3d_27pt_rows row for row (tests/test_gpu_c5.py)."""
from __future__ import annotations

import ctypes as C
import os
import subprocess

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "csrc", "lfgen_gpu.cu")
LIB = os.path.join(HERE, "liblfgen_gpu.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
_lib = None


def build(force=False):
    """nvcc -shared for sm_100a, in-tree."""
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < os.path.getmtime(SRC):
        tmp = LIB + f".tmp{os.getpid()}"
        subprocess.check_call([NVCC, "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo",
                               "-std=c++17", "-shared", "-Xcompiler", "-fPIC", "-o", tmp, SRC])
        os.replace(tmp, LIB)
    return LIB


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(LIB):
            raise RuntimeError(f"{LIB} not built (lfgen.gpu.build())")
        L = C.CDLL(LIB)
        L.lfg_grid27_nnz.argtypes = [C.c_int64] * 4
        L.lfg_grid27_nnz.restype = C.c_int64
        L.lfg_grid27_rows.argtypes = [C.c_int64, C.c_int64, C.c_int64, C.c_int64, C.c_uint64,
                                      C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p]
        L.lfg_grid27_rows.restype = C.c_int
        _lib = L
    return _lib


def grid27_rows(n, z_lo, z_hi, seed=5, nz=None, device="cuda", out=None):
    """(rowptr, col, val) torch CUDA tensors of the planes [z_lo, z_hi) of the n x n x nz
    27-point graph (rowptr rebased to 0, global column ids) -- lfgen.grid3d_27pt_rows."""
    import torch

    nz = n if nz is None else nz
    L = lib()
    rows = (z_hi - z_lo) * n * n
    Z = int(L.lfg_grid27_nnz(n, nz, z_lo, z_hi))
    if out is None:
        out = (torch.empty(rows + 1, dtype=torch.int64, device=device),
               torch.empty(Z, dtype=torch.int32, device=device),
               torch.empty(Z, dtype=torch.float32, device=device))
    rp, col, val = out
    rc = L.lfg_grid27_rows(n, nz, z_lo, z_hi, seed, C.c_void_p(rp.data_ptr()), C.c_void_p(col.data_ptr()),
                           C.c_void_p(val.data_ptr()), C.c_void_p(torch.cuda.current_stream().cuda_stream))
    if rc != 0:
        raise RuntimeError(f"lfg_grid27_rows failed ({rc})")
    return rp, col, val
