"""The C-ABI library builds, loads and exports every symbol include/lf.h declares.

CPU only: no call here reaches a CUDA API (argument checks fail before any launch).
"""
import ctypes as C
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def lib():
    from paper_conf_icpp_0002s22_b200 import _build, lf

    _build.build()
    return lf.load()


def _declared():
    src = open(os.path.join(ROOT, "include", "lf.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(lf_[a-z_]+)\s*\(", src)))


def test_exports_every_declared_symbol(lib):
    from paper_conf_icpp_0002s22_b200 import lf

    names = _declared()
    assert set(names) == set(lf.EXPORTS)
    for n in names:
        assert hasattr(lib, n), n


def test_version_and_defaults(lib):
    from paper_conf_icpp_0002s22_b200 import lf

    assert b"sm_100a" in lib.lf_version()
    o = lf.FactorOpts()
    lib.lf_factor_opts_default(C.byref(o))
    assert (o.M, o.m, o.k_m, o.p, o.seed, o.until_maximal) == (5, 5, 0, 0.5, 0, 0)


def test_workspace_size_grows_with_n(lib):
    s1 = lib.lf_factor_workspace_size(1000, 1)
    s4 = lib.lf_factor_workspace_size(1000, 4)
    assert 0 < s1 < s4
    assert lib.lf_factor_workspace_size(1000, 5) == 0


def test_invalid_arguments_rejected_before_launch(lib):
    from paper_conf_icpp_0002s22_b200 import lf

    A = lf.CSRDesc(10, 0, 1, None, None)
    o = lf.FactorOpts(5, 5, 0, 0.5, 0, 0)
    assert lib.lf_factor(C.byref(A), 5, C.byref(o), None, None, None, None, None, None, None, 0, None) == -1
    assert b"n must be" in lib.lf_last_error()
    assert lib.lf_factor(None, 2, None, None, None, None, None, None, None, None, 0, None) == -1
    A = lf.CSRDesc(2 ** 31, 0, 1, None, None)
    assert lib.lf_factor(C.byref(A), 2, None, 1, 1, None, None, None, None, None, 0, None) == -1
    o = lf.FactorOpts(5, 5, 7, 0.5, 0, 1)  # until_maximal with k_m >= m
    A = lf.CSRDesc(10, 0, 1, None, None)
    assert lib.lf_factor(C.byref(A), 2, C.byref(o), 1, 1, None, None, None, None, None, 0, None) == -1
    assert lib.lf_linear_forest(-1, None, None, None, None, None, None, None, None, None, 0, None) == -1
    assert lib.lf_tridiag(5, None, None, None, None, None, None, None, None, None) == -1
    # pair arrays read as 8-byte (int2 / float2) vectors must be 8-byte aligned
    bad, ok = C.c_void_p(0x1004), C.c_void_p(0x1000)
    assert lib.lf_linear_forest(4, bad, ok, ok, ok, ok, ok, ok, None, None, 0, None) == -1
    assert b"aligned" in lib.lf_last_error()
    assert lib.lf_tridiag(4, ok, ok, bad, ok, ok, ok, ok, ok, None) == -1
    assert b"aligned" in lib.lf_last_error()


def test_tri_solve_arguments_rejected_before_launch(lib):
    """lf_tri_solve's checks (include/lf.h): bad N, NULL, workspace size/alignment, y overlapping an input;
    N = 0 is a no-op.  None of these reaches the device."""
    from paper_conf_icpp_0002s22_b200 import lf

    L = lf.load()
    p = C.c_void_p(0x1000)
    nb = L.lf_tri_solve_workspace_size(1000)
    assert nb > 16 * 1000 and L.lf_tri_solve_workspace_size(0) == 0
    assert L.lf_tri_solve(-1, p, p, p, p, C.c_void_p(0x2000), p, nb, None) == -1
    assert L.lf_tri_solve(0, None, None, None, None, None, None, 0, None) == 0
    assert L.lf_tri_solve(1000, None, p, p, p, C.c_void_p(0x2000), p, nb, None) == -1
    assert b"NULL" in L.lf_last_error()
    assert L.lf_tri_solve(1000, p, p, p, p, C.c_void_p(0x2000), p, nb - 1, None) == -2
    assert L.lf_tri_solve(1000, p, p, p, p, C.c_void_p(0x2000), C.c_void_p(0x1010), nb, None) == -2
    assert L.lf_tri_solve(1000, p, p, p, C.c_void_p(0x3000), C.c_void_p(0x3000), p, nb, None) == -1
    assert b"overlaps" in L.lf_last_error()
    # partial overlaps (offset views) of y with x, a, b or c are rejected as well
    A, B, Cc, X = (C.c_void_p(0x10000 * k) for k in (1, 2, 3, 4))
    for y in (0x40000 + 4 * 999, 0x40000 - 4 * 999, 0x10000 + 8, 0x20000 - 4 * 999 + 4, 0x30000 + 3996):
        assert L.lf_tri_solve(1000, A, B, Cc, X, C.c_void_p(y), p, nb, None) == -1, hex(y)
        assert b"overlaps" in L.lf_last_error()


def test_product_package_does_not_import_oracle():
    pkg = os.path.join(ROOT, "paper_conf_icpp_0002s22_b200")
    for dp, _, fs in os.walk(pkg):
        for f in fs:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                txt = open(os.path.join(dp, f)).read()
                assert "import oracle" not in txt and "from oracle" not in txt, f
                assert "lf_oracle" not in txt, f


def test_validate_arguments_rejected_before_launch(lib):
    """lf_validate_csr needs lf_validate_workspace_size(n) bytes; lf_validate_factor checks
    N, n and NULL before any launch (include/lf.h)."""
    from paper_conf_icpp_0002s22_b200 import lf

    L = lf.load()
    assert L.lf_validate_workspace_size(1000) >= 1000 + 256
    A = lf.CSRDesc(1000, 5000, 0x1000, 0x2000, 0x3000)
    assert L.lf_validate_csr(C.byref(A), C.c_void_p(0x10000), 256, None) == -2
    assert b"workspace" in L.lf_last_error()
    assert L.lf_validate_factor(-1, 2, C.c_void_p(0x1000), C.c_void_p(0x10000), 256, None) == -1
    assert L.lf_validate_factor(10, 5, C.c_void_p(0x1000), C.c_void_p(0x10000), 256, None) == -1
    assert L.lf_validate_factor(10, 2, None, C.c_void_p(0x10000), 256, None) == -1
    assert L.lf_validate_factor(0, 2, None, None, 0, None) == 0
    assert L.lf_validate_factor(10, 2, C.c_void_p(0x1000), C.c_void_p(0x10000), 128, None) == -2


def test_general_input_calls_reject_bad_arguments(lib):
    from paper_conf_icpp_0002s22_b200 import lf

    A = lf.CSRDesc(10, 4, 1, 1, 1)
    assert lib.lf_symmetrize(C.byref(A), None, None, None, None, None, 0, None) == -1
    assert b"NULL" in lib.lf_last_error()
    big = lf.CSRDesc(10, 1 << 30, 1, 1, 1)
    assert lib.lf_symmetrize(C.byref(big), 1, 1, 1, 1, None, 0, None) == -1
    assert lib.lf_symmetrize_workspace_size(10, 1 << 30) == 0
    assert lib.lf_symmetrize_workspace_size(10, 100) > 0
    assert lib.lf_orig_coeffs(C.byref(A), 5, 1, 1, 1, None) == -1
    assert lib.lf_orig_coeffs(C.byref(A), 2, None, None, None, None) == -1
    ok = lf.CSRDesc(10, 4, 1, 1, 1)
    assert lib.lf_symmetrize(C.byref(ok), 1, 1, 1, 1, None, 0, None) == -2  # no workspace
