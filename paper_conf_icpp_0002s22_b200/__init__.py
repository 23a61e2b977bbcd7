"""B200-native linear forest extraction (Klein & Strzodka, ICPP'22) -- product package.

The hot path lives in liblf.so (csrc/, C ABI in include/lf.h); `lf` is its thin
ctypes binding.  This package never imports oracle/ (test infrastructure only).
"""
from . import lf  # noqa: F401
from .lf import (  # noqa: F401
    LFError,
    Pipeline,
    factor,
    linear_forest,
    pipeline_host,
    tridiag,
    validate,
)

__all__ = ["lf", "factor", "linear_forest", "tridiag", "pipeline_host", "validate", "Pipeline",
           "LFError"]
