"""Print BiCGStab iteration counts / FRE for Jacobi, TriScal, AlgTriScal on ANISO1/2
(§6, Fig. 4); see tests/test_gpu_bicgstab.py.  usage: python scripts/bicgstab_demo.py [nx]"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path[:0] = [ROOT, os.path.join(ROOT, "tests")]

import torch  # noqa: E402

import lfgen  # noqa: E402
from paper_conf_icpp_0002s22_b200 import _build, lf  # noqa: E402
from test_gpu_bicgstab import solve_all  # noqa: E402

_build.build()
lf.load()
nx = int(sys.argv[1]) if len(sys.argv) > 1 else 500
for kind in (1, 2):
    res = solve_all(torch, lf, lfgen.aniso2d(nx, kind))
    print(json.dumps({"matrix": f"ANISO{kind}", "nx": nx, "N": nx * nx, "tol": 1e-8,
                      **{k: {"iterations": it, "FRE": fre} for k, (it, fre) in res.items()}}))
