"""Diagnostics: run the C2 pipeline a few times (for printf-instrumented builds)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import lfgen
from paper_conf_icpp_0002s22_b200 import lf

A = lfgen.config(sys.argv[1] if len(sys.argv) > 1 else "C2")
rp, col, val = (torch.from_numpy(x).cuda() for x in (A.rowptr, A.col, A.val))
P = lf.Pipeline(rp, col, val)
for i in range(4):
    P.run()
    torch.cuda.synchronize()
    print("run", i, flush=True)
