"""Diagnostics: cached vs uncached factor rounds on C2, repeated; prints mismatches."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import lfgen
from paper_conf_icpp_0002s22_b200 import lf

A = lfgen.config(sys.argv[1] if len(sys.argv) > 1 else "C2")
rp, col, val = (torch.from_numpy(x).cuda() for x in (A.rowptr, A.col, A.val))
ws = lf.Workspace()
os.environ["LF_NO_CACHED_ROUNDS"] = "1"
ref = lf.factor(rp, col, val, 2, live=True, ws=ws)
torch.cuda.synchronize()
ref = {k: (v.clone() if v is not None else None) for k, v in ref.items()}
print("ref live", ref["live"].tolist(), flush=True)
del os.environ["LF_NO_CACHED_ROUNDS"]
for i in range(6):
    out = lf.factor(rp, col, val, 2, live=True, ws=ws)
    torch.cuda.synchronize()
    bad = (out["pi"] != ref["pi"]).any(dim=1).nonzero().flatten()
    print(i, "live", out["live"].tolist(), "bad rows", bad.numel(), bad[:10].tolist(), flush=True)
    if bad.numel():
        r = bad[0].item()
        print("   row", r, "got", out["pi"][r].tolist(), "want", ref["pi"][r].tolist(), flush=True)
for i in range(3):  # back to back without sync
    for _ in range(4):
        out = lf.factor(rp, col, val, 2, live=True, ws=ws)
    torch.cuda.synchronize()
    bad = (out["pi"] != ref["pi"]).any(dim=1).nonzero().flatten()
    print("b2b", i, "live", out["live"].tolist(), "bad rows", bad.numel(), flush=True)
