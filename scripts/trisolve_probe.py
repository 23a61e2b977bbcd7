"""Standalone lf_tri_solve launch on a C2-shaped dominant system (for ncu captures)."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_icpp_0002s22_b200 import lf  # noqa: E402

N = 1 << 21
rng = np.random.default_rng(0)
a = -rng.uniform(0.1, 1, N).astype(np.float32)
c = -rng.uniform(0.1, 1, N).astype(np.float32)
b = (np.abs(a) + np.abs(c) + rng.uniform(0.01, 0.5, N)).astype(np.float32)
cut = np.cumsum(rng.integers(1, 900, N // 200))
cut = cut[cut < N]
a[cut] = 0
c[cut - 1] = 0
t = [torch.from_numpy(v).cuda() for v in (a, b, c, rng.standard_normal(N).astype(np.float32))]
ws = lf.Workspace()
y = torch.empty(N, device="cuda")
for _ in range(3):
    lf.tri_solve(*t, ws=ws, out=y)
torch.cuda.synchronize()
