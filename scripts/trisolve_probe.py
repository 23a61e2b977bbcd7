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

if len(sys.argv) > 1 and sys.argv[1] == "--time":
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ts = []
    for _ in range(30):
        flush.zero_()
        e0.record()
        lf.tri_solve(*t, ws=ws, out=y)
        e1.record()
        e1.synchronize()
        ts.append(e0.elapsed_time(e1))
    ts.sort()
    print(f"{os.environ.get('LF_LIB_PATH', 'default')}: median {ts[len(ts) // 2] * 1e3:.1f} us, min {ts[0] * 1e3:.1f} us")
