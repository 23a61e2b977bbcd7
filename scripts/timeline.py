"""Diagnostics: per-kernel [first CTA start, last CTA exit] of one uninstrumented C2 step
(graph replay, PDL on, L2 flushed before), from an LF_TIMELINE build (LF_LIB_PATH)."""
import ctypes as C
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import lfgen
from paper_conf_icpp_0002s22_b200 import lf

A = lfgen.config(sys.argv[1] if len(sys.argv) > 1 else "C2")
rp, col, val = (torch.from_numpy(x).cuda() for x in (A.rowptr, A.col, A.val))
P = lf.Pipeline(rp, col, val)
for _ in range(3):
    P.run()
torch.cuda.synchronize()
g = torch.cuda.CUDAGraph()
with torch.cuda.graph(g):
    P.run()
torch.cuda.synchronize()
L = lf.load()
L.lf_debug_timeline.argtypes = [C.c_void_p, C.c_int]
flush = torch.empty(512 * 1024 * 1024, dtype=torch.uint8, device="cuda")
names = {0: "propose_stream", 2: "propose_long", 4: "mutual0", 6: "rounds_fused",
         16: "lf_full1", 18: "red_full", 20: "lf_full2", 22: "tile_prefix", 24: "perm_tri"}
acc = {}
ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
for it in range(10):
    flush.zero_()
    torch.cuda.synchronize()
    assert L.lf_debug_timeline(None, 1) == 0
    ev0.record()
    g.replay()
    ev1.record()
    torch.cuda.synchronize()
    out = np.zeros(32, dtype=np.uint64)
    assert L.lf_debug_timeline(C.c_void_p(out.ctypes.data), 0) == 0
    t0 = min(int(out[i]) for i in names)
    for i, nm in names.items():
        if int(out[i + 1]) == 0:
            continue
        acc.setdefault(nm, []).append(((int(out[i]) - t0) / 1e3, (int(out[i + 1]) - t0) / 1e3))
    acc.setdefault("_event_ms", []).append((ev0.elapsed_time(ev1), 0))
for nm, v in acc.items():
    s = np.median(np.array(v), axis=0)
    print(f"{nm:16s} start {s[0]:8.1f} us  end {s[1]:8.1f} us  dur {s[1]-s[0]:7.1f}")
