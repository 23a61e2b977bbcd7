"""Per-kernel times of the hot path on the C5 recipe (n^3 27-pt, device generator) under
several environment settings (diagnostics for DESIGN.md §5 and §8; not a bench number).
usage: python scripts/probe_c5.py [n] 'ENV=a,ENV2=b' 'ENV=c' ..."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import lfgen.gpu  # noqa: E402
from paper_conf_icpp_0002s22_b200 import _build, lf  # noqa: E402

n = sys.argv[1] if len(sys.argv) > 1 else "512"   # an n (C5 recipe on n^3) or a config name
variants = sys.argv[2:] or [""]
_build.build()
lf.load()
lfgen.gpu.build()
if n.isdigit():
    n = int(n)
    rp, col, val = lfgen.gpu.grid27_rows(n, 0, n, seed=5)
else:
    A = lfgen.config(n)
    rp, col, val = (torch.from_numpy(x).cuda() for x in (A.rowptr, A.col, A.val))
if os.environ.get("LF_L2FETCH"):  # cudaLimitMaxL2FetchGranularity (0x05) experiment
    import ctypes
    import glob
    rt = ctypes.CDLL(sorted(glob.glob(os.path.join(os.path.dirname(torch.__file__), "..", "nvidia", "cuda_runtime", "lib", "libcudart.so*")))[0])
    torch.cuda.synchronize()
    print("setlimit", rt.cudaDeviceSetLimit(0x05, ctypes.c_size_t(int(os.environ["LF_L2FETCH"]))), file=sys.stderr)
    v = ctypes.c_size_t(0)
    rt.cudaDeviceGetLimit(ctypes.byref(v), 0x05)
    print("l2 fetch granularity", v.value, file=sys.stderr)
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
P = lf.Pipeline(rp, col, val)
ref = None
for var in variants:
    env = dict(kv.split("=", 1) for kv in var.split(",") if kv)
    old = {k: os.environ.get(k) for k in env}
    os.environ.update(env)
    P.run()
    torch.cuda.synchronize()
    if ref is None:
        ref = {k: P.lf[k].clone() for k in ("perm", "path_id", "pos", "a")}
    ks, tot = {}, []
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    for it in range(5):
        flush.zero_()
        lf.profile_enable(True)
        ev0.record()
        P.run()
        ev1.record()
        torch.cuda.synchronize()
        lf.profile_enable(False)
        tot.append(ev0.elapsed_time(ev1))
        for nm, ms in lf.profile_collect():
            ks.setdefault(nm, []).append(ms)
    same = all(torch.equal(P.lf[k], ref[k]) for k in ref)
    print(json.dumps({"n": n, "env": env, "step_ms": round(sorted(tot)[2], 3), "same_as_first": same,
                      "kernels": {k: round(sorted(v)[len(v) // 2], 4)
                                  for k, v in sorted(ks.items(), key=lambda x: -sum(x[1]))}}), flush=True)
    for k, v in old.items():
        if v is None:
            os.environ.pop(k)
        else:
            os.environ[k] = v
