#!/usr/bin/env python
"""Golden digests of the CPU oracle on C5 (BASELINE.json configs[4]: the 512^3 27-point
graph, 134M vertices, 3.6e9 stored entries > 2^31) -- test infrastructure.

The GPU box cannot be assumed to hold the ~45 GB the single-threaded oracle needs at this
size, and it would take it several minutes, so this script (which calls ONLY lfgen/ and
oracle/) runs the oracle once here and stores sha256 digests of every output, plus a few
thousand sampled values for diagnosis, in tests/golden/c5_<n>_n2.json.  The GPU test
(tests/test_gpu_c5.py) regenerates the graph on the device, runs the CUDA path and compares
digests -- bit-exact parity at full size.  No value here comes from the
CUDA path.

    python scripts/make_c5_goldens.py            # n = 512 (~45 GB RAM, ~30 min)
    python scripts/make_c5_goldens.py --n 48     # small replica (the CPU test checks that
                                                 # the script agrees with the plain oracle)
"""
from __future__ import annotations

import argparse
import hashlib
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import lfgen  # noqa: E402
import oracle  # noqa: E402

CHUNK = 1 << 28  # bytes hashed per update


def sha(a: np.ndarray) -> str:
    h = hashlib.sha256()
    b = np.ascontiguousarray(a).reshape(-1).view(np.uint8)
    for i in range(0, b.shape[0], CHUNK):
        h.update(memoryview(b[i:i + CHUNK]))
    return h.hexdigest()


def sample_idx(N, k, seed):
    rng = np.random.default_rng(seed)
    return np.unique(np.concatenate([np.arange(min(N, 64)), np.arange(max(0, N - 64), N),
                                     rng.integers(0, N, size=k)])).astype(np.int64)


def goldens(n: int, seed: int = 5, log=print) -> dict:
    t0 = time.time()
    A = lfgen.grid3d_27pt_big(n, seed)
    N, Z = A.N, A.nnz
    log(f"generated n={n}: N={N} Z={Z} in {time.time() - t0:.0f}s")
    out = {"config": "C5" if n == 512 else f"C5-recipe {n}^3", "n": n, "seed": seed, "N": N, "nnz": Z,
           "E": A.n_edges, "deg": 2, "M": 5, "m": 5, "k_m": 0, "p": 0.5, "charge_seed": 0,
           "generator": "lfgen.grid3d_27pt_big", "oracle": "oracle/lf_oracle.c"}
    out["sha256"] = {"rowptr": sha(A.rowptr), "col": sha(A.col), "val": sha(A.val)}
    log(f"hashed CSR {time.time() - t0:.0f}s")
    pi, pw, rounds, lr, ln = oracle.factor(A, 2, counters=True)
    log(f"oracle factor {time.time() - t0:.0f}s rounds={rounds}")
    out["rounds"] = rounds
    out["live_rows"] = [int(x) for x in lr]
    out["live_nnz"] = [int(x) for x in ln]
    out["sha256"].update(pi=sha(pi), pi_w=sha(pw))
    lf = oracle.linear_forest(pi, pw)
    log(f"oracle linear forest {time.time() - t0:.0f}s cycles={lf['n_cycles']}")
    out["n_cycles"] = lf["n_cycles"]
    for k in ("forest", "path_id", "pos", "perm", "iperm"):
        out["sha256"][k] = sha(lf[k])
    a, b, c = oracle.tridiag(A, lf["forest"], lf["perm"])
    log(f"oracle tridiag {time.time() - t0:.0f}s")
    out["sha256"].update(a=sha(a), b=sha(b), c=sha(c))
    ip = lf["iperm"]
    # owner order (row iperm[v] of Q^T A Q listed at vertex v): what lf_part_tridiag returns
    out["sha256"].update(a_owner=sha(a[ip]), b_owner=sha(b[ip]), c_owner=sha(c[ip]))
    idx = sample_idx(N, 4000, 17)
    out["sample_idx"] = idx.tolist()
    out["sample"] = {
        "pi": pi[idx].tolist(), "pi_w_bits": pw[idx].view(np.uint32).tolist(),
        "forest": lf["forest"][idx].tolist(), "path_id": lf["path_id"][idx].tolist(),
        "pos": lf["pos"][idx].tolist(), "perm": lf["perm"][idx].tolist(), "iperm": ip[idx].tolist(),
        "a_bits": a[idx].view(np.uint32).tolist(), "b_bits": b[idx].view(np.uint32).tolist(),
        "c_bits": c[idx].view(np.uint32).tolist(),
    }
    out["oracle_seconds"] = round(time.time() - t0, 1)
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=512)
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    oracle.build()
    g = goldens(args.n, log=lambda s: print(s, flush=True))
    path = args.out or os.path.join(ROOT, "tests", "golden", f"c5_{args.n}_n2.json")
    os.makedirs(os.path.dirname(path), exist_ok=True)
    with open(path, "w") as f:
        json.dump(g, f)
    print("wrote", path)


if __name__ == "__main__":
    main()
