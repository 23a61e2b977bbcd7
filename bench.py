#!/usr/bin/env python
"""Benchmark of the hot path: [0,2]-factor (M=5) + linear forest + permutation + tridiag.

Contract: `python bench.py --gpus N --steps K --warmup W` prints ONE JSON
line on rank 0.  A step is one pass of the whole hot path over one synthetic graph resident
in HBM; `value` is whole-job Medges/s (undirected edges E / step time).  Device time with
CUDA events per step, L2 flushed between steps, max over ranks.

* N = 1: the headline is C5 (BASELINE.json configs[4], the 512^3 27-point graph, 134M
  vertices, 1.74e9 edges, 3.6e9 stored entries) on one B200 -- the largest configuration
  and the one the metric is quoted on.  C2 (n = 1..4, the paper's Fig. 3 sweep), C3 and C4
  are measured in the same run and reported under "configs".
* N > 1: C5 strong scaling -- rank r owns the z-slab [512 r / N, 512 (r+1) / N), generated
  on its own GPU, and runs the row-partitioned path (NCCL halo exchange, boundary-end list).
* `--impl reference` times the CPU oracle (the reference arm of this tier) on a bounded
  sample of the same workload.
"""
from __future__ import annotations

import argparse
import json
import os
import platform
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "ms and Medges/s per [0,2]-factor+linear forest at 1/2/4/8 B200; % HBM peak"
NOMINAL_GBS = 8000.0  # north_star's "~8 TB/s" (SURVEY.md §8(d) headline denominator)
CONFIG_DESC = {
    "C1": "2D 5-pt 64x64 (4,096 vertices), n=2",
    "C2": "3D 7-pt anisotropic 128^3 (2.1M vertices, 6.24M edges), n=2",
    "C3": "FEM-like jittered 27-pt 100^3 bricks (1M vertices), n=2",
    "C4": "Chung-Lu power-law 5M vertices, n=2",
    "C5": "3D 27-pt 512^3 (134M vertices, 1.74B edges, 3.61e9 stored entries), n=2",
}
C5_N = 512
SAMPLE_N = 96  # the CPU oracle's bounded sample of C5: the same 27-pt recipe on 96^3


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="C5")
    ap.add_argument("--extra", default="C2,C2n1,C2n3,C2n4,C3,C4,G3,B3",
                    help="other configs measured in the same run ('' for none)")
    ap.add_argument("--no-graph", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--cpu-runs", type=int, default=3)
    ap.add_argument("--force-multi", action="store_true",
                    help="use the row-partitioned multi-GPU path even at one rank (testing)")
    ap.add_argument("--grid", type=int, default=C5_N,
                    help="N > 1 / --force-multi: the C5 recipe on grid^3 (512 = C5; smaller for tests)")
    return ap.parse_args()


def dist_env():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md)"


def cpu_info():
    model = platform.processor() or ""
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                model = line.split(":", 1)[1].strip()
                break
    except OSError:
        pass
    return {"os_cpu_count": os.cpu_count(), "cpu_model": model}


class Clocks:
    """nvidia-smi clock/throttle sampler running during the timed region."""

    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index):
        self.gpu = gpu_index
        self.proc = None
        self.path = f"/tmp/lf_clocks_{os.getpid()}.csv"

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", f"--id={self.gpu}", f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits",
                 "-lms", "100"], stdout=open(self.path, "w"), stderr=subprocess.DEVNULL)
        except Exception:
            self.proc = None

    def n_samples(self):
        try:
            return sum(1 for _ in open(self.path))
        except OSError:
            return 0

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in open(self.path):
            f = [x.strip() for x in line.split(",")]
            if len(f) < 9:
                continue
            try:
                sm.append(float(f[1]))
                mx = float(f[2])
            except ValueError:
                continue
            for nm, val in zip(names, f[5:9]):
                if val.lower().startswith("active"):
                    reasons.add(nm)
        sm.sort()
        med = sm[len(sm) // 2] if sm else None
        return {"sm_mhz": med, "sm_max_mhz": mx, "reasons": sorted(reasons), "samples": len(sm)}


# ---------------------------------------------------------------------------
# byte model
# ---------------------------------------------------------------------------

def survey_bytes(N, n, live_rows, live_nnz, with_lf=True):
    """B_factor = sum_k [8 Z_a(k) + (16 + 16n) N_a(k) + 2N], B_LF = 40N,
    B_tri = 36N (the live counters come from the device and equal the oracle's)."""
    bf = sum(8 * z + (16 + 16 * n) * r + 2 * N for r, z in zip(live_rows, live_nnz))
    blf = 40 * N if with_lf else 0
    btri = 36 * N if with_lf else 0
    return {"B_factor": int(bf), "B_LF": int(blf), "B_main": int(bf + blf), "B_tri": int(btri),
            "B_alg": int(bf + blf + btri)}


def kernel_bytes(name, N, Z, n, live_rows, live_nnz, rows_ran=False):
    """Algorithmic HBM bytes of one launch: what the method must move.
    Rounds 1..M-1 run in ONE of two kernels (rows_ran: the rows mode did, the cached mode
    only raised its bail flag); their bytes go to that one."""
    base = name.split("[")[0]
    k = int(name.split("[")[1].rstrip("]")) if "[" in name else -1
    if base == "rows_propose":  # rounds 1..M-1 as per-round kernels (large graphs)
        base = "propose"
    if base == "rows_mutual":
        base = "mutual"
    if base == "propose":
        if k == 0:  # whole CSR + rowptr; write prop (j, value) and the diagonal
            return 8 * Z + 8 * (N + 1) + 8 * n * N + 4 * N
        Na, Za = live_rows[k], live_nnz[k]
        # live rows' CSR payload + rowptr pair + worklist + state + pi; write prop
        return 8 * Za + 16 * Na + 4 * Na + Na + 4 * n * Na + 8 * n * Na
    if base == "mutual":
        if k == 0:  # read prop (j, value); write pi, pi_w, pi_val, state, worklist
            return 8 * n * N + 12 * n * N + N + 4 * live_rows[1 if len(live_rows) > 1 else 0]
        Na = live_rows[k]
        nxt = live_rows[k + 1] if k + 1 < len(live_rows) else 0
        return 4 * Na + 8 * n * Na + 8 * n * Na + Na + 4 * nxt
    if base in ("rounds_fused", "rounds_rows"):  # rounds 1..M-1: live rows' propose + mutual traffic
        if (base == "rounds_rows") != rows_ran:
            return 0
        return sum(kernel_bytes(f"propose[{kk}]", N, Z, n, live_rows, live_nnz)
                   + kernel_bytes(f"mutual[{kk}]", N, Z, n, live_rows, live_nnz)
                   for kk in range(1, len(live_rows)))
    # linear forest: B_LF = 40N attributed to the kernel that moves it;
    # block-local intermediates and boundary records are implementation traffic
    if base == "lf_tile":
        return 16 * N  # read pi2 + pi2_w
    if base == "lf_expand":
        return 16 * N  # write forest, path_id, pos
    if base == "red_scan":
        return 0
    if base == "lf_local1":
        return 16 * N
    if base == "lf_local2":
        return 8 * N
    if base == "lf_local3":
        return 8 * N
    if base == "perm":
        return 8 * N
    if base == "perm_tridiag":  # write perm, iperm; read forest, pi2, pi2_val, diag; write a, b, c
        return 8 * N + 8 * N + 8 * N + 8 * N + 4 * N + 12 * N
    # global ruling set: the pack reads the factor, the emit pass writes every
    # output (and reads signed values and diag for a, b, c); walks and the reduced scan are
    # implementation traffic
    if base == "grs_pack":
        return 16 * N
    if base == "grs_emit_tri":  # write forest, path_id, pos, iperm; read signed values + diag
        return 8 * N + 12 * N + 12 * N
    if base == "grs_emit":
        return 8 * N + 12 * N
    if base == "grs_split_tri":  # write perm, a, b, c
        return 16 * N
    if base == "grs_split":
        return 4 * N
    if base == "tridiag":
        return 8 * N + 4 * N + 8 * N + 8 * N + 4 * N + 12 * N
    return 0


def ncu_profile(cfg):
    """Per-launch dram bytes / warp instructions of the step's kernels from the committed
    ncu capture of this config (profiles/traffic_<cfg>.json)."""
    p = os.path.join(ROOT, "profiles", f"traffic_{cfg}.json")
    try:
        return json.load(open(p))
    except (OSError, ValueError):
        return {}


# ---------------------------------------------------------------------------
# graphs
# ---------------------------------------------------------------------------

def make_graph(torch, name):
    """Device CSR of a BASELINE config (C5 generated on the GPU slab by slab; the others
    with numpy on the host and uploaded).  Input generation is outside every timed region."""
    import lfgen

    if name == "C5":
        import lfgen.gpu

        lfgen.gpu.build()
        rp, col, val = lfgen.gpu.grid27_rows(C5_N, 0, C5_N, seed=5)
        torch.cuda.synchronize()
        N, Z = rp.numel() - 1, col.numel()
        return {"name": name, "N": N, "Z": Z, "E": (Z - N) // 2, "rp": rp, "col": col, "val": val}
    A = lfgen.config(name)
    return {"name": name, "N": A.N, "Z": A.nnz, "E": A.n_edges, "rp": torch.from_numpy(A.rowptr).cuda(),
            "col": torch.from_numpy(A.col).cuda(), "val": torch.from_numpy(A.val).cuda()}


def measure_general(torch, lf, name, steps, warmup, flush):
    """SURVEY.md §8(f) f3 on a general input: G<k> = lfgen.nonsymmetric(C<k>); a step is
    lf_symmetrize + lf_factor(S) + lf_orig_coeffs + lf_linear_forest_tridiag (one host read
    of nnz(S) inside, to size S).  Medges/s over the undirected edges of S."""
    import lfgen

    A = lfgen.nonsymmetric(lfgen.config("C" + name[1:]), seed=7)
    rp, col, val = (torch.from_numpy(x).cuda() for x in (A.rowptr, A.col, A.val))
    ws = lf.Workspace()
    S, _, _ = lf.general_pipeline(rp, col, val, ws=ws)
    E = S[1].numel() // 2
    stream = torch.cuda.current_stream()
    for _ in range(warmup):
        lf.general_pipeline(rp, col, val, ws=ws)
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ts = []
    for _ in range(steps):
        flush.zero_()
        torch.cuda.synchronize()
        ev0.record(stream)
        lf.general_pipeline(rp, col, val, ws=ws)
        ev1.record(stream)
        ev1.synchronize()
        ts.append(ev0.elapsed_time(ev1))
    t = sorted(ts)[len(ts) // 2]
    return {"name": name, "N": A.N, "Z": int(A.rowptr[-1]), "E_S": int(E), "n": 2,
            "scope": "symmetrize + factor(S) + original coefficients + linear forest + perm + tridiag",
            "input": f"lfgen.nonsymmetric(C{name[1:]}, seed=7): 15% of the directed entries dropped, "
                     "2% explicit zeros, a_ij != a_ji",
            "ms_per_step": round(t, 4), "Medges_per_s": round(E / (t * 1e-3) / 1e6, 1)}


def measure_block(torch, lf, name, steps, warmup, flush):
    """SURVEY.md §8(f) f1 AlgTriBlockPrecond on C<k>: a step is the [0,1]-factor, lf_coarsen,
    the [0,2]-factor + linear forest of the coarse graph and lf_block_tridiag (two host reads
    inside: the coarse sizes).  Medges/s over the fine graph's edges."""
    import lfgen

    A = lfgen.config("C" + name[1:])
    rp, col, val = (torch.from_numpy(x).cuda() for x in (A.rowptr, A.col, A.val))
    ws = lf.Workspace()
    g = lf.block_pipeline(rp, col, val, ws=ws)
    nc = int(g["members"].shape[0])
    stream = torch.cuda.current_stream()
    for _ in range(warmup):
        lf.block_pipeline(rp, col, val, ws=ws)
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ts = []
    for _ in range(steps):
        flush.zero_()
        torch.cuda.synchronize()
        ev0.record(stream)
        lf.block_pipeline(rp, col, val, ws=ws)
        ev1.record(stream)
        ev1.synchronize()
        ts.append(ev0.elapsed_time(ev1))
    t = sorted(ts)[len(ts) // 2]
    return {"name": name, "N": A.N, "E": A.n_edges, "coarse_N": nc,
            "scope": "[0,1]-factor + coarse graph + coarse [0,2]-factor + coarse linear forest + 2x2 blocks",
            "ms_per_step": round(t, 4), "Medges_per_s": round(A.n_edges / (t * 1e-3) / 1e6, 1)}


# ---------------------------------------------------------------------------
# one config, one GPU
# ---------------------------------------------------------------------------

def measure(torch, lf, g, n, steps, warmup, flush, use_graph=True):
    """Times the hot path on one device graph: n = 2 -> lf_factor + lf_linear_forest_tridiag
    (the step); other n -> the [0,n]-factor alone (Fig. 3's sweep).  Returns the record."""
    stream = torch.cuda.current_stream()
    if n == 2:
        P = lf.Pipeline(g["rp"], g["col"], g["val"])
        run = P.run
    else:
        box = {}

        def run():
            box["fac"] = lf.factor(g["rp"], g["col"], g["val"], n, live=True, want_val=False, want_diag=False,
                                   out=box.get("fac"), ws=box.setdefault("ws", lf.Workspace()))
    for _ in range(max(warmup, 3)):
        run()
    torch.cuda.synchronize()

    def capture(prof):
        lf.profile_enable(prof)
        gr = torch.cuda.CUDAGraph()
        with torch.cuda.graph(gr):
            run()
        torch.cuda.synchronize()
        gr.replay()
        torch.cuda.synchronize()
        lf.profile_enable(False)
        return gr

    graph = graph_prof = None
    if use_graph:
        try:
            s = torch.cuda.Stream()
            s.wait_stream(stream)
            with torch.cuda.stream(s):
                run()
            torch.cuda.synchronize()
            graph = capture(False)
            graph_prof = capture(True)
        except Exception as e:  # capture unsupported -> eager launches
            print(f"# graph capture failed ({e}); timing eager launches", file=sys.stderr)
            graph = graph_prof = None

    def step(prof=False):
        if graph is not None:
            (graph_prof if prof else graph).replay()
        else:
            lf.profile_enable(prof)
            run()
            lf.profile_enable(False)

    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    step_ms, kern, launches = [], {}, None
    for _ in range(steps):
        flush.zero_()  # > L2 (126 MB) written between steps
        ev0.record(stream)
        step()
        ev1.record(stream)
        ev1.synchronize()
        step_ms.append(ev0.elapsed_time(ev1))
    for _ in range(min(steps, 10)):
        flush.zero_()
        step(prof=True)
        torch.cuda.synchronize()
        recs = lf.profile_collect()
        # one record per profiled group; groups of several kernels: perm (k_tile_prefix +
        # k_perm_tri), grs_pack (pack, k_tile_prefix, list), grs_walk (walk, meet), grs_len
        # (len, cyccand, cycfind, lenscan, k_tile_prefix); every lf_linear_forest call starts
        # with the (unrecorded) control-block kernel k_ctl_zero
        mult = {"perm": 2, "perm_tridiag": 2, "grs_pack": 3, "grs_walk": 2, "grs_len": 5}
        launches = sum(mult.get(nm, 1) for nm, _ in recs) + (1 if n == 2 else 0)
        for nm, ms in recs:
            kern.setdefault(nm, []).append(ms)
    t = sorted(step_ms)[len(step_ms) // 2]
    fac = P.fac if n == 2 else box["fac"]
    live = fac["live"].cpu().numpy()
    M = 5
    lr, ln = [int(x) for x in live[:M]], [int(x) for x in live[M:2 * M]]
    kavg = {nm: sum(v) / len(v) for nm, v in kern.items()}
    N, Z, E = g["N"], g["Z"], g["E"]
    rec = {"name": g["name"] + ("" if n == 2 else f"n{n}"), "N": N, "E": E, "nnz": Z, "n": n,
           "scope": "factor+linear forest+perm+tridiag" if n == 2 else f"[0,{n}]-factor only",
           "ms_per_step": round(t, 4), "ms_mean": round(sum(step_ms) / len(step_ms), 4),
           "Medges_per_s": round(E / (t * 1e-3) / 1e6, 1), "live_rows": lr, "live_nnz": ln,
           "kernels_ms": {k: round(v, 5) for k, v in sorted(kavg.items(), key=lambda x: -x[1])},
           "graph": graph is not None, "launches": launches}
    sb = survey_bytes(N, n, lr, ln, with_lf=(n == 2))
    peak, _ = load_peaks()
    rec["bytes"] = sb
    Bs = sb["B_alg"]
    rec["frac_of_peak"] = round(Bs / (t * 1e-3) / 1e9 / peak, 4)
    rec["frac_of_nominal_8TBs"] = round(Bs / (t * 1e-3) / 1e9 / NOMINAL_GBS, 4)
    rec["_kavg"] = kavg
    rec["_pipeline"] = P if n == 2 else None
    return rec


def roofline(rec, cfg, sm_mhz, sm_count):
    kavg = rec["_kavg"]
    if not kavg:
        return None
    dom = max(kavg, key=kavg.get)
    N, Z, n = rec["N"], rec["nnz"], rec["n"]
    rows_ran = kavg.get("rounds_rows", 0.0) > 2 * kavg.get("rounds_fused", 0.0)
    b = kernel_bytes(dom, N, Z, n, rec["live_rows"], rec["live_nnz"], rows_ran)
    peak, kind = load_peaks()
    ach = b / (kavg[dom] * 1e-3) / 1e9
    prof = ncu_profile(cfg)
    out = {"kernel": dom, "bound": "hbm", "achieved": round(ach, 1), "peak": peak, "peak_kind": kind,
           "unit": "GB/s", "frac": round(ach / peak, 4),
           "traffic": prof.get("bytes_per_launch", {}).get(dom),
           "alg_bytes_per_launch": int(b), "ms_per_launch": round(kavg[dom], 5),
           "traffic_source": prof.get("source")}
    inst = prof.get("warp_inst_per_launch", {}).get(dom)
    if inst and sm_mhz:
        a2 = inst / (kavg[dom] * 1e-3) / 1e9
        p2 = 4 * sm_count * sm_mhz * 1e6 / 1e9
        out["issue_view"] = {"bound": "issue", "achieved": round(a2, 1), "peak": round(p2, 1),
                             "unit": "G warp-inst/s", "frac": round(a2 / p2, 4), "warp_inst_per_launch": inst}
    return out


def cpu_sample(n_grid=SAMPLE_N):
    import lfgen

    return lfgen.grid3d_27pt_big(n_grid, seed=5, planes_per_chunk=16)


def cpu_baseline(A, runs, cfg):
    import oracle

    oracle.build()
    t0 = time.perf_counter()
    for _ in range(runs):
        oracle.run_pipeline(A)
    dt = (time.perf_counter() - t0) / runs
    what = (f"the C5 recipe (27-pt, seed 5) on {SAMPLE_N}^3 (N={A.N}, E={A.n_edges}) as a bounded sample of"
            f" the 512^3 graph" if cfg == "C5" else f"full {A.name} graph (N={A.N}, E={A.n_edges})")
    return {"value": round(A.n_edges / dt / 1e6, 3), "unit": "Medges/s", "cores": 1, "kind": "oracle",
            "ms_per_graph": round(dt * 1e3, 1),
            "sample": f"{what}, oracle pipeline (Alg. 2 M=5 + walks + sort + tridiag) x{runs}, single thread",
            **cpu_info()}


def run_reference(args):
    ws, rank, _ = dist_env()
    if rank != 0:
        return
    import lfgen
    import oracle

    oracle.build()
    A = cpu_sample() if args.config == "C5" else lfgen.config(args.config)
    for _ in range(args.warmup):
        oracle.run_pipeline(A)
    ts = []
    for _ in range(args.steps):
        t0 = time.perf_counter()
        oracle.run_pipeline(A)
        ts.append(time.perf_counter() - t0)
    ms = 1e3 * sum(ts) / len(ts)
    val = A.n_edges / (ms / 1e3) / 1e6
    sample = (f"the C5 recipe (27-pt, seed 5) on {SAMPLE_N}^3 (N={A.N}, E={A.n_edges}) per step, a bounded "
              f"sample of the 512^3 graph, single thread" if args.config == "C5"
              else f"full {A.name} graph per step, single thread")
    out = {
        "impl": "reference", "metric": METRIC, "value": round(val, 3), "unit": "Medges/s",
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms, 3),
        "higher_is_better": True, "scaling": "strong" if args.config == "C5" else "weak",
        "vs_baseline": None, "dtype": "f32", "data": "synthetic",
        "config": {"workload": CONFIG_DESC.get(args.config, args.config), "name": args.config,
                   "n": 2, "M": 5, "m": 5, "k_m": 0, "sample_N": A.N, "sample_E": A.n_edges},
        "cpu_baseline": {"value": round(val, 3), "unit": "Medges/s", "cores": 1, "kind": "oracle",
                         "sample": sample, **cpu_info()},
        "e2e": {"value": round(val, 3), "unit": "Medges/s", "h2d_bytes_per_step": 0,
                "d2h_bytes_per_step": 0},
    }
    emit_line(out)


# ---------------------------------------------------------------------------
# N > 1: C5 strong scaling over z-slabs
# ---------------------------------------------------------------------------

def run_multi(args, ws, rank, local):
    """C5 row-partitioned over `ws` ranks: rank r generates and owns the z-planes
    [512 r / ws, 512 (r+1) / ws) and runs the partitioned factor (NCCL halo exchange), the
    boundary-end-list linear forest and the tridiagonal extraction."""
    import torch
    import torch.distributed as tdist

    import lfgen.gpu
    from paper_conf_icpp_0002s22_b200 import _build, dist, lf

    torch.cuda.set_device(local)
    tdist.init_process_group("nccl", device_id=torch.device("cuda", local))
    _build.build()
    lf.load()
    lfgen.gpu.build()
    n = args.grid
    bounds = dist.slab_bounds(n, n * n, ws)
    z0, z1 = int(bounds[rank]) // (n * n), int(bounds[rank + 1]) // (n * n)
    rpd, cold, vald = lfgen.gpu.grid27_rows(n, z0, z1, seed=5)
    torch.cuda.synchronize()
    N = n ** 3
    Z = int(lfgen.gpu.lib().lfg_grid27_nnz(n, n, 0, n))
    E = (Z - N) // 2
    uid = dist.broadcast_unique_id()
    comm = dist.Comm.nccl(rank, ws, uid)
    part = dist.Partition(rpd, cold, vald, bounds, rank, n=2)
    stream = torch.cuda.current_stream()
    flush = torch.empty(512 * 1024 * 1024, dtype=torch.uint8, device="cuda")

    def step():
        dist.factor([part], comm)
        dist.linear_forest([part], comm)
        dist.tridiag([part], comm)

    clocks = Clocks(local)
    clocks.start()
    for _ in range(max(args.warmup, 3)):
        step()
    torch.cuda.synchronize()
    t_end = time.time() + 5.0
    while clocks.n_samples() < 3 and time.time() < t_end:
        step()
        torch.cuda.synchronize()
    tdist.barrier()
    torch.cuda.synchronize()
    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    step_ms = []
    for _ in range(args.steps):
        flush.zero_()
        torch.cuda.synchronize()
        tdist.barrier()
        ev0.record(stream)
        step()
        ev1.record(stream)
        ev1.synchronize()
        step_ms.append(ev0.elapsed_time(ev1))
    torch.cuda.synchronize()
    tdist.barrier()
    kern = {}
    for _ in range(min(args.steps, 3)):
        flush.zero_()
        lf.profile_enable(True)
        step()
        lf.profile_enable(False)
        torch.cuda.synchronize()
        for nm, ms in lf.profile_collect():
            kern.setdefault(nm, []).append(ms)
    clk = clocks.stop()
    t = torch.tensor([sorted(step_ms)[len(step_ms) // 2]], dtype=torch.float64, device="cuda")
    tdist.all_reduce(t, op=tdist.ReduceOp.MAX)
    t_step = float(t.item())
    e2e = None
    if not args.no_e2e:
        # own slab from pinned host memory, partition setup, the three stages, results back
        rp_h, col_h, val_h = (x.cpu().pin_memory() for x in (rpd, cold, vald))
        n_own = int(bounds[rank + 1] - bounds[rank])
        outs_h = [torch.empty(n_own, dtype=dt, pin_memory=True) for dt in (torch.int32, torch.int32, torch.int32,
                                                                            torch.float32, torch.float32, torch.float32)]
        e2e_ms = []
        for _ in range(max(2, min(args.steps, 3))):
            torch.cuda.synchronize()
            tdist.barrier()
            ev0.record(stream)
            d = [x.cuda(non_blocking=True) for x in (rp_h, col_h, val_h)]
            p2 = dist.Partition(d[0], d[1], d[2], bounds, rank, n=2)
            dist.factor([p2], comm)
            dist.linear_forest([p2], comm)
            a, b, c = dist.tridiag([p2], comm)[0]
            fe = p2.forest_export()
            for dst, src in zip(outs_h, (fe["iperm"], fe["path_id"], fe["pos"], a, b, c)):
                dst.copy_(src, non_blocking=True)
            ev1.record(stream)
            ev1.synchronize()
            e2e_ms.append(ev0.elapsed_time(ev1))
            p2.close()
            del d
        te = torch.tensor([sum(e2e_ms) / len(e2e_ms)], dtype=torch.float64, device="cuda")
        tdist.all_reduce(te, op=tdist.ReduceOp.MAX)
        e2e = {"value": round(E / (float(te.item()) * 1e-3) / 1e6, 2), "unit": "Medges/s",
               "ms_per_step": round(float(te.item()), 3),
               "h2d_bytes_per_step": int(8 * (N + ws) + 8 * Z), "d2h_bytes_per_step": int(24 * N),
               "includes": "H2D of every rank's slab, partition setup (ghost relabeling, halo plan), the three "
                           "stages, D2H of iperm/path_id/pos/a/b/c"}
    info = part.info()
    if rank == 0:
        kavg = {nm: sum(v) / len(v) for nm, v in kern.items()}
        dom = max(kavg, key=kavg.get) if kavg else None
        peak, peak_kind = load_peaks()
        out = {
            "metric": METRIC,
            "value": round(E / (t_step * 1e-3) / 1e6, 2),
            "unit": "Medges/s",
            "n_gpus": ws,
            "steps": args.steps,
            "warmup": args.warmup,
            "ms_per_step": round(t_step, 4),
            "higher_is_better": True,
            "scaling": "strong",
            "vs_baseline": None,
            "dtype": "f32",
            "data": "synthetic",
            "config": {
                "workload": (CONFIG_DESC["C5"] if n == C5_N else f"C5 recipe (27-pt, seed 5) on {n}^3")
                + f", z-slabs of {n // ws} planes per rank",
                "name": "C5" if n == C5_N else f"C5-{n}", "N": N, "E": E, "nnz": Z, "n": 2, "M": 5, "m": 5, "k_m": 0,
                "parallelism": f"row-partitioned z-slabs x{ws}, NCCL halo exchange + boundary-end list",
                "halo_entries_per_exchange_rank0": info["halo_sent"],
                "l2": "flushed between steps (512 MB write)", "graph": False,
            },
            "kernels_ms_rank0": {k: round(v, 5) for k, v in sorted(kavg.items(), key=lambda x: -x[1])},
            "roofline": {"kernel": dom, "bound": "hbm", "achieved": None, "peak": peak,
                         "peak_kind": peak_kind, "unit": "GB/s", "frac": None, "traffic": None,
                         "ms_per_launch": round(kavg[dom], 5) if dom else None},
            "gpu_launches": sum(len(v) for v in kern.values()) // max(1, min(args.steps, 3)),
            "clocks": clk,
        }
        if e2e:
            out["e2e"] = e2e
        emit_line(out)
    part.close()
    comm.close()
    tdist.destroy_process_group()


# ---------------------------------------------------------------------------
# N = 1
# ---------------------------------------------------------------------------

def e2e_single(torch, lf, g, steps):
    """The same metric through lf_pipeline_host with HOST buffers: H2D of the CSR, the three
    stages, D2H of perm/path_id/pos/a/b/c, all inside the timed region."""
    try:
        hs = [x.cpu().pin_memory() for x in (g["rp"], g["col"], g["val"])]
        pinned = True
    except RuntimeError:
        hs = [x.cpu() for x in (g["rp"], g["col"], g["val"])]
        pinned = False
    ws = lf.Workspace()
    outs = lf.pipeline_host(*hs, ws=ws)
    stream = torch.cuda.current_stream()
    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    ms = []
    for _ in range(steps):
        ev0.record(stream)
        outs = lf.pipeline_host(*hs, ws=ws, outs=outs)
        ev1.record(stream)
        ev1.synchronize()
        ms.append(ev0.elapsed_time(ev1))
    del ws, outs, hs
    torch.cuda.empty_cache()
    t = sorted(ms)[len(ms) // 2]
    N, Z = g["N"], g["Z"]
    return {"value": round(g["E"] / (t * 1e-3) / 1e6, 2), "unit": "Medges/s", "ms_per_step": round(t, 3),
            "h2d_bytes_per_step": int(8 * (N + 1) + 8 * Z), "d2h_bytes_per_step": int(24 * N),
            "host_buffers": "pinned" if pinned else "pageable"}


_STDOUT_FD = None


def emit_line(obj):
    """The one JSON line on the real stdout (native libraries' banners -- e.g. NCCL's version
    line -- were sent to stderr by quiet_native_stdout)."""
    line = (json.dumps(obj) + "\n").encode()
    if _STDOUT_FD is not None:
        os.write(_STDOUT_FD, line)
    else:
        sys.stdout.write(line.decode())
        sys.stdout.flush()


def quiet_native_stdout():
    global _STDOUT_FD
    sys.stdout.flush()
    _STDOUT_FD = os.dup(1)
    os.dup2(2, 1)


def main():
    quiet_native_stdout()
    args = parse()
    if args.impl == "reference":
        run_reference(args)
        return
    ws_env, _, _ = dist_env()
    if ws_env > 1 or args.force_multi:
        if ws_env == 1:
            os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
            os.environ.setdefault("MASTER_PORT", "29533")
            os.environ.setdefault("RANK", "0")
            os.environ.setdefault("WORLD_SIZE", "1")
            os.environ.setdefault("LOCAL_RANK", "0")
        run_multi(args, *dist_env())
        return
    import torch

    from paper_conf_icpp_0002s22_b200 import _build, lf

    torch.cuda.set_device(0)
    _build.build()
    lf.load()
    sm_count = torch.cuda.get_device_properties(0).multi_processor_count
    flush = torch.empty(512 * 1024 * 1024, dtype=torch.uint8, device="cuda")
    clocks = Clocks(0)
    clocks.start()
    head = make_graph(torch, args.config)
    rec = measure(torch, lf, head, 2, args.steps, args.warmup, flush, use_graph=not args.no_graph)
    fstats = lf.forest_stats(head["N"], rec["_pipeline"].ws_l)
    rec["_pipeline"] = None
    clk = clocks.stop()
    e2e = None if args.no_e2e else e2e_single(torch, lf, head, max(3, min(args.steps, 5)))
    del head
    torch.cuda.empty_cache()

    extras = {}
    for cfg in [c for c in args.extra.split(",") if c]:
        if cfg.startswith("G"):  # a general (non-symmetric) input, SURVEY.md §8(f) f3
            extras[cfg] = measure_general(torch, lf, cfg, max(5, args.steps // 2), 3, flush)
            torch.cuda.empty_cache()
            continue
        if cfg.startswith("B"):  # AlgTriBlockPrecond construction, SURVEY.md §8(f) f1
            extras[cfg] = measure_block(torch, lf, cfg, max(5, args.steps // 2), 3, flush)
            torch.cuda.empty_cache()
            continue
        name, n = (cfg.split("n")[0], int(cfg.split("n")[1])) if "n" in cfg else (cfg, 2)
        g = make_graph(torch, name)
        r = measure(torch, lf, g, n, max(5, args.steps // 2), 3, flush, use_graph=not args.no_graph)
        if n == 2:
            r["roofline"] = roofline(r, name, clk.get("sm_mhz"), sm_count)
        for k in ("_kavg", "_pipeline"):
            r.pop(k, None)
        extras[r["name"]] = r
        del g
        torch.cuda.empty_cache()

    cpu = None
    if not args.no_cpu_baseline:
        A = cpu_sample() if args.config == "C5" else __import__("lfgen").config(args.config)
        cpu = cpu_baseline(A, args.cpu_runs, args.config)

    t = rec["ms_per_step"]
    rl = roofline(rec, args.config, clk.get("sm_mhz"), sm_count)
    kavg = rec.pop("_kavg")
    out = {
        "metric": METRIC,
        "value": rec["Medges_per_s"],
        "unit": "Medges/s",
        "n_gpus": 1,
        "steps": args.steps,
        "warmup": args.warmup,
        "ms_per_step": t,
        "higher_is_better": True,
        "scaling": "strong" if args.config == "C5" else "weak",
        "vs_baseline": None,
        "dtype": "f32",
        "data": "synthetic",
        "config": {
            "workload": CONFIG_DESC.get(args.config, args.config), "name": args.config,
            "N": rec["N"], "E": rec["E"], "nnz": rec["nnz"], "n": 2, "M": 5, "m": 5, "k_m": 0,
            "per_rank": "single graph", "l2": "flushed between steps (512 MB write)",
            "graph": rec["graph"], "step_time": "median of the timed steps",
        },
        "survey_roofline": {**rec["bytes"], "t_step_ms": t, "frac_B_alg_of_measured_peak": rec["frac_of_peak"],
                            "frac_B_alg_of_nominal_8TBs": rec["frac_of_nominal_8TBs"],
                            "formula": "SURVEY.md §8(d): B_alg = sum_k[8 Z_a + (16+16n) N_a + 2N] + 40N + 36N "
                                       "over the timed step (factor + linear forest + perm + tridiag)"},
        "roofline": rl,
        "kernels_ms": rec["kernels_ms"],
        "stages_ms": {"factor": round(sum(v for k, v in kavg.items() if k.split("[")[0] in (
            "propose", "mutual", "rounds_fused", "propose_long", "init_state", "diag", "finalize")), 4)},
        "forest_stats": fstats,
        "live_rows": rec["live_rows"],
        "live_nnz": rec["live_nnz"],
        "gpu_launches": rec["launches"],
        "clocks": clk,
        "configs": extras,
    }
    out["stages_ms"]["linear_forest_tridiag"] = round(sum(kavg.values()) - out["stages_ms"]["factor"], 4)
    if e2e:
        out["e2e"] = e2e
    if cpu:
        out["cpu_baseline"] = cpu
    emit_line(out)


if __name__ == "__main__":
    main()
