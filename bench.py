#!/usr/bin/env python
"""Benchmark of the hot path: [0,2]-factor (M=5) + linear forest + permutation + tridiag.

Contract: `python bench.py --gpus N --steps K --warmup W` prints ONE
JSON line on rank 0.  A step is one pass of the whole hot path over one synthetic graph
resident in HBM; `value` is whole-job Medges/s (undirected edges E / step time, summed
over ranks).  Device time with CUDA events per step, L2 flushed between steps, max over
ranks.  `--impl reference` times the CPU oracle (the reference arm of this tier).
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "ms and Medges/s per [0,2]-factor+linear forest at 1/2/4/8 B200; % HBM peak"
CONFIG_DESC = {
    "C1": "2D 5-pt 64x64 (4,096 vertices), n=2",
    "C2": "3D 7-pt anisotropic 128^3 (2.1M vertices, 6.24M edges), n=2",
    "C3": "FEM-like jittered 27-pt 100^3 bricks (1M vertices), n=2",
    "C4": "Chung-Lu power-law 5M vertices, n=2",
}


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="C2")
    ap.add_argument("--no-graph", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-runs", type=int, default=8)
    ap.add_argument("--force-multi", action="store_true",
                    help="use the row-partitioned multi-GPU path even at one rank (testing)")
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
        return float(d["hbm_gbs"]), "measured"
    return 6650.0, "fallback"


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


def kernel_bytes(name, N, Z, n, live_rows, live_nnz, cluster_ran=False):
    """Algorithmic HBM bytes of one launch: what the method must move."""
    base = name.split("[")[0]
    k = int(name.split("[")[1].rstrip("]")) if "[" in name else -1
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
    if base == "rounds_fused" and cluster_ran:  # skipped: k_rounds_cluster ran the rounds
        return 0
    if base in ("rounds_fused", "rounds_cluster"):  # rounds 1..M-1: live rows' propose + mutual traffic
        return sum(kernel_bytes(f"propose[{kk}]", N, Z, n, live_rows, live_nnz)
                   + kernel_bytes(f"mutual[{kk}]", N, Z, n, live_rows, live_nnz)
                   for kk in range(1, len(live_rows)))
    # linear forest: B_LF = 40N attributed to the kernel that moves it;
    # block-local intermediates (loc1/loc2, boundary records) are implementation traffic
    # single-pass forest: the tile pass reads the factor; the tile pass (local
    # vertices) and the expand pass (the rest) together write forest, path_id, pos once each
    if base == "lf_tile":
        return 16 * N  # read pi2 + pi2_w
    if base == "lf_expand":
        return 16 * N  # write forest, path_id, pos
    if base == "red_scan":
        return 0  # boundary records only: implementation traffic
    if base == "lf_local1":
        return 16 * N  # read pi2 + pi2_w
    if base == "lf_local2":
        return 8 * N  # write forest
    if base == "lf_local3":
        return 8 * N  # write path_id, pos
    if base == "perm":
        return 8 * N  # write perm, iperm
    if base == "perm_tridiag":  # write perm, iperm; read forest, pi2, pi2_val, diag; write a, b, c
        return 8 * N + 8 * N + 8 * N + 8 * N + 4 * N + 12 * N
    if base == "tridiag":
        return 8 * N + 4 * N + 8 * N + 8 * N + 4 * N + 12 * N
    return 0


def ncu_traffic(kernel, key="bytes_per_launch"):
    """dram bytes (or warp instructions) per launch of `kernel` from the committed ncu
    capture (profiles/traffic.json)."""
    p = os.path.join(ROOT, "profiles", "traffic.json")
    try:
        return json.load(open(p))[key].get(kernel)
    except (OSError, ValueError, KeyError):
        return None


def issue_view(kernel, ms, sm_count, mhz):
    """The dominant kernel against the SM issue rate (4 warp instructions per SM per cycle):
    its ncu warp-instruction count per launch over its live launch time."""
    inst = ncu_traffic(kernel, "warp_inst_per_launch")
    if not inst or not ms or not mhz:
        return None
    ach = inst / (ms * 1e-3) / 1e9
    peak = 4 * sm_count * mhz * 1e6 / 1e9
    return {"bound": "issue", "achieved": round(ach, 1), "peak": round(peak, 1),
            "unit": "G warp-inst/s", "frac": round(ach / peak, 4), "warp_inst_per_launch": inst,
            "source": "ncu smsp__inst_executed.sum (profiles/traffic.json) / live launch time"}


def cpu_baseline(A, runs):
    import oracle

    oracle.build()
    t0 = time.perf_counter()
    for _ in range(runs):
        oracle.run_pipeline(A)
    dt = (time.perf_counter() - t0) / runs
    return {"value": A.n_edges / dt / 1e6, "unit": "Medges/s", "cores": 1, "kind": "oracle",
            "ms_per_graph": dt * 1e3,
            "sample": f"full {A.name} graph (N={A.N}, E={A.n_edges}), oracle pipeline "
                      f"(Alg. 2 M=5 + walks + sort + tridiag) x{runs}, single thread"}


def run_reference(args):
    ws, rank, _ = dist_env()
    if rank != 0:
        return
    import lfgen
    import oracle

    oracle.build()
    A = lfgen.config(args.config)
    for _ in range(args.warmup):
        oracle.run_pipeline(A)
    ts = []
    for _ in range(args.steps):
        t0 = time.perf_counter()
        oracle.run_pipeline(A)
        ts.append(time.perf_counter() - t0)
    ms = 1e3 * sum(ts) / len(ts)
    val = A.n_edges / (ms / 1e3) / 1e6
    out = {
        "impl": "reference", "metric": METRIC, "value": round(val, 3), "unit": "Medges/s",
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms, 3),
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f32",
        "data": "synthetic", "config": {"workload": CONFIG_DESC.get(args.config, args.config),
                                        "name": args.config, "N": A.N, "E": A.n_edges, "nnz": A.nnz},
        "cpu_baseline": {"value": round(val, 3), "unit": "Medges/s", "cores": 1, "kind": "oracle",
                         "sample": f"full {A.name} graph per step, single thread"},
        "e2e": {"value": round(val, 3), "unit": "Medges/s", "h2d_bytes_per_step": 0,
                "d2h_bytes_per_step": 0},
    }
    print(json.dumps(out), flush=True)


def run_multi(args, ws, rank, local):
    """N > 1: weak scaling.  The graph is the C2 recipe on a 128 x 128 x (128 N) grid; rank r
    owns z-planes [128 r, 128 r + 128) (one C2-sized slab, 2.1M vertices) and runs the
    row-partitioned factor with NCCL halo exchanges, the boundary-end-list linear forest
    and the tridiagonal extraction."""
    import torch
    import torch.distributed as tdist

    import lfgen
    from paper_conf_icpp_0002s22_b200 import _build, dist, lf

    torch.cuda.set_device(local)
    tdist.init_process_group("nccl", device_id=torch.device("cuda", local))
    _build.build()
    lf.load()
    n = 128
    nz = n * ws
    rp, col, val, lo, hi = lfgen.grid3d_7pt_aniso_rows(n, nz, rank * n, (rank + 1) * n)
    bounds = dist.slab_bounds(nz, n * n, ws)
    N = n * n * nz
    E_rank = (int(rp[-1]) - (hi - lo)) // 2  # undirected edges per rank (halo edges counted half)
    E_tot = torch.tensor([int(rp[-1]) - (hi - lo)], dtype=torch.int64, device="cuda")
    tdist.all_reduce(E_tot)
    E = int(E_tot.item()) // 2
    rpd, cold, vald = (torch.from_numpy(x).cuda() for x in (rp, col, val))
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
        for _ in range(5):
            step()
        torch.cuda.synchronize()
    tdist.barrier()
    torch.cuda.synchronize()
    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    step_ms = []
    for _ in range(args.steps):
        flush.zero_()
        tdist.barrier()
        ev0.record(stream)
        step()
        ev1.record(stream)
        ev1.synchronize()
        step_ms.append(ev0.elapsed_time(ev1))
    torch.cuda.synchronize()
    tdist.barrier()
    # per-kernel breakdown from one instrumented step per timed step count (rank-local)
    kern = {}
    for _ in range(min(args.steps, 5)):
        flush.zero_()
        lf.profile_enable(True)
        step()
        lf.profile_enable(False)
        torch.cuda.synchronize()
        for nm, ms in lf.profile_collect():
            kern.setdefault(nm, []).append(ms)
    clk = clocks.stop()
    t = torch.tensor([sum(step_ms) / len(step_ms)], dtype=torch.float64, device="cuda")
    tdist.all_reduce(t, op=tdist.ReduceOp.MAX)
    t_step = float(t.item())
    # e2e: own slab from pinned host memory, partition setup, the three stages, results back
    rp_h, col_h, val_h = (torch.from_numpy(x).pin_memory() for x in (rp, col, val))
    n_own = hi - lo
    outs_h = [torch.empty(n_own, dtype=dt, pin_memory=True) for dt in (torch.int32, torch.int32, torch.int32,
                                                                        torch.float32, torch.float32, torch.float32)]
    e2e_ms = []
    for _ in range(max(2, min(args.steps, 5))):
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
    te = torch.tensor([sum(e2e_ms) / len(e2e_ms)], dtype=torch.float64, device="cuda")
    tdist.all_reduce(te, op=tdist.ReduceOp.MAX)
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
            "scaling": "weak",
            "vs_baseline": None,
            "dtype": "f32",
            "data": "synthetic",
            "config": {
                "workload": f"C2 recipe on a 128x128x{nz} grid, one 128^3 z-slab (2.1M vertices) per rank",
                "name": "C2-slabs", "N": N, "E": E, "n": 2, "M": 5, "m": 5, "k_m": 0,
                "parallelism": f"row-partitioned z-slabs x{ws}, NCCL halo exchange + boundary-end list",
                "halo_entries_per_exchange_rank0": info["halo_sent"],
                "l2": "flushed between steps (512 MB write)", "graph": False,
            },
            "kernels_ms_rank0": {k: round(v, 5) for k, v in sorted(kavg.items(), key=lambda x: -x[1])},
            "roofline": {"kernel": dom, "bound": "hbm", "achieved": None, "peak": peak,
                         "peak_kind": peak_kind, "unit": "GB/s", "frac": None, "traffic": None,
                         "ms_per_launch": round(kavg[dom], 5) if dom else None},
            "e2e": {"value": round(E / (float(te.item()) * 1e-3) / 1e6, 2), "unit": "Medges/s",
                    "ms_per_step": round(float(te.item()), 3),
                    "h2d_bytes_per_step": int(8 * (n_own + 1) + 8 * int(rp[-1])) * ws,
                    "d2h_bytes_per_step": int(24 * n_own) * ws,
                    "includes": "partition setup (ghost relabeling, halo plan)"},
            "gpu_launches": sum(len(v) for v in kern.values()) // max(1, min(args.steps, 5)),
            "clocks": clk,
        }
        E_rank  # noqa: B018  (per-rank share; the metric uses the global E)
        print(json.dumps(out), flush=True)
    part.close()
    comm.close()
    tdist.destroy_process_group()


def main():
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
    import numpy as np
    import torch

    import lfgen
    from paper_conf_icpp_0002s22_b200 import _build, lf

    ws, rank, local = dist_env()
    torch.cuda.set_device(local)
    if ws > 1:
        import torch.distributed as dist

        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    _build.build()
    lf.load()

    A = lfgen.config(args.config)
    N, Z, E = A.N, A.nnz, A.n_edges
    rp = torch.from_numpy(A.rowptr).cuda()
    col = torch.from_numpy(A.col).cuda()
    val = torch.from_numpy(A.val).cuda()
    P = lf.Pipeline(rp, col, val)
    flush = torch.empty(512 * 1024 * 1024, dtype=torch.uint8, device="cuda")
    stream = torch.cuda.current_stream()

    clocks = Clocks(local)
    clocks.start()
    for _ in range(max(args.warmup, 3)):
        P.run()
    torch.cuda.synchronize()

    def capture(prof):
        lf.profile_enable(prof)
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            P.run()
        torch.cuda.synchronize()
        g.replay()
        torch.cuda.synchronize()
        return g

    graph = graph_prof = None
    if not args.no_graph:
        try:
            s = torch.cuda.Stream()
            s.wait_stream(stream)
            with torch.cuda.stream(s):
                P.run()  # warm a side stream once before capture
            torch.cuda.synchronize()
            graph = capture(False)       # the timed step: no instrumentation
            graph_prof = capture(True)   # same launches + event records per kernel
            lf.profile_enable(False)
        except Exception as e:  # capture unsupported -> eager launches
            print(f"# graph capture failed ({e}); timing eager launches", file=sys.stderr)
            graph = graph_prof = None
    launches_per_step = None

    def step(prof=False):
        if graph is not None:
            (graph_prof if prof else graph).replay()
        else:
            lf.profile_enable(prof)
            P.run()

    # keep the GPU busy until the clock sampler is producing samples (bounded)
    t_end = time.time() + 5.0
    while clocks.n_samples() < 3 and time.time() < t_end:
        for _ in range(10):
            step()
        torch.cuda.synchronize()
    if ws > 1:
        torch.distributed.barrier()
    torch.cuda.synchronize()
    step_ms, prof_step_ms, kern = [], [], {}
    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    # timed region: K steps of the plain graph (L2 flushed before each)
    for _ in range(args.steps):
        flush.zero_()  # write 512 MB > 126 MB L2 between steps
        ev0.record(stream)
        step()
        ev1.record(stream)
        ev1.synchronize()
        step_ms.append(ev0.elapsed_time(ev1))
    # per-kernel breakdown: K steps of the instrumented graph, same conditions
    for _ in range(args.steps):
        flush.zero_()
        ev0.record(stream)
        step(prof=True)
        ev1.record(stream)
        ev1.synchronize()
        prof_step_ms.append(ev0.elapsed_time(ev1))
        recs = lf.profile_collect()
        # one record per stage; the perm stage launches k_tile_prefix + k_perm_tri, and every
        # lf_linear_forest call starts with the (unrecorded) control-block kernel k_ctl_zero
        launches_per_step = sum(2 if nm in ("perm", "perm_tridiag") else 1 for nm, _ in recs) + 1
        for nm, ms in recs:
            kern.setdefault(nm, []).append(ms)
    torch.cuda.synchronize()
    if ws > 1:
        torch.distributed.barrier()
    t_end = time.time() + 1.0
    n0 = clocks.n_samples()
    while clocks.n_samples() < n0 + 2 and time.time() < t_end:
        time.sleep(0.05)
    clk = clocks.stop()
    lf.profile_enable(False)

    t_step = sum(step_ms) / len(step_ms)
    if ws > 1:
        t = torch.tensor([t_step], device="cuda", dtype=torch.float64)
        torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
        t_step = float(t.item())

    fstats = lf.forest_stats(N, P.ws_l)
    live = P.fac["live"].cpu().numpy()
    M = P.M
    lr, ln = [int(x) for x in live[:M]], [int(x) for x in live[M:2 * M]]
    kavg = {nm: sum(v) / len(v) for nm, v in kern.items()}
    FACTOR_K = ("propose", "mutual", "rounds", "init_state", "diag", "rounds_fused", "rounds_cluster",
                "finalize", "propose_long")
    stage = {"factor": sum(t for nm, t in kavg.items() if nm.split("[")[0] in FACTOR_K),
             "linear_forest_tridiag": sum(t for nm, t in kavg.items() if nm.split("[")[0] not in FACTOR_K)}
    dom = max(kavg, key=kavg.get) if kavg else None
    peak, peak_kind = load_peaks()
    n = 2
    # k_rounds_cluster ran the rounds iff the fused fallback found its `done` flag (a few us)
    cl_ran = "rounds_cluster" in kavg and kavg.get("rounds_fused", 0.0) < 0.25 * kavg["rounds_cluster"]
    dom_bytes = kernel_bytes(dom, N, Z, n, lr, ln, cl_ran) if dom else 0
    dom_ach = dom_bytes / (kavg[dom] * 1e-3) / 1e9 if dom else None
    b_main = sum(kernel_bytes(nm, N, Z, n, lr, ln, cl_ran) for nm in kavg)
    t_main = stage["factor"] + stage["linear_forest_tridiag"]

    # e2e through the C ABI with HOST buffers (pinned), copies inside the timed region
    rp_h = torch.from_numpy(A.rowptr).pin_memory()
    col_h = torch.from_numpy(A.col).pin_memory()
    val_h = torch.from_numpy(A.val).pin_memory()
    e2e_ws = lf.Workspace()
    outs = None
    for _ in range(2):
        outs = lf.pipeline_host(rp_h, col_h, val_h, ws=e2e_ws, outs=outs)
    e2e_ms = []
    for _ in range(max(3, min(args.steps, 10))):
        ev0.record(stream)
        outs = lf.pipeline_host(rp_h, col_h, val_h, ws=e2e_ws, outs=outs)
        ev1.record(stream)
        ev1.synchronize()
        e2e_ms.append(ev0.elapsed_time(ev1))
    e2e_t = sum(e2e_ms) / len(e2e_ms)
    if ws > 1:
        t = torch.tensor([e2e_t], device="cuda", dtype=torch.float64)
        torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
        e2e_t = float(t.item())

    # SURVEY.md §8(f) f2 (next row, not part of the step): apply the preconditioner,
    # y = T^{-1} x on the step's (a, b, c); L2 flushed before each launch; 20 B/row
    # algorithmic (read a, b, c, x; write y), DESIGN.md §4.6
    ta, tb, tc = P.tri
    xr = torch.randn(N, device="cuda", dtype=torch.float32, generator=torch.Generator("cuda").manual_seed(1))
    ts_ws, ts_y = lf.Workspace(), torch.empty(N, device="cuda", dtype=torch.float32)
    for _ in range(3):
        lf.tri_solve(ta, tb, tc, xr, ws=ts_ws, out=ts_y)
    ts_ms, ts_k = [], {}
    for prof in (False, True):
        for _ in range(max(3, args.steps)):
            flush.zero_()
            lf.profile_enable(prof)
            ev0.record(stream)
            lf.tri_solve(ta, tb, tc, xr, ws=ts_ws, out=ts_y)
            ev1.record(stream)
            ev1.synchronize()
            if not prof:
                ts_ms.append(ev0.elapsed_time(ev1))
                continue
            for nm, ms in lf.profile_collect():
                ts_k.setdefault(nm, []).append(ms)
    lf.profile_enable(False)
    ts_t = sum(ts_ms) / len(ts_ms)
    ts_bytes = 20 * N
    tri_solve_rec = {"ms": round(ts_t, 5), "Mrows_per_s": round(N / (ts_t * 1e-3) / 1e6, 1),
                     "kernels_ms": {k: round(sum(v) / len(v), 5) for k, v in ts_k.items()},
                     "roofline": {"bound": "hbm", "alg_bytes": ts_bytes,
                                  "achieved": round(ts_bytes / (ts_t * 1e-3) / 1e9, 1), "peak": peak,
                                  "unit": "GB/s", "frac": round(ts_bytes / (ts_t * 1e-3) / 1e9 / peak, 4)}}

    cpu = None
    if rank == 0 and ws == 1 and not args.no_cpu_baseline:
        cpu = cpu_baseline(A, args.cpu_runs)

    if rank == 0:
        value = ws * E / (t_step * 1e-3) / 1e6
        out = {
            "metric": METRIC,
            "value": round(value, 2),
            "unit": "Medges/s",
            "n_gpus": ws,
            "steps": args.steps,
            "warmup": args.warmup,
            "ms_per_step": round(t_step, 4),
            "higher_is_better": True,
            "scaling": "weak",
            "vs_baseline": None,
            "dtype": "f32",
            "data": "synthetic",
            "config": {
                "workload": CONFIG_DESC.get(args.config, args.config), "name": args.config,
                "N": N, "E": E, "nnz": Z, "n": 2, "M": 5, "m": 5, "k_m": 0,
                "per_rank": "one independent graph per rank" if ws > 1 else "single graph",
                "l2": "flushed between steps (512 MB write)",
                "graph": graph is not None,
            },
            "stages_ms": {k: round(v, 4) for k, v in stage.items()},
            "instrumented_ms_per_step": round(sum(prof_step_ms) / len(prof_step_ms), 4),
            "t_main_ms": round(t_main, 4),
            "B_main_bytes": int(b_main),
            "main_frac_of_peak": round(b_main / (t_main * 1e-3) / 1e9 / peak, 4) if t_main > 0 else None,
            "roofline": {
                "kernel": dom, "bound": "hbm", "achieved": round(dom_ach, 1) if dom_ach else None,
                "peak": peak, "peak_kind": peak_kind, "unit": "GB/s",
                "frac": round(dom_ach / peak, 4) if dom_ach else None,
                "traffic": ncu_traffic(dom) if args.config == "C2" else None,
                "issue_view": issue_view(dom, kavg.get(dom), torch.cuda.get_device_properties(0).multi_processor_count,
                                         clk.get("sm_mhz")) if args.config == "C2" and dom else None,
                "alg_bytes_per_launch": int(dom_bytes),
                "ms_per_launch": round(kavg[dom], 5) if dom else None,
            },
            "kernels_ms": {k: round(v, 5) for k, v in sorted(kavg.items(), key=lambda t: -t[1])},
            "forest_stats": fstats,
            "live_rows": lr,
            "live_nnz": ln,
            "e2e": {"value": round(ws * E / (e2e_t * 1e-3) / 1e6, 2), "unit": "Medges/s",
                    "ms_per_step": round(e2e_t, 3),
                    "h2d_bytes_per_step": int(8 * (N + 1) + 8 * Z),
                    "d2h_bytes_per_step": int(24 * N)},
            "gpu_launches": launches_per_step,
            "clocks": clk,
            "next_rows": {"f2_tri_solve": tri_solve_rec},
        }
        if cpu is not None:
            out["cpu_baseline"] = cpu
        print(json.dumps(out), flush=True)
    if ws > 1:
        torch.distributed.destroy_process_group()


if __name__ == "__main__":
    main()
