"""Summarise an ncu launch list (--metrics gpu__time_duration.sum,dram__bytes_read.sum,
dram__bytes_write.sum,smsp__inst_executed.sum --csv) of `bench.py --steps S --no-graph`:
the launches of the LAST step, each kernel's share of the step, its DRAM traffic per launch
and its warp instructions; writes profiles/<tag>_launch_summary.md and
profiles/traffic_<cfg>.json (bytes / instructions per launch, keyed like lf_profile names).
usage: python scripts/launch_summary.py gpurun_out/launches_c5.csv r02 C5"""
import csv
import json
import os
import re
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
path, tag, cfg = sys.argv[1], sys.argv[2], sys.argv[3]
lines = [ln for ln in open(path) if ln.startswith('"')]  # drop ncu's ==PROF== / ==WARNING== lines
rows = list(csv.DictReader(lines))
launches = {}
for r in rows:
    k = int(r["ID"])
    d = launches.setdefault(k, {"name": r["Kernel Name"]})
    try:
        d[r["Metric Name"]] = float(r["Metric Value"].replace(",", ""))
    except ValueError:
        d[r["Metric Name"]] = 0.0


def short(n):
    m = re.search(r"(k_[A-Za-z0-9_]+)", n)
    return m.group(1) if m else n[:40]


seq = [launches[k] for k in sorted(launches)]
names = [short(x["name"]) for x in seq]
# the last step starts at the last round-0 propose (k_propose_stream)
starts = [i for i, n in enumerate(names) if n == "k_propose_stream"]
step = seq[starts[-1]:]
PROF = {"k_propose_stream": "propose[0]", "k_propose_long_blk": "propose_long", "k_mutual0": "mutual[0]",
        "k_rounds_fused": "rounds_fused", "k_rows_propose_k": "rows_propose", "k_rows_long_k": "rows_long",
        "k_rows_mutual_k": "rows_mutual", "k_grs_pack": "grs_pack", "k_grs_walk": "grs_walk",
        "k_red_full": "red_scan", "k_grs_meet": "grs_walk", "k_grs_len": "grs_len", "k_grs_cycfind": "grs_len", "k_grs_lenscan": "grs_len",
        "k_tile_prefix": "grs_len", "k_grs_emit": "grs_emit_tri", "k_grs_split": "grs_split_tri", "k_ctl_zero": "ctl_zero",
        "k_grs_list": "grs_pack", "k_grs_cyccand": "grs_len", "k_grs_desc": "grs_desc",
        "k_lf_full1": "lf_tile", "k_lf_full2": "lf_expand", "k_perm_tri": "perm_tridiag"}
tot = sum(x["gpu__time_duration.sum"] for x in step)
agg = {}
ridx = {"rows_propose": 0, "rows_long": 0, "rows_mutual": 0, "propose_long": -1}
for x in step:
    n = short(x["name"])
    p = PROF.get(n, n)
    if p in ridx:
        ridx[p] += 1
        p = f"{p}[{ridx[p] if p != 'propose_long' else 0}]" if p != "propose_long" else "propose_long[0]"
    a = agg.setdefault(p, {"ns": 0.0, "dram": 0.0, "inst": 0.0, "launches": 0})
    a["ns"] += x["gpu__time_duration.sum"]
    nz = lambda v: 0.0 if v != v else v  # noqa: E731  (NaN: metric not collected)
    a["dram"] += nz(x.get("dram__bytes_read.sum", 0)) + nz(x.get("dram__bytes_write.sum", 0))
    a["inst"] += nz(x.get("smsp__inst_executed.sum", 0))
    a["launches"] += 1
out = [f"# {tag}: ncu launch list of one bench step ({cfg}), cold-cache serialised launches",
       "", f"source: `{os.path.basename(path)}` ({len(step)} launches in the last step, "
       f"{tot / 1e6:.2f} ms summed); compare SHARES with the bench's per-kernel CUDA-event times, not absolutes.",
       "", "| kernel (profile name) | launches | ms | share | DRAM bytes | DRAM GB/s | warp inst |",
       "|---|---|---|---|---|---|---|"]
for p, a in sorted(agg.items(), key=lambda t: -t[1]["ns"]):
    out.append(f"| {p} | {a['launches']} | {a['ns'] / 1e6:.3f} | {a['ns'] / tot:.1%} | {a['dram']:.3e} | "
               f"{a['dram'] / a['ns']:.1f} | {a['inst']:.3e} |")
open(os.path.join(ROOT, "profiles", f"{tag}_{cfg}_launch_summary.md"), "w").write("\n".join(out) + "\n")
tr = {"source": f"profiles/{tag}_{cfg}_launch_summary.md (ncu launch list, one step)",
      "bytes_per_launch": {p: int(a["dram"] / a["launches"]) for p, a in agg.items()},
      "warp_inst_per_launch": {p: int(a["inst"] / a["launches"]) for p, a in agg.items()},
      "ms_per_launch_ncu": {p: round(a["ns"] / a["launches"] / 1e6, 4) for p, a in agg.items()}}
json.dump(tr, open(os.path.join(ROOT, "profiles", f"traffic_{cfg}.json"), "w"), indent=1)
print("\n".join(out))
