#!/usr/bin/env python
"""Summarise ncu outputs for profiles/: launch list shares and --set full key metrics.

usage: python scripts/ncu_summary.py <tag> [launches.csv] [prof1.ncu-rep ...] > profiles/<tag>.md
"""
import csv
import io
import subprocess
import sys
from collections import defaultdict

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "launch__registers_per_thread",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__grid_size",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_bytes.sum",
        "launch__occupancy_limit_registers"]


def launches(path):
    rows = list(csv.reader(open(path)))
    h = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
    hdr, data = rows[h], rows[h + 1:]
    ki, vi, ui = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Unit")
    tot = defaultdict(float)
    cnt = defaultdict(int)
    for r in data:
        name = r[ki].split("(")[0].replace("void ", "")
        v = float(r[vi].replace(",", ""))
        v = v / 1e3 if r[ui] == "ns" else (v * 1e3 if r[ui] == "ms" else v)  # -> us
        tot[name] += v
        cnt[name] += 1
    s = sum(tot.values())
    out = ["| kernel | launches | total us | share |", "|---|---|---|---|"]
    for k, v in sorted(tot.items(), key=lambda t: -t[1]):
        out.append(f"| `{k}` | {cnt[k]} | {v:.1f} | {100 * v / s:.1f}% |")
    return "\n".join(out)


def full(path):
    txt = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    if not rows:
        return f"(no data in {path})"
    hdr = rows[0]
    idx = [(k, hdr.index(k)) for k in KEYS if k in hdr]
    ni = hdr.index("Kernel Name")
    out = ["| kernel | " + " | ".join(k.split("__", 1)[1] for k, _ in idx) + " |",
           "|---|" + "---|" * len(idx)]
    for r in rows[2:]:
        out.append(f"| `{r[ni][:40]}` | " + " | ".join(r[i] for _, i in idx) + " |")
    return "\n".join(out)


if __name__ == "__main__":
    tag = sys.argv[1]
    print(f"# ncu summary {tag}\n")
    for a in sys.argv[2:]:
        if a.endswith(".csv"):
            print(f"## launch list ({a}; cold-cache, serialised: compare shares)\n")
            print(launches(a))
        else:
            print(f"\n## ncu --set full ({a})\n")
            print(full(a))
        print()


NAME_MAP = {  # ncu kernel name prefix -> bench.py kernel record name (first launch of a step)
    "k_lf_local1": "lf_local1", "k_lf_local2": "lf_local2", "k_lf_local3": "lf_local3",
    "k_propose_stream": "propose[0]", "k_propose_tile": "propose[0]", "k_rounds_fused": "rounds_fused",
    "k_mutual": "mutual[0]", "k_tridiag": "tridiag", "k_red_scan<1>": "red_scan_cycles",
    "k_red_scan<0>": "red_scan_ranks", "k_perm": "perm",
}


def traffic(path):
    """dram read+write bytes per launch from a --set full capture, keyed like bench.py."""
    txt = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    hdr = rows[0]
    ni, ri, wi = hdr.index("Kernel Name"), hdr.index("dram__bytes_read.sum"), hdr.index("dram__bytes_write.sum")
    units = rows[1]
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
    out = {}
    for r in rows[2:]:
        name = r[ni].replace("void ", "")
        for pre, key in NAME_MAP.items():
            if name.startswith(pre) and key not in out:
                b = float(r[ri].replace(",", "")) * scale.get(units[ri], 1) + \
                    float(r[wi].replace(",", "")) * scale.get(units[wi], 1)
                out[key] = int(b)
    return out
