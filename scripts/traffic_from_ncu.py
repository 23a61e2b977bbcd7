"""profiles/traffic.json from an ncu --set full capture of the step's kernels:
dram bytes (read + write) and warp instructions per launch, keyed by bench stage name.

usage: python scripts/traffic_from_ncu.py gpurun_out/prof_<tag>.ncu-rep <tag>
"""
import csv
import io
import json
import os
import subprocess
import sys

STAGE = {"k_propose_stream": "propose[0]", "k_mutual0": "mutual[0]", "k_rounds_fused": "rounds_fused",
         "k_lf_full1": "lf_tile", "k_red_full": "red_scan", "k_lf_full2": "lf_expand",
         "k_perm_tri": "perm_tridiag"}
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "inst": 1, "": 1}


def main(rep, tag):
    txt = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    hdr, units = rows[0], rows[1]
    ki = hdr.index("Kernel Name")
    cols = {k: hdr.index(k) for k in ("dram__bytes_read.sum", "dram__bytes_write.sum", "smsp__inst_executed.sum")}

    def val(r, k):
        i = cols[k]
        return float(r[i].replace(",", "")) * SCALE.get(units[i], 1)

    out_b, out_i = {}, {}
    for r in rows[2:]:
        for k, st in STAGE.items():
            if k in r[ki] and st not in out_b:
                out_b[st] = int(val(r, "dram__bytes_read.sum") + val(r, "dram__bytes_write.sum"))
                out_i[st] = int(val(r, "smsp__inst_executed.sum"))
    path = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles", "traffic.json")
    json.dump({"source": f"profiles/{tag}_ncu.md (ncu --set full, C2, one launch each)",
               "bytes_per_launch": out_b, "warp_inst_per_launch": out_i}, open(path, "w"), indent=1)
    print(json.dumps(out_b), json.dumps(out_i))


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2])
