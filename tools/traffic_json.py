"""Rebuild profiles/traffic.json (bench.py's roofline.traffic) from the per-launch ncu metric CSVs of a
profiling pass: python tools/traffic_json.py <dir with *_traffic.csv> <round tag>"""
import csv
import io
import json
import os
import sys

KEYS = {"bfs_worker": ("bfs_s26_traffic.csv", "C5 RMAT S26 EF16 seed 5, source seed 105, degree layout"),
        "pr_worker": ("pr_s22_traffic.csv", "C3 RMAT S22 EF16 seed 3, alpha 0.85 eps 1e-6"),
        "pr_worker_c5": ("pr_s26_traffic.csv", "C5 RMAT S26 EF16 seed 5, alpha 0.85 eps 1e-6, degree layout"),
        "color_worker": ("gc_s20_traffic.csv", "C4 Kronecker S20 EF64 seed 4, seed 1")}


def metrics(path):
    rows = [r for r in csv.reader(io.StringIO(open(path).read())) if r]
    h = None
    out, kern = {}, None
    for r in rows:
        if r[0] == "ID":
            h = r
            continue
        if h and len(r) == len(h):
            d = dict(zip(h, r))
            kern = d["Kernel Name"]
            v = d["Metric Value"].replace(",", "")
            unit = d["Metric Unit"]
            x = float(v)
            if unit == "Gbyte":
                x *= 1e9
            elif unit == "Mbyte":
                x *= 1e6
            elif unit == "Kbyte":
                x *= 1e3
            elif unit == "ms":
                x *= 1e6  # -> ns
            elif unit == "us":
                x *= 1e3
            out[d["Metric Name"]] = x
    return kern, out


def main():
    src, tag = sys.argv[1], sys.argv[2]
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    res = {"_note": "dram__bytes_read.sum + dram__bytes_write.sum of ONE launch of the dominant kernel, from "
                    "`ncu --metrics ... -c 1` (tools/profile_r02.sh; CSVs under profiles/). bench.py reports it as "
                    "roofline.traffic next to the algorithmic bytes."}
    for key, (fn, wl) in KEYS.items():
        kern, m = metrics(os.path.join(src, fn))
        res[key] = {"kernel": kern, "workload": wl,
                    "dram_bytes_per_launch": int(m["dram__bytes_read.sum"] + m["dram__bytes_write.sum"]),
                    "dram_read": int(m["dram__bytes_read.sum"]), "dram_write": int(m["dram__bytes_write.sum"]),
                    "duration_ms_under_ncu": m["gpu__time_duration.sum"] / 1e6,
                    "l2_sectors_from_sm": int(m["lts__t_sectors_srcunit_tex.sum"]),
                    "l2_hit_rate_pct": m["lts__t_sector_hit_rate.pct"],
                    "l2_atom_sectors": int(m["lts__t_sectors_op_atom.sum"]),
                    "l2_red_sectors": int(m["lts__t_sectors_op_red.sum"]),
                    "registers_per_thread": int(m.get("launch__registers_per_thread", 0)),
                    "warps_active_pct": m.get("sm__warps_active.avg.pct_of_peak_sustained_active"),
                    "csv": f"profiles/{tag}_{fn}"}
    json.dump(res, open(os.path.join(root, "profiles", "traffic.json"), "w"), indent=2)
    print(json.dumps(res, indent=1))


if __name__ == "__main__":
    main()
