"""Summarise an ncu --set full report: key throughput metrics, stall reasons, hot source lines."""
import csv
import io
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sectors_op_atom.sum", "lts__t_sectors_op_red.sum",
        "lts__t_sector_hit_rate.pct", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "lts__throughput.avg.pct_of_peak_sustained_elapsed",
        "smsp__inst_executed.sum", "launch__occupancy_limit_registers", "launch__occupancy_limit_shared_mem"]


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    return rows[0], rows[1], rows[2:]


def main(rep, nsrc=25):
    h, u, vals = raw(rep)
    for row in vals:
        name = row[h.index("Kernel Name")] if "Kernel Name" in h else "?"
        print(f"== {name[:120]}")
        for k in KEYS:
            if k in h:
                i = h.index(k)
                print(f"  {k:60s} {row[i]:>16s} {u[i]}")
        st = []
        for i, n in enumerate(h):
            if n.startswith("smsp__average_warps_issue_stalled_") and n.endswith("_per_issue_active.ratio"):
                try:
                    st.append((float(row[i]), n.replace("smsp__average_warps_issue_stalled_", "").replace(
                        "_per_issue_active.ratio", "")))
                except ValueError:
                    pass
        print("  stalls (warps per issue):", ", ".join(f"{n}={x:.1f}" for x, n in sorted(st, reverse=True)[:8]))
    # source hot spots
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    if not rows:
        return
    hdr = rows[0]
    try:
        si = [i for i, n in enumerate(hdr) if n.startswith("Warp Stall Sampling (All")][0]
    except IndexError:
        print("no source sampling column; headers:", hdr[:12])
        return
    li = hdr.index("# Line") if "# Line" in hdr else 0
    src = hdr.index("Source") if "Source" in hdr else 1
    recs = []
    for r in rows[1:]:
        try:
            recs.append((float(r[si] or 0), r[li], r[src].strip()[:110]))
        except (ValueError, IndexError):
            pass
    tot = sum(x for x, _, _ in recs) or 1
    print(f"  hot source lines (share of warp-stall samples):")
    for x, l, s in sorted(recs, reverse=True)[:nsrc]:
        print(f"  {100 * x / tot:5.1f}%  L{l:>5s}  {s}")


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 25)
