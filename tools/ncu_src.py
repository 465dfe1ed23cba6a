"""Per-CUDA-source-line metrics from an ncu report captured with --import-source on (inlined lines included).

usage: python tools/ncu_src.py REPORT.ncu-rep [N] [sort_key]
sort_key: stall (default) | inst | l2sec | l2exc"""
import csv
import io
import subprocess
import sys


def rows(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                         capture_output=True, text=True).stdout
    f, hdr, res = "?", None, []
    for r in csv.reader(io.StringIO(out)):
        if not r:
            continue
        if r[0] == "File Path":
            f = r[1].split("/")[-1]
            continue
        if r[0] == "Line No":
            hdr = r
            continue
        if hdr is None or not r[0].isdigit():
            continue
        d = dict(zip(hdr[2:], r[2:]))  # skip 'Line No','Source'
        d["_src"] = r[1].strip()[:90]
        d["_key"] = f"{f}:{r[0]}"
        res.append(d)
    return res


def num(d, k):
    try:
        return float(d.get(k, "0") or 0)
    except ValueError:
        return 0.0


def main():
    rep = sys.argv[1]
    n = int(sys.argv[2]) if len(sys.argv) > 2 else 30
    key = sys.argv[3] if len(sys.argv) > 3 else "stall"
    rs = rows(rep)
    col = {"stall": "Warp Stall Sampling (All Samples)", "inst": "Instructions Executed",
           "l2sec": "L2 Theoretical Sectors Global", "l2exc": "L2 Theoretical Sectors Global Excessive"}[key]
    ts = sum(num(d, "Warp Stall Sampling (All Samples)") for d in rs) or 1
    ti = sum(num(d, "Instructions Executed") for d in rs) or 1
    tl = sum(num(d, "L2 Theoretical Sectors Global") for d in rs) or 1
    print(f"total inst {ti:.3e}  stall samples {ts:.0f}  L2 theoretical global sectors {tl:.3e}")
    print(" stall%  inst%   L2sec(G)  L2exc(G)  L1tagreq(G) line / source")
    for d in sorted(rs, key=lambda d: -num(d, col))[:n]:
        print(f"{100*num(d,'Warp Stall Sampling (All Samples)')/ts:6.1f} {100*num(d,'Instructions Executed')/ti:6.1f} "
              f"{num(d,'L2 Theoretical Sectors Global')/1e9:9.3f} {num(d,'L2 Theoretical Sectors Global Excessive')/1e9:9.3f} "
              f"{num(d,'L1 Tag Requests Global')/1e9:9.3f}  {d['_key']}  {d['_src']}")


if __name__ == "__main__":
    main()
