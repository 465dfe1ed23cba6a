"""Attribute ncu per-SASS-instruction counts/stall samples to CUDA source lines.

usage: python tools/ncu_lines.py REPORT.ncu-rep OBJECT.o KERNEL_SUBSTRING [N]
Needs the object compiled with -lineinfo (build_lib does).  Instructions are
matched by position within the function (ncu's SASS listing and nvdisasm's)."""
import csv
import os
import io
import re
import subprocess
import sys
from collections import defaultdict


def sass_rows(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr = rows[1]
    ie, ws, si = hdr.index("Instructions Executed"), hdr.index("Warp Stall Sampling (All Samples)"), hdr.index("Source")
    return [(int(r[ie] or 0), int(r[ws] or 0), r[si].strip()) for r in rows[2:] if len(r) > ws and r[ie].isdigit()]


def disasm_lines(obj, kern):
    cub = subprocess.run(["cuobjdump", "-xelf", "all", os.path.abspath(obj)], capture_output=True, text=True, cwd="/tmp").stdout
    name = re.findall(r"Extracting ELF file\s+\d+:\s+(\S+)", cub)[0]
    txt = subprocess.run(["nvdisasm", "--print-line-info", "-c", "/tmp/" + name], capture_output=True, text=True).stdout
    funcs = {}
    cur, line = None, "?"
    for l in txt.splitlines():
        m = re.match(r"\s*\.text\.(\S+):", l)
        if m:
            cur = m.group(1)
            funcs[cur] = []
            continue
        m = re.search(r'line (\d+)', l) if "//## File" in l else None
        if m:
            f = re.search(r'File "([^"]+)"', l)
            line = (f.group(1).split("/")[-1] if f else "?") + ":" + m.group(1)
            continue
        if cur and re.match(r"\s*/\*[0-9a-f]{4,}\*/", l):
            funcs[cur].append(line)
    cands = [k for k in funcs if kern in k]
    return funcs[cands[0]] if cands else []


def main():
    rep, obj, kern = sys.argv[1:4]
    n = int(sys.argv[4]) if len(sys.argv) > 4 else 30
    rows = sass_rows(rep)
    lines = disasm_lines(obj, kern)
    print(f"{len(rows)} ncu instructions, {len(lines)} disassembled")
    agg = defaultdict(lambda: [0, 0])
    for i, (ie, ws, _) in enumerate(rows):
        key = lines[i] if i < len(lines) else "?"
        agg[key][0] += ie
        agg[key][1] += ws
    ti = sum(v[0] for v in agg.values()) or 1
    ts = sum(v[1] for v in agg.values()) or 1
    print("top lines by instructions executed (inst%, stall%)")
    for k, v in sorted(agg.items(), key=lambda x: -x[1][0])[:n]:
        print(f"  {100 * v[0] / ti:5.1f}% {100 * v[1] / ts:5.1f}%  {k}")
    print("top lines by stall samples")
    for k, v in sorted(agg.items(), key=lambda x: -x[1][1])[:n]:
        print(f"  {100 * v[0] / ti:5.1f}% {100 * v[1] / ts:5.1f}%  {k}")


if __name__ == "__main__":
    main()
