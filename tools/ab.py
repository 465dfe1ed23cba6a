"""A/B timing of compile-time variants of libatos (tools only; replaces the one-off exp*.sh launchers).

  python tools/ab.py build TAG [-DNAME[=V] ...]        # here: variants/libatos_TAG.so (nvcc, sm_100a)
  python tools/ab.py run --tags base,TAG1,... [--apps bfs-rmat,bfs-mesh,pr,gc] [--rounds 2] [--reps 3]
                         [--extra k=v,...] [--scale S]
                                                        # on the GPU: tools/sweep.py per (round, app, tag),
                                                        # tags interleaved so clock drift hits all alike
`base` is the in-tree libatos.so.  Prints one summary line per (app, tag): median over rounds of the
median device ms (stats.kernel_ms) and of the worker-kernel ms."""
import argparse
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
GRID = {"bfs-rmat": "256:256:1", "bfs-mesh": "256:256:1", "bfs-road": "256:256:1", "pr": "512:512:1",
        "gc": "1024:48:1"}


def lib_of(tag):
    return os.path.join(ROOT, "paper_conf_icpp_chenbpbyo22_b200", "libatos.so") if tag == "base" else \
        os.path.join(ROOT, "variants", f"libatos_{tag}.so")


def build(tag, defines):
    from paper_conf_icpp_chenbpbyo22_b200 import build_lib
    os.makedirs(os.path.join(ROOT, "variants"), exist_ok=True)
    print(build_lib.build(force=True, out=lib_of(tag), defines=[d[2:] for d in defines]))


def run(a):
    import numpy as np
    res = {}
    for rnd in range(a.rounds):
        for app in a.apps.split(","):
            for tag in a.tags.split(","):
                cmd = [sys.executable, os.path.join(ROOT, "tools", "sweep.py"), app, "--reps", str(a.reps),
                       "--grid", a.grid or GRID[app]]
                if a.scale:
                    cmd += ["--scale", str(a.scale)]
                if a.extra:
                    cmd += ["--extra", a.extra]
                if app == "bfs-rmat":
                    cmd += ["--sources", "8"]
                env = dict(os.environ, ATOS_LIB=lib_of(tag))
                out = subprocess.run(cmd, capture_output=True, text=True, env=env, timeout=900).stdout
                for line in out.splitlines():
                    mm = re.search(r"^\s*(\S+)\s+ms med\s+([\d.]+).*worker\s+([\d.]+).*edges/m\s+([\d.]+)"
                                   r"(?:.*colors\s+(\d+))?", line)
                    if mm:
                        key = (app, mm.group(1), tag)
                        vals = [float(x) for x in mm.groups()[1:4]] + [float(mm.group(5) or 0)]
                        res.setdefault(key, []).append(tuple(vals))
                        print(f"round {rnd} {app:9s} {mm.group(1):12s} {tag:14s} {vals}", flush=True)
                    elif "ERROR" in line:
                        print(f"[{app} {tag}] {line.strip()}", flush=True)
                if not out.strip():
                    print(f"[{app} {tag}] no output", flush=True)
    print("# app spec tag: median ms, median worker ms, edges/m, colours (over rounds)")
    for (app, spec, tag), v in sorted(res.items()):
        v = np.array(v)
        print(f"{app:9s} {spec:12s} {tag:14s} ms {np.median(v[:, 0]):9.3f}  worker {np.median(v[:, 1]):9.3f}  "
              f"edges/m {np.median(v[:, 2]):7.3f}" + (f"  colours {np.median(v[:, 3]):.0f}" if v[0, 3] else "")
              + f"  (n={len(v)})", flush=True)


def main():
    if len(sys.argv) > 1 and sys.argv[1] == "build":
        build(sys.argv[2], sys.argv[3:])
        return
    ap = argparse.ArgumentParser()
    ap.add_argument("cmd")
    ap.add_argument("--tags", default="base")
    ap.add_argument("--apps", default="bfs-rmat")
    ap.add_argument("--rounds", type=int, default=2)
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--grid", default=None)
    ap.add_argument("--extra", default="")
    ap.add_argument("--scale", type=int, default=None)
    run(ap.parse_args())


if __name__ == "__main__":
    main()
