"""Knob sweep (worker size x FETCH_SIZE x kernel strategy, the paper's Fig. 4 design space).

  python tools/sweep.py bfs-mesh|bfs-rmat|pr|gc [--scale S] [--side N] [--reps R] [--grid "w:f:p,w:f:p,..."]

Prints one line per configuration: median / min device ms of the whole call (stats.kernel_ms) and work
counters.  Inputs are the seeded generators of gen.py; timings are CUDA-event based (inside the library).
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_icpp_chenbpbyo22_b200 as atos  # noqa: E402
from paper_conf_icpp_chenbpbyo22_b200 import gen  # noqa: E402

DEFAULT_GRID = {
    "bfs-mesh": "256:256:1,256:256:0,256:64:1,128:128:1,128:32:1,64:64:1,64:16:1,32:1:1,32:4:1,32:8:1,1:1:1,"
                "1:4:1,256:64:0,32:8:0",
    "bfs-road": "256:256:1,256:256:0,128:32:1,64:16:1,32:4:1,32:8:1,1:4:1",
    "bfs-rmat": "256:256:1,512:512:1,512:256:1,128:128:1,1024:1024:1,256:256:0,512:512:0,32:8:1,32:32:1",
    "pr": "256:256:1,512:512:1,128:128:1,1024:1024:1,256:256:0,512:512:0,32:8:1",
    "gc": "512:128:1,256:128:1,1024:128:1,512:64:1,32:8:1,512:128:0",
}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("app")
    ap.add_argument("--scale", type=int, default=None)
    ap.add_argument("--side", type=int, default=4900)
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--grid", default=None)
    ap.add_argument("--extra", default="", help="k=v,k=v knobs added to every configuration")
    ap.add_argument("--layout", default="auto", help="CSR layout: auto | degree | input")
    ap.add_argument("--sources", type=int, default=1, help="bfs-rmat: cycle over the bench's first N sources")
    a = ap.parse_args()
    extra = {k: int(v) for k, v in (kv.split("=") for kv in a.extra.split(",") if kv)}
    if a.app in ("bfs-mesh", "bfs-road"):
        g = gen.mesh(a.side, a.side, 0.6 if a.app == "bfs-road" else 1.0, 2, device="cuda")
        src = gen.mesh_centre_source(g, a.side, a.side)
    elif a.app == "bfs-rmat":
        g = gen.rmat(a.scale or 26, 16, 5, device="cuda")
        srcs = [gen.pick_source(g, 105 + i) for i in range(a.sources)]
        src = srcs[0]
    elif a.app == "pr":
        g = gen.rmat(a.scale or 22, 16, 3, device="cuda")
        src = None
    else:
        g = gen.rmat(a.scale or 20, 64, 4, device="cuda")
        src = None
    csr = atos.CSR.from_graph(g, layout=a.layout)
    n, m = g.n, g.m
    del g
    torch.cuda.empty_cache()
    print(f"# {a.app} n={n} m={m}", flush=True)
    grid = (a.grid or DEFAULT_GRID[a.app]).split(",")
    for spec in grid:
        w, f, p = (int(x) for x in spec.split(":"))
        knobs = dict(worker=w, fetch_size=f, persistent=p, timeout_s=20, **extra)
        ms, wms, st = [], [], None
        try:
            for it in range(a.reps + 1):
                if a.app == "bfs-rmat":
                    _, st = atos.bfs(csr, srcs[it % len(srcs)], **knobs)
                elif a.app.startswith("bfs"):
                    _, st = atos.bfs(csr, src, **knobs)
                elif a.app == "pr":
                    _, st = atos.pagerank(csr, 0.85, 1e-6, **knobs)
                else:
                    _, st = atos.color(csr, 1, **knobs)
                ms.append(st["kernel_ms"])
                wms.append(st["worker_ms"])
        except RuntimeError as e:
            print(f"{spec:>14}  ERROR {e}", flush=True)
            continue
        ms, wms = ms[1:], wms[1:]
        print(f"{spec:>14}  ms med {np.median(ms):9.3f} min {np.min(ms):9.3f}  worker {np.median(wms):9.3f}  "
              f"pops/n {st['pops'] / n:7.3f}  edges/m {st['edges'] / m:7.3f}  rounds {st['rounds']}"
              + (f"  colors {st['colors_used']}" if a.app == "gc" else ""), flush=True)


if __name__ == "__main__":
    main()
