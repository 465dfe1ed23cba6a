"""Normalized throughput vs time (Figs. 1-3; definition) on the synthetic configs.

  python tools/normalized_tp.py bfs|pr|gc [--scale S] [--ef EF] [--rows R]

Runs the Atos call with cfg.timeline, the in-framework BSP baseline for the overwork factor (BFS /
PageRank; colouring uses |V|), and prints R rows of (t_ms, raw tasks/us, normalized tasks/us)."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_icpp_chenbpbyo22_b200 as atos  # noqa: E402
from paper_conf_icpp_chenbpbyo22_b200 import analysis, gen  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("app")
    ap.add_argument("--scale", type=int, default=None)
    ap.add_argument("--ef", type=int, default=None)
    ap.add_argument("--rows", type=int, default=20)
    ap.add_argument("--mesh", type=int, default=0, help="BFS on an N x N mesh instead of RMAT")
    a = ap.parse_args()
    if a.mesh:
        g = gen.mesh(a.mesh, a.mesh, device="cuda")
        src = gen.mesh_centre_source(g, a.mesh, a.mesh)
    else:
        scale = a.scale or {"bfs": 26, "pr": 22, "gc": 20}[a.app]
        ef = a.ef or (64 if a.app == "gc" else 16)
        g = gen.rmat(scale, ef, {"bfs": 5, "pr": 3, "gc": 4}[a.app], device="cuda")
        src = gen.pick_source(g, 105)
    csr = atos.CSR.from_graph(g)
    cap = 1 << 16
    tl = torch.zeros(4 * cap, dtype=torch.int64, device="cuda")
    run = {"bfs": lambda **k: atos.bfs(csr, src, **k), "pr": lambda **k: atos.pagerank(csr, 0.85, 1e-6, **k),
           "gc": lambda **k: atos.color(csr, 1, **k)}[a.app]
    bsp = {"bfs": lambda: atos.bfs_bsp(csr, src), "pr": lambda: atos.pagerank_bsp(csr, 0.85, 1e-6),
           "gc": None}[a.app]
    run()
    _, st = run(timeline=tl, timeline_interval_ns=20000)
    sb = bsp()[1] if bsp else None
    ow = analysis.overwork_factor(a.app, st["pops"], bsp_pops=sb["pops"] if sb else None, n=g.n)
    tab = atos.timeline_table(tl, st).numpy().astype(np.float64)
    t, tp = analysis.throughput_series(tab)
    _, nt = analysis.normalized_throughput(tab, ow)
    print(f"# {a.app} n={g.n} m={g.m} tasks={st['pops']} bsp_tasks={sb['pops'] if sb else None} overwork={ow:.3f} "
          f"kernel_ms={st['kernel_ms']:.3f} samples={len(tab)}")
    print("#   t_ms   tasks/us  normalized/us")
    idx = sorted(set(int(i * (len(t) - 1) / max(1, a.rows - 1)) for i in range(a.rows))) if len(t) else []
    for i in idx:
        print(f"{t[i] / 1e3:8.3f} {tp[i]:10.1f} {nt[i]:10.1f}")


if __name__ == "__main__":
    main()
