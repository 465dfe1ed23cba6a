"""A/B of RUNTIME environment knobs of libatos in one process (tools only).

  python tools/env_ab.py bfs-rmat|bfs-mesh|bfs-road|pr|gc --var ATOS_HUB_CACHE --values 0,8192,16384 \
                         [--scale S] [--rounds 5] [--sources 8]

The graph is built once; the settings are interleaved round by round (clock drift hits all alike) with a
512 MiB L2 flush before every call.  Prints per setting the median device ms (stats.kernel_ms) and worker ms,
and checks that every setting returns the same BFS depths as the first one (bit-exact) / the same colour
validity / PageRank ranks within 1e-6 relative of the first."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_icpp_chenbpbyo22_b200 as atos  # noqa: E402
from paper_conf_icpp_chenbpbyo22_b200 import gen  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("app")
    ap.add_argument("--var", required=True)
    ap.add_argument("--values", required=True)
    ap.add_argument("--scale", type=int, default=None)
    ap.add_argument("--rounds", type=int, default=5)
    ap.add_argument("--sources", type=int, default=8)
    ap.add_argument("--side", type=int, default=4900)
    ap.add_argument("--layout", default="auto")
    a = ap.parse_args()
    vals = a.values.split(",")
    if a.app in ("bfs-mesh", "bfs-road"):
        g = gen.mesh(a.side, a.side, 0.6 if a.app == "bfs-road" else 1.0, 2, device="cuda")
        srcs = [gen.mesh_centre_source(g, a.side, a.side)]
    elif a.app == "bfs-rmat":
        g = gen.rmat(a.scale or 26, 16, 5, device="cuda")
        srcs = [gen.pick_source(g, 105 + i) for i in range(a.sources)]
    elif a.app == "pr":
        g = gen.rmat(a.scale or 22, 16, 3, device="cuda")
        srcs = [None]
    else:
        g = gen.rmat(a.scale or 20, 64, 4, device="cuda")
        srcs = [None]
    csr = atos.CSR.from_graph(g, layout=a.layout)
    n, m = g.n, g.m
    del g
    torch.cuda.empty_cache()
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    print(f"# {a.app} n={n} m={m} layout={csr.layout if hasattr(csr, 'layout') else '?'} {a.var} in {vals}",
          flush=True)
    ms = {v: [] for v in vals}
    wk = {v: [] for v in vals}
    ref = {}
    bad = {v: 0 for v in vals}
    for rnd in range(a.rounds):
        for v in vals:
            os.environ[a.var] = v
            tot, wtot = 0.0, 0.0
            for i, s in enumerate(srcs):
                flush.fill_(rnd & 0xFF)
                torch.cuda.synchronize()
                if a.app.startswith("bfs"):
                    out, st = atos.bfs(csr, s)
                elif a.app == "pr":
                    out, st = atos.pagerank(csr, 0.85, 1e-6)
                else:
                    out, st = atos.color(csr, 1)
                torch.cuda.synchronize()
                tot += st["kernel_ms"]
                wtot += st.get("worker_ms", 0.0)
                if rnd == 0:
                    if i not in ref:
                        ref[i] = out.clone()
                    elif a.app.startswith("bfs"):
                        bad[v] += int(not torch.equal(out, ref[i]))
                    elif a.app == "pr":
                        rel = ((out - ref[i]).abs() / ref[i].abs().clamp_min(1e-300)).max().item()
                        bad[v] += int(rel > 1e-4)
            ms[v].append(tot)
            wk[v].append(wtot)
            print(f"round {rnd} {a.var}={v:>8s} ms {tot:9.3f} worker {wtot:9.3f} rounds {st.get('rounds')} "
                  f"pops {st.get('pops')} edges {st.get('edges')} colours {st.get('colors_used')}", flush=True)
    print(f"# {a.var}: median over {a.rounds} rounds of the summed device ms over {len(srcs)} call(s)")
    for v in vals:
        print(f"{a.var}={v:>8s} ms {np.median(ms[v]):9.3f} worker {np.median(wk[v]):9.3f} "
              f"min {np.min(ms[v]):9.3f} mismatches_vs_first {bad[v]}", flush=True)


if __name__ == "__main__":
    main()
