"""C5 (RMAT S26) BFS / PageRank: single partition vs P loopback partitions on one GPU (tools only).

  python tools/part_scan.py [--scale 26] [--parts 1,2,4,8] [--apps bfs,pr] [--reps 2]

Prints ms (stats.kernel_ms, CUDA events inside the library), rounds and bytes exchanged per run,
and checks every partitioned result against the single-partition one (BFS equal, PageRank L1).
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_icpp_chenbpbyo22_b200 as atos  # noqa: E402
from paper_conf_icpp_chenbpbyo22_b200 import gen  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--scale", type=int, default=26)
    ap.add_argument("--parts", default="1,2,4,8")
    ap.add_argument("--apps", default="bfs,pr")
    ap.add_argument("--reps", type=int, default=2)
    a = ap.parse_args()
    g = gen.rmat(a.scale, 16, 5, device="cuda")
    src = gen.pick_source(g, 105)
    print(f"# rmat S{a.scale} n={g.n} m={g.m} src={src}", flush=True)
    ref = {}
    for P in [int(x) for x in a.parts.split(",")]:
        csr = atos.CSR.from_graph(g, num_parts=P)
        for app in a.apps.split(","):
            ms = []
            for _ in range(a.reps + 1):
                if app == "bfs":
                    out, st = atos.bfs(csr, src)
                else:
                    out, st = atos.pagerank(csr, 0.85, 1e-6)
                torch.cuda.synchronize()
                ms.append(st["kernel_ms"])
            ms = ms[1:] or ms
            chk = ""
            if app not in ref:
                ref[app] = out.clone()
            elif app == "bfs":
                chk = "equal" if torch.equal(out, ref[app]) else "MISMATCH"
            else:
                chk = f"L1 {(out - ref[app]).abs().sum().item():.3e}"
            print(f"{app:4s} P={P}  ms min {min(ms):9.2f} med {sorted(ms)[len(ms) // 2]:9.2f}  rounds {st['rounds']}"
                  f"  bytes_exch {st['bytes_exchanged']}  pops/n {st['pops'] / g.n:.3f}  edges/m {st['edges'] / g.m:.3f}"
                  f"  {chk}", flush=True)
        csr.close()
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
