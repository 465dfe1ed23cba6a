"""Barrier-free vs exchange-round partitioned PageRank on C3 (RMAT S22 EF16 seed 3), loopback partitions.

python tools/nb_ab.py [scale]  -- prints one line per (P, protocol): device ms, worker ms, edge relaxations/m,
pops/n and the L1 distance of rank/n to the single-partition result."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_icpp_chenbpbyo22_b200 as atos  # noqa: E402
from paper_conf_icpp_chenbpbyo22_b200 import gen  # noqa: E402


def main():
    scale = int(sys.argv[1]) if len(sys.argv) > 1 else 22
    bfs_only = len(sys.argv) > 2 and sys.argv[2] == "bfs"
    g = gen.rmat(scale, 16, 3, device="cuda")
    one = atos.CSR.from_graph(g)
    if not bfs_only:
        ref, st = atos.pagerank(one, 0.85, 1e-6)
        ref, st = atos.pagerank(one, 0.85, 1e-6)
        print(f"single: {st['kernel_ms']:.1f} ms edges/m {st['edges'] / g.m:.1f} pops/n {st['pops'] / g.n:.1f}",
              flush=True)
    one.close()
    for P in (2, 4, 8):
        pc = atos.CSR.from_graph(g, num_parts=P)
        for bf in (() if bfs_only else (0, 1)):
            for _ in range(2):
                r, st = atos.pagerank(pc, 0.85, 1e-6, barrier_free=bf)
            torch.cuda.synchronize()
            l1 = float((r - ref).abs().sum().item())
            print(f"P={P} {'barrier_free' if bf else 'rounds      '}: {st['kernel_ms']:8.1f} ms  worker "
                  f"{st['worker_ms']:8.1f} ms  edges/m {st['edges'] / g.m:6.1f}  pops/n {st['pops'] / g.n:5.1f}  "
                  f"rounds {st['rounds']}  l1 {l1:.2e}", flush=True)
        src = gen.pick_source(g, 105)
        for bf in (0, 1):
            for _ in range(2):
                d, st = atos.bfs(pc, src, barrier_free=bf)
            torch.cuda.synchronize()
            print(f"P={P} BFS {'barrier_free' if bf else 'rounds      '}: {st['kernel_ms']:8.2f} ms  edges/m "
                  f"{st['edges'] / g.m:5.2f}  rounds {st['rounds']}", flush=True)
        pc.close()


if __name__ == "__main__":
    main()
