"""Unloaded per-hop latency of the queue chain: BFS on a path graph (one vertex per level), so every level
is one publish -> claim -> gather -> begin -> expand -> publish round with nothing else running.
  python tools/hop_latency.py [n] -- prints ms, levels and us/level per worker configuration (tools only)"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_icpp_chenbpbyo22_b200 as atos  # noqa: E402
from paper_conf_icpp_chenbpbyo22_b200 import gen  # noqa: E402


def main():
    n = int(sys.argv[1]) if len(sys.argv) > 1 else 20000
    src = torch.arange(n - 1, dtype=torch.int64)
    g = gen.csr_from_edges(n, src, src + 1, symmetric=True)
    csr = atos.CSR(g.row_ptr.cuda(), g.col.cuda(), layout="input")
    for kn in (dict(), dict(worker=256, fetch_size=256, num_blocks=148), dict(worker=256, fetch_size=256, num_blocks=1),
               dict(worker=32, fetch_size=8), dict(worker=32, fetch_size=8, num_blocks=1), dict(persistent=0)):
        atos.bfs(csr, 0, **kn)
        ms = []
        for _ in range(3):
            d, st = atos.bfs(csr, 0, **kn)
            ms.append(st["worker_ms"])
        m = min(ms)
        print(f"{str(kn):70s} worker ms {m:8.3f}  levels {n - 1}  us/level {1e3 * m / (n - 1):7.3f}  "
              f"rounds {st['rounds']} flags {st['flags']}", flush=True)


if __name__ == "__main__":
    main()
