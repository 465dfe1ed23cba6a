"""One barrier-free PageRank call on C3 with P loopback partitions (for ncu): python tools/nb_one.py [P] [scale]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_chenbpbyo22_b200 as atos  # noqa: E402
from paper_conf_icpp_chenbpbyo22_b200 import gen  # noqa: E402

P = int(sys.argv[1]) if len(sys.argv) > 1 else 4
scale = int(sys.argv[2]) if len(sys.argv) > 2 else 22
g = gen.rmat(scale, 16, 3, device="cuda")
pc = atos.CSR.from_graph(g, num_parts=P)
r, st = atos.pagerank(pc, 0.85, 1e-6, barrier_free=1)
print({k: st[k] for k in ("kernel_ms", "worker_ms", "pops", "edges")})
