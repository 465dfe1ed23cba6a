"""Per-BFS-level work profile of a generated graph: vertices, edges (sum of degrees) and max degree per level
(explains where a traversal's time goes; run on the GPU box).  python tools/level_stats.py [scale] [src_seed]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_icpp_chenbpbyo22_b200 as atos  # noqa: E402
from paper_conf_icpp_chenbpbyo22_b200 import gen  # noqa: E402

scale = int(sys.argv[1]) if len(sys.argv) > 1 else 26
sseed = int(sys.argv[2]) if len(sys.argv) > 2 else 105
g = gen.rmat(scale, 16, 5, device="cuda")
csr = atos.CSR.from_graph(g)
src = gen.pick_source(g, sseed)
d, st = atos.bfs(csr, src)
deg = g.degrees()
print(f"n={g.n} m={g.m} src={src} deg(src)={int(deg[src])} ms={st['kernel_ms']:.2f}")
L = int(d[d != -1].max().item())
cum = 0
for lv in range(L + 1):
    mask = d == lv
    nv = int(mask.sum().item())
    de = deg[mask]
    e = int(de.sum().item())
    cum += e
    big = int((de > 4096).sum().item())
    ebig = int(de[de > 4096].sum().item()) if big else 0
    print(f"level {lv}: vertices {nv:>10} edges {e:>11} ({100 * e / g.m:5.1f}%, cum {100 * cum / g.m:5.1f}%) "
          f"max deg {int(de.max().item()) if nv else 0:>8}  deg>4096: {big} vertices {ebig} edges")
# degree distribution of reached vertices
dr = deg[d != -1].float()
for q in (0.5, 0.9, 0.99, 0.999):
    print(f"deg quantile {q}: {torch.quantile(dr[:10_000_000], q).item():.0f}")
for t in (16, 64, 256, 1024, 4096, 65536):
    sel = deg[d != -1] > t
    print(f"deg > {t}: {int(sel.sum())} vertices, {int(deg[d != -1][sel].sum()) / g.m * 100:.1f}% of edges")
