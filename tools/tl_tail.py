"""Print the end of the progress timeline of slow BFS runs (tools only)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_icpp_chenbpbyo22_b200 as atos
from paper_conf_icpp_chenbpbyo22_b200 import gen
g = gen.rmat(26, 16, 5, device="cuda")
csr = atos.CSR.from_graph(g)
src = gen.pick_source(g, 105)
deg = g.degrees()
for rep in range(10):
    tl = torch.zeros(4 * 20000, dtype=torch.int64, device="cuda")
    d, st = atos.bfs(csr, src, timeline=tl)
    t = atos.timeline_table(tl, st)
    print(f"rep {rep}: worker_ms {st['worker_ms']:.2f} samples {t.shape[0]} maxdepth {int((d[d >= 0]).max())}")
    if st["worker_ms"] > 20.5:
        n = t.shape[0]
        # print samples in the last 3 ms, every 10th
        tend = t[-1, 0].item()
        sel = [i for i in range(n) if t[i, 0].item() > tend - 3.0e6][::8]
        for i in sel:
            print(f"   {t[i,0].item()/1e3:9.1f} us  done {t[i,1].item()-t[0,1].item():10d}  tail {t[i,2].item()-t[0,1].item():10d}  head {t[i,3].item()-t[0,1].item():10d}")
        # depth histogram of vertices
        h = torch.bincount(d[d >= 0].long())
        print("   depth histogram:", h.tolist())
        break
