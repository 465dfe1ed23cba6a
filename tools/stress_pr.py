"""Stress the PageRank path with a given knob set; report failure modes."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import oracle
import paper_conf_icpp_chenbpbyo22_b200 as atos
from paper_conf_icpp_chenbpbyo22_b200 import gen

args = dict(a.split("=") for a in sys.argv[1:])
reps = int(args.pop("reps", 30))
scale = int(args.pop("scale", 13))
knobs = {k: int(v) for k, v in args.items()}
g = gen.rmat(scale, 16, seed=11)
rp, ci = g.numpy()
ref, _, _ = oracle.pagerank_jacobi(rp, ci, 0.85)
csr = atos.CSR.from_graph(g.to("cuda"))
n = g.n
iso = int((np.diff(rp) == 0).sum())
bad = 0
for i in range(reps):
    try:
        r, st = atos.pagerank(csr, 0.85, 1e-6, timeout_s=5.0, **knobs)
    except RuntimeError as e:
        print("rep", i, "ERROR", e); bad += 1; continue
    x, xs = r.cpu().numpy() * n, ref * n
    over = np.max(x - xs * (1 + 1e-9))
    under = np.max(xs - x - 1e-6 * xs / 0.15 * (1 + 1e-6))
    cons = x.sum() + st["residual_sum"] / 0.15 - (n - 0.85 * iso)
    if over > 1e-12 or under > 1e-12 or abs(cons) > 1e-9 * n:
        bad += 1
        print(f"rep {i}: over={over:.3e} under={under:.3e} cons={cons:.3e} pops={st['pops']} argmax_over={int(np.argmax(x - xs))}")
print(f"{bad}/{reps} bad", knobs)
