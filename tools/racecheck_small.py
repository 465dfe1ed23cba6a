"""Small launches for compute-sanitizer racecheck (tools only): few CTAs, tiny graphs, every worker mode."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import paper_conf_icpp_chenbpbyo22_b200 as atos  # noqa: E402
from paper_conf_icpp_chenbpbyo22_b200 import gen  # noqa: E402

g = gen.rmat(9, 8, seed=3)
rp, ci = g.numpy()
csr = atos.CSR.from_graph(g.to("cuda"), layout="degree")
src = gen.pick_source(g, 1)
for knobs in (dict(worker=256, fetch_size=256), dict(worker=32, fetch_size=4), dict(worker=1, fetch_size=2),
              dict(worker=256, fetch_size=256, persistent=0)):
    d, _ = atos.bfs(csr, src, num_blocks=4, **knobs)
    assert np.array_equal(d.cpu().numpy().view(np.uint32), oracle.bfs(rp, ci, src)), knobs
    r, _ = atos.pagerank(csr, 0.85, 1e-4, num_blocks=4, **knobs)
    c, _ = atos.color(csr, 1, num_blocks=2, **({} if knobs.get("worker") == 1 else knobs))
    assert oracle.validate_color(rp, ci, c.cpu().numpy()) == 0
print("racecheck_small ok", flush=True)
