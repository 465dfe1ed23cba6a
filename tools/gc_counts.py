"""Colouring overwork by degree bucket (tools only): needs a -DATOS_GC_COUNTS build (tools/ab.py build gccnt
-DATOS_GC_COUNTS) selected with ATOS_LIB.  python tools/gc_counts.py [scale] [ef] [knob=v ...]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_icpp_chenbpbyo22_b200 as atos  # noqa: E402
from paper_conf_icpp_chenbpbyo22_b200 import gen  # noqa: E402


def main():
    scale = int(sys.argv[1]) if len(sys.argv) > 1 else 20
    ef = int(sys.argv[2]) if len(sys.argv) > 2 else 64
    knobs = {k: int(v) for k, v in (a.split("=") for a in sys.argv[3:])}
    g = gen.rmat(scale, ef, 4, device="cuda")
    csr = atos.CSR.from_graph(g)
    deg = g.degrees().cpu().numpy()
    path = "/tmp/gc_counts.bin"
    os.environ["ATOS_GC_COUNTS"] = path
    c, st = atos.color(csr, 1, **knobs)
    cnt = np.fromfile(path, dtype=np.uint32).reshape(-1, 2)
    m = g.m
    print(f"n={g.n} m={m} colours={st['colors_used']} tasks/n={st['pops']/g.n:.3f} edges/m={st['edges']/m:.3f} "
          f"ms={st['kernel_ms']:.3f} knobs={knobs}")
    print(" degree bucket      verts   assigns/v  checks/v   edge-visit share   max assigns")
    order = np.argsort(-deg)
    edges_tot = float((cnt[:, 0] + cnt[:, 1]).astype(np.float64) @ deg)
    lo = 0
    for hi in (16, 128, 1024, 8192, 65536, len(order)):
        hi = min(hi, len(order))
        if hi <= lo:
            continue
        idx = order[lo:hi]
        a, k = cnt[idx, 0].astype(np.float64), cnt[idx, 1].astype(np.float64)
        share = float((a + k) @ deg[idx]) / edges_tot
        print(f" top[{lo:7d},{hi:7d}) deg {deg[idx].min():6d}-{deg[idx].max():6d}  {len(idx):7d}  {a.mean():8.2f}  "
              f"{k.mean():8.2f}   {share:8.3f}          {int(a.max())}")
        lo = hi


if __name__ == "__main__":
    main()
