"""NEXT-3 colouring ordering study: vertex-ID order vs seeded permutation of the
initial queue (permute_init), on a Kronecker graph with its NATURAL ids (hubs at low ids: the analogue of
the paper's semantically ordered web-crawl ids) and with permuted ids (the default recipe), for the
persistent and discrete kernels with warp and CTA workers.

  python tools/gc_order_study.py [--scale 20] [--ef 64] [--reps 3]
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_icpp_chenbpbyo22_b200 as atos  # noqa: E402
from paper_conf_icpp_chenbpbyo22_b200 import gen  # noqa: E402

VARIANTS = [("persist-CTA", dict(worker=1024, fetch_size=128, persistent=1)),
            ("persist-warp", dict(worker=32, fetch_size=8, persistent=1)),
            ("discrete-warp", dict(worker=32, fetch_size=8, persistent=0)),
            ("discrete-CTA", dict(worker=1024, fetch_size=128, persistent=0))]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--scale", type=int, default=20)
    ap.add_argument("--ef", type=int, default=64)
    ap.add_argument("--reps", type=int, default=3)
    a = ap.parse_args()
    print("graph_ids    kernel          permute_init      ms  colours  tasks/n  edges/m")
    for ids, permute in (("natural", False), ("permuted", True)):
        g = gen.rmat(a.scale, a.ef, 4, device="cuda", permute=permute)
        csr = atos.CSR.from_graph(g)
        n, m = g.n, g.m
        for name, knobs in VARIANTS:
            for pi in (0, 1):
                ms, st = [], None
                try:
                    for _ in range(a.reps + 1):
                        _, st = atos.color(csr, 1, permute_init=pi, timeout_s=60, **knobs)
                        ms.append(st["kernel_ms"])
                except RuntimeError as e:
                    print(f"{ids:12s} {name:15s} {pi:12d}  ERROR {e}", flush=True)
                    continue
                print(f"{ids:12s} {name:15s} {pi:12d} {np.median(ms[1:]):8.2f} {st['colors_used']:8d} "
                      f"{st['pops'] / n:8.3f} {st['edges'] / m:8.3f}", flush=True)
        del csr, g
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
