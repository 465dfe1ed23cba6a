"""PageRank threshold schedule on ONE partition (tools only): the round protocol with a 1-rank
communicator runs local phases to quiescence at eps_k = max(eps, eps0 * f^k) (ATOS_PR_EPS0 / ATOS_PR_EPSF),
re-seeding between phases -- compared with the plain single-partition call on the same graph.

  python tools/pr_sched.py [--scale 22] [--seed 3]
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
    ap.add_argument("--scale", type=int, default=22)
    ap.add_argument("--seed", type=int, default=3)
    ap.add_argument("--reps", type=int, default=2)
    a = ap.parse_args()
    g = gen.rmat(a.scale, 16, a.seed, device="cuda")
    csr = atos.CSR.from_graph(g)
    comm = atos.Comm(1, 0, atos.Comm.unique_id(), 0)
    part = comm.partition(g.n, 0, g.n, g.row_ptr, g.col)
    ref = None
    for name, c in (("single", csr), ("rounds", part)):
        ms = []
        for _ in range(a.reps + 1):
            r, st = atos.pagerank(c, 0.85, 1e-6)
            torch.cuda.synchronize()
            ms.append(st["kernel_ms"])
        if ref is None:
            ref = r.clone()
        l1 = (r - ref).abs().sum().item()
        print(f"{name:7s} eps0={os.environ.get('ATOS_PR_EPS0', 'default')} f={os.environ.get('ATOS_PR_EPSF', '-')}"
              f"  ms {min(ms[1:]):9.2f}  rounds {st['rounds']}  pops/n {st['pops'] / g.n:.3f}"
              f"  edges/m {st['edges'] / g.m:.3f}  L1 vs single {l1:.3e}  resid {st['residual_sum']:.6e}", flush=True)


if __name__ == "__main__":
    main()
