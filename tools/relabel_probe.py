"""Probe (tools only): the same RMAT graph with vertex ids relabelled by descending degree (hubs packed at
low ids, so their per-vertex state shares L2 lines) vs the generator's random permutation."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_icpp_chenbpbyo22_b200 as atos  # noqa: E402
from paper_conf_icpp_chenbpbyo22_b200 import gen  # noqa: E402


def relabel(g, spread=0):
    """rank r by descending degree -> new id r, or with spread T: ranks r < 16T go to
    (r % T) * 16 + r // T (the top T vertices on T distinct 128-B lines of an f64 array)."""
    deg = g.row_ptr[1:] - g.row_ptr[:-1]
    rank_order = torch.argsort(deg, descending=True, stable=True)  # rank r -> old id
    pos = torch.arange(g.n, device=deg.device)
    if spread:
        T = spread
        r = pos[:16 * T]
        pos[:16 * T] = (r % T) * 16 + r // T
    order = torch.empty_like(rank_order)
    order[pos] = rank_order  # new id i -> old id order[i]
    newid = torch.empty_like(order)
    newid[order] = torch.arange(g.n, device=order.device)
    ndeg = deg[order]
    rp = torch.zeros(g.n + 1, dtype=torch.int64, device=order.device)
    rp[1:] = torch.cumsum(ndeg, 0)
    # gather rows in new order
    src_start = g.row_ptr[:-1][order]
    idx = torch.repeat_interleave(src_start - rp[:-1], ndeg) + torch.arange(g.m, device=order.device)
    col = newid[g.col[idx].long()].to(torch.int32)
    return gen.Graph(g.n, g.m, rp, col, g.name + "-deg"), newid


def main():
    scale = int(sys.argv[1]) if len(sys.argv) > 1 else 26
    seed = int(sys.argv[2]) if len(sys.argv) > 2 else 5
    g = gen.rmat(scale, 16, seed, device="cuda")
    src = gen.pick_source(g, 105)
    runs = [("random-ids", g, src)]
    for sp in (0, 1 << 14, 1 << 16):
        h, newid = relabel(g, sp)
        runs.append((f"deg-sp{sp}", h, int(newid[src])))
    for name, gg, s in runs:
        csr = atos.CSR.from_graph(gg)
        for app in ("bfs", "pr"):
            ms = []
            for _ in range(3):
                if app == "bfs":
                    _, st = atos.bfs(csr, s)
                else:
                    _, st = atos.pagerank(csr, 0.85, 1e-6)
                ms.append(st["kernel_ms"])
            print(f"{name:10s} {app:3s} ms {min(ms[1:]):9.2f}  pops/n {st['pops'] / g.n:.3f}  edges/m {st['edges'] / g.m:.3f}",
                  flush=True)
        csr.close()
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
