"""Probe (tools only): does sorting each adjacency row by the degree layout's new ids help the C5 BFS?
Builds the degree-relabelled graph in torch -- ids by descending degree -- once with rows in the
generator's (old-id) order and once with every row sorted by new id, creates both with layout="input"
(the library keeps them as given) and times the BFS from the bench's 8 sources (L2 flushed before each)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_icpp_chenbpbyo22_b200 as atos  # noqa: E402
from paper_conf_icpp_chenbpbyo22_b200 import gen  # noqa: E402


def main():
    scale = int(sys.argv[1]) if len(sys.argv) > 1 else 26
    g = gen.rmat(scale, 16, 5, device="cuda")
    n = g.n
    srcs = [gen.pick_source(g, 105 + i) for i in range(8)]
    deg = (g.row_ptr[1:] - g.row_ptr[:-1])
    order = torch.argsort(deg, descending=True, stable=True)     # new id -> old id
    o2n = torch.empty_like(order)
    o2n[order] = torch.arange(n, device="cuda", dtype=order.dtype)
    ndeg = deg[order]
    nrp = torch.zeros(n + 1, dtype=torch.int64, device="cuda")
    nrp[1:] = torch.cumsum(ndeg, 0)
    # gather rows in new order (old-id order inside each row), then map the column ids
    rows = torch.repeat_interleave(torch.arange(n, device="cuda"), ndeg)          # new row of each new edge
    old_start = g.row_ptr[:-1][order]
    pos = torch.arange(int(nrp[-1]), device="cuda", dtype=torch.int64) - nrp[:-1][rows] + old_start[rows]
    del rows, old_start
    ncol = o2n[g.col[pos].long()].int()
    del pos
    res = {}
    # the library's own degree layout on the caller's ids (mapped output pass included)
    csr = atos.CSR.from_graph(g)
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    ms, wms = [], []
    for rnd in range(3):
        for s in srcs:
            flush.fill_(rnd)
            torch.cuda.synchronize()
            d, st = atos.bfs(csr, s)
            if rnd:
                ms.append(st["kernel_ms"])
                wms.append(st["worker_ms"])
    print("library", csr.layout, "ms per BFS", round(sum(ms) / len(ms), 3), "worker", round(sum(wms) / len(wms), 3),
          flush=True)
    csr.close()
    del flush
    for tag in ("unsorted", "sorted"):
        if tag == "sorted":
            rows = torch.repeat_interleave(torch.arange(n, device="cuda"), ndeg)
            key = rows * n + ncol.long()
            del rows
            key, _ = torch.sort(key)
            ncol = (key % n).int()
            del key
        torch.cuda.empty_cache()
        csr = atos.CSR(nrp, ncol, layout="input")
        flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
        ms, wms = [], []
        for rnd in range(3):
            for s in srcs:
                flush.fill_(rnd)
                torch.cuda.synchronize()
                d, st = atos.bfs(csr, int(o2n[s]))
                if rnd:
                    ms.append(st["kernel_ms"])
                    wms.append(st["worker_ms"])
        res[tag] = sum(ms) / len(ms)
        print(tag, "ms per BFS", round(res[tag], 3), "worker", round(sum(wms) / len(wms), 3), flush=True)
        if tag == "unsorted":
            break
        csr.close()
        del flush
    print(res)


if __name__ == "__main__":
    main()
