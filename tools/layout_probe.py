"""Probe (tools only): the degree layout's hub interleave width T (ATOS_LAYOUT_T) against C5 BFS (8 bench
sources, L2 flushed) and C5 PageRank, one CSR per T.  python tools/layout_probe.py T1,T2,... [scale]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_icpp_chenbpbyo22_b200 as atos  # noqa: E402
from paper_conf_icpp_chenbpbyo22_b200 import gen  # noqa: E402


def main():
    Ts = sys.argv[1].split(",")
    scale = int(sys.argv[2]) if len(sys.argv) > 2 else 26
    pr = int(os.environ.get("PROBE_PR", "1"))
    g = gen.rmat(scale, 16, 5, device="cuda")
    srcs = [gen.pick_source(g, 105 + i) for i in range(8)]
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    for rnd in range(2):
        for T in Ts:
            os.environ["ATOS_LAYOUT_T"] = T
            csr = atos.CSR.from_graph(g)
            ms, wms = [], []
            for k in range(2):
                for s in srcs:
                    flush.fill_(k)
                    torch.cuda.synchronize()
                    d, st = atos.bfs(csr, s)
                    if k:
                        ms.append(st["kernel_ms"])
                        wms.append(st["worker_ms"])
            line = f"round {rnd} T={T:>6s} {csr.layout} bfs ms {sum(ms) / len(ms):7.3f} worker {sum(wms) / len(wms):7.3f}"
            if pr:
                flush.fill_(3)
                torch.cuda.synchronize()
                r, st = atos.pagerank(csr, 0.85, 1e-6)
                line += f"  pr ms {st['kernel_ms']:8.1f}"
            print(line, flush=True)
            csr.close()
            torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
