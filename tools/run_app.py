"""Run one app once (for ncu captures): python tools/run_app.py bfs|pr|gc --scale S [--ef EF] [knob=value ...]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_icpp_chenbpbyo22_b200 as atos  # noqa: E402
from paper_conf_icpp_chenbpbyo22_b200 import gen  # noqa: E402


def main():
    app = sys.argv[1]
    args = dict(a.split("=") for a in sys.argv[2:] if "=" in a)
    scale = int(args.pop("scale", 22))
    ef = int(args.pop("ef", 16))
    seed = int(args.pop("seed", {"bfs": 5, "pr": 3, "gc": 4}[app]))
    reps = int(args.pop("reps", 1))
    tl = int(args.pop("timeline", 0))
    knobs = {k: int(v) for k, v in args.items() if k not in ("mesh", "keep")}
    mesh = int(args.pop("mesh", 0))
    if mesh:
        g = gen.mesh(mesh, mesh, float(args.pop("keep", 1.0)), 2, device="cuda")
        csr = atos.CSR.from_graph(g)
        src = gen.mesh_centre_source(g, mesh, mesh)
    else:
        g = gen.rmat(scale, ef, seed, device="cuda")
        csr = atos.CSR.from_graph(g)
        src = gen.pick_source(g, 105)
    if args.pop("free_graph", None) or True:
        # keep only what the solver needs on the device (smaller ncu replay backups)
        stats = g.stats()
        g = gen.Graph(g.n, g.m, g.row_ptr[:1], g.col[:1], g.name)
        torch.cuda.empty_cache()
    torch.cuda.synchronize()
    print(stats, flush=True)
    for _ in range(reps):
        if tl:
            knobs["timeline"] = torch.zeros(4 * tl, dtype=torch.int64, device="cuda")
        if app == "bfs":
            d, st = atos.bfs(csr, src, **knobs)
        elif app == "pr":
            d, st = atos.pagerank(csr, 0.85, 1e-6, **knobs)
        else:
            d, st = atos.color(csr, 1, **knobs)
        tlb = knobs.pop("timeline", None)
        print(app, scale, knobs, {k: (round(v, 3) if isinstance(v, float) else v) for k, v in st.items()}, flush=True)
        if tlb is not None:
            t = atos.timeline_table(tlb, st)
            n = t.shape[0]
            nrow = int(os.environ.get("TL_ROWS", "25"))
            idx = sorted(set([int(i * (n - 1) / (nrow - 1)) for i in range(nrow)])) if n else []
            print("  t_us      done        tail        head")
            for i in idx:
                print(f"  {t[i,0].item()/1e3:8.1f} {t[i,1].item():11d} {t[i,2].item():11d} {t[i,3].item():11d}")


if __name__ == "__main__":
    main()
