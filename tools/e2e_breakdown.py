"""Where the end-to-end (host buffers) time of one C5 BFS goes: handle creation (H2D + device narrowing +
checks), the solver call with a host output (D2H), and destroy.  Tools only."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_icpp_chenbpbyo22_b200 as atos
from paper_conf_icpp_chenbpbyo22_b200 import gen
g = gen.rmat(int(sys.argv[1]) if len(sys.argv) > 1 else 26, 16, 5, device="cuda")
src = gen.pick_source(g, 105)
rp = g.row_ptr.cpu().pin_memory()
ci = g.col.cpu().pin_memory()
out = torch.empty(g.n, dtype=torch.int32).pin_memory()
del g
torch.cuda.empty_cache()
t = time.perf_counter(); x = torch.empty_like(ci, device="cuda"); x.copy_(ci); torch.cuda.synchronize()
print(f"raw H2D of col ({ci.numel() * 4 / 1e9:.2f} GB): {1e3 * (time.perf_counter() - t):.1f} ms")
del x
torch.cuda.empty_cache()
for k in range(int(os.environ.get("E2E_STEPS", "4"))):
    t0 = time.perf_counter()
    csr = atos.CSR(rp, ci, device=0)
    t1 = time.perf_counter()
    _, st = atos.bfs(csr, src, out=out)
    t2 = time.perf_counter()
    csr.close()
    t3 = time.perf_counter()
    print(f"step {k}: create {1e3 * (t1 - t0):.1f} ms  bfs(host out) {1e3 * (t2 - t1):.1f} ms (device {st['kernel_ms']:.1f})"
          f"  destroy {1e3 * (t3 - t2):.1f} ms  total {1e3 * (t3 - t0):.1f} ms", flush=True)
