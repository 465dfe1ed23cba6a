"""Run the atomics microbenchmark on the C3 graph's edge targets (tools only)."""
import ctypes, os, subprocess, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import torch
from paper_conf_icpp_chenbpbyo22_b200 import gen
here = os.path.dirname(os.path.abspath(__file__))
so = os.path.join(here, "libatomics.so")
subprocess.check_call(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-shared", "-Xcompiler", "-fPIC",
                       "-o", so, os.path.join(here, "atomics.cu")])
lib = ctypes.CDLL(so)
lib.atom_bench.restype = ctypes.c_float
lib.atom_bench.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_void_p, ctypes.c_int, ctypes.c_int, ctypes.c_int,
                           ctypes.c_void_p]
scale = int(sys.argv[1]) if len(sys.argv) > 1 else 22
g = gen.rmat(scale, 16, 3, device="cuda")
res = torch.zeros(g.n, dtype=torch.float64, device="cuda")
out = torch.zeros(1, dtype=torch.int64, device="cuda")
names = ["atom.add.f64 (ret)", "red.add.f64", "atom.add.u64 (ret)", "red.add.u64", "atom.add.f32 (ret)"]
for kind in range(5):
    for grid, block in ((148 * 8, 256), (148 * 16, 256)):
        lib.atom_bench(g.col.data_ptr(), g.m, res.data_ptr(), kind, grid, block, out.data_ptr())
        ms = min(lib.atom_bench(g.col.data_ptr(), g.m, res.data_ptr(), kind, grid, block, out.data_ptr())
                 for _ in range(3))
        print(f"{names[kind]:20s} grid={grid}: {ms:.3f} ms  {g.m / ms / 1e6:.1f} G atomics/s", flush=True)
# sorted targets (locality) for reference
cs = torch.sort(g.col)[0]
for kind in (0, 2):
    ms = min(lib.atom_bench(cs.data_ptr(), g.m, res.data_ptr(), kind, 148 * 8, 256, out.data_ptr()) for _ in range(3))
    print(f"{names[kind]:20s} sorted targets: {ms:.3f} ms  {g.m / ms / 1e6:.1f} G atomics/s", flush=True)
