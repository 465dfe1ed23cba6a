"""Run the gather microbenchmark on the C5 graph (tools only)."""
import ctypes, os, subprocess, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import torch
from paper_conf_icpp_chenbpbyo22_b200 import gen
here = os.path.dirname(os.path.abspath(__file__))
so = os.path.join(here, "libgather.so")
subprocess.check_call(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-shared", "-Xcompiler", "-fPIC",
                       "-o", so, os.path.join(here, "gather.cu")])
lib = ctypes.CDLL(so)
lib.gather_bench.restype = ctypes.c_float
lib.gather_bench.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_void_p]
scale = int(sys.argv[1]) if len(sys.argv) > 1 else 26
g = gen.rmat(scale, 16, 5, device="cuda")
sh = torch.randint(0, 8, (g.n,), dtype=torch.uint8, device="cuda")
out = torch.zeros(1, dtype=torch.int64, device="cuda")
for U in (1, 2, 4, 8):
    for grid, block in ((148 * 8, 256), (148 * 16, 256), (148 * 4, 512)):
        lib.gather_bench(g.col.data_ptr(), sh.data_ptr(), g.m, U, grid, block, out.data_ptr())
        ms = min(lib.gather_bench(g.col.data_ptr(), sh.data_ptr(), g.m, U, grid, block, out.data_ptr()) for _ in range(3))
        print(f"U={U} grid={grid} block={block}: {ms:.2f} ms  {g.m / ms / 1e6:.1f} G edges/s  col {4 * g.m / ms / 1e6:.0f} GB/s")
