"""Random-gather throughput vs footprint (tools only): the C5 edge stream gathering one byte per edge from
an array of S MB (targets folded modulo S) -- is the effective L2 capacity for a shared random array ~63 MB
(one partition) or ~126 MB?"""
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
g = gen.rmat(26, 16, 5, device="cuda")
out = torch.zeros(1, dtype=torch.int64, device="cuda")
col = g.col
for mb in (8, 16, 32, 48, 64, 80, 96, 128, 256):
    size = mb << 20
    c2 = (col.to(torch.int64) * 2654435761 % size).to(torch.int32) if size < g.n else col
    sh = torch.randint(0, 8, (max(size, g.n),), dtype=torch.uint8, device="cuda")
    ms = min(lib.gather_bench(c2.data_ptr(), sh.data_ptr(), g.m, 4, 148 * 8, 256, out.data_ptr()) for _ in range(3))
    print(f"{mb:4d} MB footprint: {ms:.2f} ms  {g.m / ms / 1e6:.1f} G gathers/s", flush=True)
    del c2, sh
