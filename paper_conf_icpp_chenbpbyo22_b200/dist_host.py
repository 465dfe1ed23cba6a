"""Host-side helpers of the multi-process (one process per GPU) path: the 1D
vertex-block partition of a CSR (the same blocks atos_partition_range defines)
and max/sum reductions of timings over ranks.  Pure host logic: exercised by
the world-size-2 gloo tests on CPU and by bench.py under torchrun."""
from __future__ import annotations

import torch


def block_range(n: int, nparts: int, part: int):
    """[v_begin, v_end) owned by `part`: blocks of ceil(n / nparts) (mirrors atos_partition_range)."""
    if nparts < 1 or not 0 <= part < nparts or n < 0:
        raise ValueError("bad partition arguments")
    chunk = (n + nparts - 1) // nparts
    return min(n, part * chunk), min(n, (part + 1) * chunk)


def local_rows(row_ptr: torch.Tensor, col: torch.Tensor, v_begin: int, v_end: int):
    """Rows [v_begin, v_end) of a CSR: (row_ptr_local starting at 0, col_local with GLOBAL ids)."""
    eb, ee = int(row_ptr[v_begin]), int(row_ptr[v_end])
    rp = (row_ptr[v_begin:v_end + 1] - eb).contiguous()
    return rp, col[eb:ee].contiguous()


def reduce_over_ranks(x: float, op: str = "max", group=None, device=None) -> float:
    """max / sum of a host float over all ranks (identity without torch.distributed)."""
    import torch.distributed as dist
    if not dist.is_available() or not dist.is_initialized():
        return x
    if device is None:
        device = "cuda" if dist.get_backend(group) == "nccl" else "cpu"
    t = torch.tensor([x], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX if op == "max" else dist.ReduceOp.SUM, group=group)
    return float(t.item())
