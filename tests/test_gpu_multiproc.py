"""The multi-process (one process per partition) path of SURVEY 8(e), run for real with 2 and 3 ranks:
every rank is its own process with its own CUDA context on the one GPU of this box, its own partition
(atos_csr_create_part, rows built by gen.rmat(rows=...)), and the exchange rounds' counts -> payload ->
apply -> termination allreduce go through atos_comm_create_host over torch.distributed gloo (NCCL refuses
two ranks on one device).  Every rank checks its depth / rank slice against the oracle."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, scale, q):
    try:
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        dist.init_process_group("gloo", rank=rank, world_size=world)
        import sys
        sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
        import oracle
        import paper_conf_icpp_chenbpbyo22_b200 as atos
        from paper_conf_icpp_chenbpbyo22_b200 import dist_host, gen
        from _gpu import check_pr
        full = gen.rmat(scale, 16, seed=9)
        rp, ci = full.numpy()
        vb, ve = dist_host.block_range(full.n, world, rank)
        part = gen.rmat(scale, 16, seed=9, rows=(vb, ve))
        comm = atos.Comm.host(world, rank, 0)
        csr = comm.partition(full.n, vb, ve, part.row_ptr, part.col)  # host tensors
        for s in (gen.pick_source(full, 1), gen.pick_source(full, 2), 0):
            d, st = atos.bfs(csr, s)
            want = oracle.bfs(rp, ci, s)
            np.testing.assert_array_equal(d.cpu().numpy().view(np.uint32), want[vb:ve])
            assert st["rounds"] >= 1
            # atos_comm_gather: the whole depth vector on rank 0
            allv = comm.gather(full.n, d)
            if rank == 0:
                np.testing.assert_array_equal(allv.cpu().numpy().view(np.uint32), want)
            else:
                assert allv is None
        # PageRank: each rank checks its slice against the Jacobi fixed point (same tolerance as the
        # single-GPU tests); conservation holds for the SUM over ranks
        ref, _, ok = oracle.pagerank_jacobi(rp, ci, 0.85)
        r, st = atos.pagerank(csr, 0.85, 1e-6)
        x = r.cpu().numpy()
        rel = np.abs(x - ref[vb:ve]) / np.maximum(ref[vb:ve], 1e-300)
        assert rel.max() <= 1e-4
        assert np.all(x <= ref[vb:ve] * (1 + 1e-9) + 1e-15)
        tot = torch.tensor([x.sum() * full.n], dtype=torch.float64)
        dist.all_reduce(tot)
        iso = int(np.sum(np.diff(rp) == 0))
        # stats.residual_sum of a distributed call is already the sum over ranks (allreduce in the library)
        assert abs(tot[0].item() + st["residual_sum"] / 0.15 - (full.n - 0.85 * iso)) < 1e-9 * full.n
        # NEXT-4 across processes: the barrier-free kernel with every peer's rings / state mapped through CUDA
        # IPC (the ranks' kernels time-share the one GPU here); bit-exact BFS, in-tolerance PageRank
        for s in (gen.pick_source(full, 1), 0):
            d, st = atos.bfs(csr, s, barrier_free=1, timeout_s=120)
            np.testing.assert_array_equal(d.cpu().numpy().view(np.uint32), oracle.bfs(rp, ci, s)[vb:ve])
        r, st = atos.pagerank(csr, 0.85, 1e-6, barrier_free=1, timeout_s=120)
        x = r.cpu().numpy()
        assert (np.abs(x - ref[vb:ve]) / np.maximum(ref[vb:ve], 1e-300)).max() <= 1e-4
        assert np.all(x <= ref[vb:ve] * (1 + 1e-9) + 1e-15)
        tot = torch.tensor([x.sum() * full.n], dtype=torch.float64)
        dist.all_reduce(tot)
        assert abs(tot[0].item() + st["residual_sum"] / 0.15 - (full.n - 0.85 * iso)) < 1e-9 * full.n
        csr.close()
        comm.close()
        q.put((rank, "ok"))
    except Exception as e:  # reported to the parent
        import traceback
        q.put((rank, traceback.format_exc()))
    finally:
        if dist.is_initialized():
            dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_partitioned_multiprocess_host_comm(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, 13, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=600) for _ in procs]
    for p in procs:
        p.join(timeout=60)
    assert all(m == "ok" for _, m in res), res
