"""World-size-2 gloo tests (CPU) of the multi-process host logic: the 1D block
partition each rank builds must tile the graph exactly and agree with
atos_partition_range; reductions over ranks give the max/sum the bench uses."""
import os
import socket

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    try:
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        dist.init_process_group("gloo", rank=rank, world_size=world)
        import paper_conf_icpp_chenbpbyo22_b200 as atos
        from paper_conf_icpp_chenbpbyo22_b200 import dist_host, gen
        g = gen.rmat(10, 8, seed=3)
        vb, ve = dist_host.block_range(g.n, world, rank)
        assert (vb, ve) == atos.partition_range(g.n, world, rank)
        rp, ci = dist_host.local_rows(g.row_ptr, g.col, vb, ve)
        assert rp[0] == 0 and rp[-1] == ci.numel()
        # gather every rank's rows and compare with the global CSR
        sizes = [None] * world
        dist.all_gather_object(sizes, (vb, ve, rp.tolist(), ci.tolist()))
        sizes.sort()
        rows, cols, cur = [0], [], 0
        for (b, e, r, c) in sizes:
            assert b == cur
            cur = e
            rows += [x + len(cols) for x in r[1:]]
            cols += c
        assert cur == g.n
        assert rows == g.row_ptr.tolist() and cols == g.col.tolist()
        mx = dist_host.reduce_over_ranks(float(rank + 1), "max")
        sm = dist_host.reduce_over_ranks(float(rank + 1), "sum")
        assert mx == world and sm == world * (world + 1) / 2
        # the NCCL unique id travels as bytes through a broadcast (bench.py); here its stand-in
        obj = [b"x" * 128 if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        assert obj[0] == b"x" * 128
        q.put((rank, "ok"))
    except Exception as e:  # pragma: no cover - reported to the parent
        q.put((rank, repr(e)))
    finally:
        if dist.is_initialized():
            dist.destroy_process_group()


@pytest.mark.parametrize("world", [2])
def test_partition_tiles_graph_gloo(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    res = [q.get(timeout=180) for _ in ps]
    for p in ps:
        p.join(timeout=60)
    assert all(m == "ok" for _, m in res), res


def test_block_range_matches_library():
    import paper_conf_icpp_chenbpbyo22_b200 as atos
    from paper_conf_icpp_chenbpbyo22_b200 import dist_host
    for n in (0, 1, 7, 1000, 1 << 20):
        for P in (1, 2, 3, 8):
            for p in range(P):
                assert dist_host.block_range(n, P, p) == atos.partition_range(n, P, p)
