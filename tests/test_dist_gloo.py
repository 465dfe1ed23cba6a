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


def test_bench_dry_run_two_ranks_gloo():
    """`bench.py --gpus 2 --dry-run` outside torchrun relaunches itself with 2 ranks (gloo here), each rank
    builds ONLY its row block of the C5-recipe graph (small scale) and picks the 8 sources from the
    all-gathered degrees: the blocks tile [0, n), their edges add up to the full graph's, and the sources
    equal the single-process choice."""
    import json
    import subprocess
    import sys

    from paper_conf_icpp_chenbpbyo22_b200 import gen
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run([sys.executable, os.path.join(root, "bench.py"), "--gpus", "2", "--dry-run", "--scale", "12"],
                       capture_output=True, text=True, timeout=600, cwd=root)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [json.loads(x) for x in r.stdout.splitlines() if x.startswith("{")]
    assert sorted(x["rank"] for x in lines) == [0, 1]
    g = gen.rmat(12, 16, 5)
    lines.sort(key=lambda x: x["rank"])
    assert lines[0]["v_begin"] == 0 and lines[0]["v_end"] == lines[1]["v_begin"] and lines[1]["v_end"] == g.n
    assert lines[0]["m_local"] + lines[1]["m_local"] == g.m == lines[0]["m_total"]
    assert int(g.row_ptr[lines[0]["v_end"]]) == lines[0]["m_local"]
    want = [gen.pick_source(g, 105 + i) for i in range(8)]
    assert lines[0]["sources"] == want and lines[1]["sources"] == want
