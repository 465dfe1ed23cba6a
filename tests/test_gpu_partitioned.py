"""GPU: the partitioned (multi-GPU) BFS / PageRank protocol of S10 run with P
loopback partitions on one device -- same rounds, ghost combining, packing,
exchange and apply as the NCCL path, exchange by device copies.  BFS must stay
bit-exact and PageRank within the north_star tolerance + conservation (ghost
mass must never be lost)."""
import numpy as np
import pytest

import oracle
import paper_conf_icpp_chenbpbyo22_b200 as atos
from paper_conf_icpp_chenbpbyo22_b200 import gen

import _graphs as G
from _gpu import DEV, as_u32, check_pr, csr_of

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def rmat13():
    g = gen.rmat(13, 16, seed=21)
    rp, ci = g.numpy()
    return g, rp, ci


@pytest.mark.parametrize("P", [2, 3, 4, 8])
@pytest.mark.parametrize("knobs", [dict(), dict(worker=32, fetch_size=8), dict(dedupe=0)], ids=["cta", "warp", "nodedupe"])
def test_bfs_loopback_rmat(rmat13, P, knobs):
    g, rp, ci = rmat13
    csr = atos.CSR.from_graph(g.to(DEV), num_parts=P)
    for s in (gen.pick_source(g, 1), 0, g.n - 1):
        d, st = atos.bfs(csr, s, **knobs)
        np.testing.assert_array_equal(as_u32(d), oracle.bfs(rp, ci, s))
        assert st["rounds"] >= 1


@pytest.mark.parametrize("P", [2, 5])
def test_bfs_loopback_mesh(P):
    R, C = 120, 97
    g = gen.mesh(R, C)
    csr = atos.CSR.from_graph(g.to(DEV), num_parts=P)
    r, c = np.divmod(np.arange(R * C), C)
    for (r0, c0) in ((0, 0), (R // 2, C // 2)):
        for knobs in (dict(), dict(depth_state=2)):
            d, st = atos.bfs(csr, r0 * C + c0, **knobs)
            np.testing.assert_array_equal(as_u32(d), np.abs(r - r0) + np.abs(c - c0))
            # byte state unless forced to u32 words; the corner source (depth 215) re-runs with u32 words
            assert bool(st["flags"] & 1) == (not knobs and r0 == 0)


def test_bfs_loopback_directed_and_host_output():
    import torch
    rp, ci = G.csr_from_edges(7, [(0, 1), (1, 2), (2, 3), (3, 4), (4, 5), (5, 6), (6, 0)])
    csr = csr_of(rp, ci, num_parts=3)
    out = torch.empty(7, dtype=torch.int32)
    d, st = atos.bfs(csr, 4, out=out)
    np.testing.assert_array_equal(d.numpy().view(np.uint32), oracle.bfs(rp, ci, 4))


@pytest.mark.parametrize("P", [2, 4, 7])
def test_pagerank_loopback_rmat(rmat13, P):
    g, rp, ci = rmat13
    ref, _, _ = oracle.pagerank_jacobi(rp, ci, 0.85)
    csr = atos.CSR.from_graph(g.to(DEV), num_parts=P)
    for knobs in (dict(), dict(worker=32, fetch_size=4)):
        r, st = atos.pagerank(csr, 0.85, 1e-6, **knobs)
        err = check_pr(rp, ci, r, st, 1e-6, ref=ref)
        assert abs(err) < 1e-9 * g.n, "ghost mass lost or duplicated"
        assert st["bytes_exchanged"] > 0


def test_pagerank_loopback_star():
    n = 5001
    rp, ci = G.star(n)
    csr = csr_of(rp, ci, num_parts=4)
    r, st = atos.pagerank(csr, 0.85, 1e-10)
    a = 0.85
    xc = (1 + a * (n - 1)) / (1 + a)
    xl = (1 - a) + a * xc / (n - 1)
    x = r.cpu().numpy() * n
    np.testing.assert_allclose(x[0], xc, rtol=1e-8)
    np.testing.assert_allclose(x[1:], xl, rtol=1e-8)


def test_color_partitioned_unsupported(rmat13):
    g, rp, ci = rmat13
    csr = atos.CSR.from_graph(g.to(DEV), num_parts=2)
    with pytest.raises(RuntimeError, match="UNSUPPORTED"):
        atos.color(csr, 1)


def test_nccl_single_rank_communicator(rmat13):
    """The NCCL path end to end with one rank (self send/recv + allreduce): dlopen,
    unique id, communicator, partition creation, exchange rounds."""
    g, rp, ci = rmat13
    uid = atos.Comm.unique_id()
    assert len(uid) == 128
    comm = atos.Comm(1, 0, uid, 0)
    vb, ve = atos.partition_range(g.n, 1, 0)
    part = comm.partition(g.n, vb, ve, g.row_ptr.to(DEV), g.col.to(DEV))
    s = gen.pick_source(g, 1)
    d, st = atos.bfs(part, s)
    np.testing.assert_array_equal(as_u32(d), oracle.bfs(rp, ci, s))
    r, st = atos.pagerank(part, 0.85, 1e-6)
    check_pr(rp, ci, r, st, 1e-6)
    # the cross-process barrier-free path over NCCL (IPC handle all-gather by grouped send/recv)
    d, st = atos.bfs(part, s, barrier_free=1)
    np.testing.assert_array_equal(as_u32(d), oracle.bfs(rp, ci, s))
    r, st = atos.pagerank(part, 0.85, 1e-6, barrier_free=1)
    check_pr(rp, ci, r, st, 1e-6)
    # atos_comm_gather over NCCL: the (only) slice lands on rank 0
    full = comm.gather(g.n, d)
    np.testing.assert_array_equal(as_u32(full), oracle.bfs(rp, ci, s))
    with pytest.raises(RuntimeError, match="INVALID_ARG"):
        comm.partition(g.n, 0, g.n - 1, g.row_ptr[:-1].to(DEV), g.col.to(DEV))
    part.close()
    comm.close()


# ---- NEXT-4: barrier-free partitioned PageRank (nobarrier.cu) ----

@pytest.mark.parametrize("P", [2, 3, 8])
def test_pagerank_barrier_free_rmat(rmat13, P):
    """One persistent kernel, remote mass straight into the owner's residue slice: same north_star bound
    as the exchange rounds and the same conservation (no mass lost or duplicated)."""
    g, rp, ci = rmat13
    ref, _, _ = oracle.pagerank_jacobi(rp, ci, 0.85)
    csr = atos.CSR.from_graph(g.to(DEV), num_parts=P)
    for eps in (1e-6, 1e-9):
        r, st = atos.pagerank(csr, 0.85, eps, barrier_free=1)
        err = check_pr(rp, ci, r, st, eps, ref=ref)
        assert abs(err) < 1e-9 * g.n, "mass lost or duplicated"
        assert st["rounds"] == 1 and st["bytes_exchanged"] == 0
        assert st["pops"] >= 1 and st["edges"] >= 1


def test_pagerank_barrier_free_star_closed_form():
    n = 5001
    rp, ci = G.star(n)
    csr = csr_of(rp, ci, num_parts=4)
    r, st = atos.pagerank(csr, 0.85, 1e-10, barrier_free=1)
    a = 0.85
    xc = (1 + a * (n - 1)) / (1 + a)
    xl = (1 - a) + a * xc / (n - 1)
    x = r.cpu().numpy() * n
    np.testing.assert_allclose(x[0], xc, rtol=1e-8)
    np.testing.assert_allclose(x[1:], xl, rtol=1e-8)


def test_pagerank_barrier_free_ragged_and_dangling():
    """n not a multiple of P (short last partition), isolated and dangling vertices, host output."""
    import torch
    rp, ci = G.csr_from_edges(11, [(0, 1), (1, 0), (1, 2), (2, 1), (3, 4), (4, 3), (5, 6), (6, 7), (7, 5),
                                   (8, 9)])
    ref, _, _ = oracle.pagerank_jacobi(rp, ci, 0.85)
    csr = csr_of(rp, ci, num_parts=3)
    out = torch.empty(11, dtype=torch.float64)
    r, st = atos.pagerank(csr, 0.85, 1e-12, out=out, barrier_free=1)
    check_pr(rp, ci, r, st, 1e-12, ref=ref)


def test_barrier_free_unsupported(rmat13):
    g, rp, ci = rmat13
    csr = atos.CSR.from_graph(g.to(DEV), num_parts=1)
    with pytest.raises(RuntimeError, match="UNSUPPORTED"):
        atos.pagerank(csr, 0.85, 1e-6, barrier_free=1)
    with pytest.raises(RuntimeError, match="UNSUPPORTED"):
        atos.bfs(csr, 0, barrier_free=1)


@pytest.mark.parametrize("P", [2, 3, 8])
def test_bfs_barrier_free_rmat(rmat13, P):
    """Barrier-free BFS over loopback partitions: remote atomicMin straight into the owner's depth slice,
    in-queue bit dedupe; label-correcting, so bit-exact against the oracle."""
    g, rp, ci = rmat13
    csr = atos.CSR.from_graph(g.to(DEV), num_parts=P)
    for s in (gen.pick_source(g, 1), 0, g.n - 1):
        d, st = atos.bfs(csr, s, barrier_free=1)
        np.testing.assert_array_equal(as_u32(d), oracle.bfs(rp, ci, s))
        assert st["rounds"] == 1 and st["bytes_exchanged"] == 0


@pytest.mark.parametrize("P", [2, 5])
def test_bfs_barrier_free_mesh(P):
    R, C = 120, 97
    g = gen.mesh(R, C)
    csr = atos.CSR.from_graph(g.to(DEV), num_parts=P)
    r, c = np.divmod(np.arange(R * C), C)
    for (r0, c0) in ((0, 0), (R // 2, C // 2)):
        d, st = atos.bfs(csr, r0 * C + c0, barrier_free=1)
        np.testing.assert_array_equal(as_u32(d), np.abs(r - r0) + np.abs(c - c0))


def test_bfs_barrier_free_directed_host_output():
    import torch
    rp, ci = G.csr_from_edges(7, [(0, 1), (1, 2), (2, 3), (3, 4), (4, 5), (5, 6), (6, 0)])
    csr = csr_of(rp, ci, num_parts=3)
    out = torch.empty(7, dtype=torch.int32)
    d, st = atos.bfs(csr, 4, out=out, barrier_free=1)
    np.testing.assert_array_equal(d.numpy().view(np.uint32), oracle.bfs(rp, ci, 4))


def test_barrier_free_rejects_ignored_knobs(rmat13):
    g, rp, ci = rmat13
    csr = atos.CSR.from_graph(g.to(DEV), num_parts=2)
    for knob in (dict(persistent=0), dict(dedupe=0), dict(worker=32), dict(fetch_size=64),
                 dict(queue_capacity=1 << 20), dict(depth_state=2), dict(engine_variant=1)):
        with pytest.raises(RuntimeError, match="UNSUPPORTED"):
            atos.bfs(csr, 0, barrier_free=1, **knob)


def test_barrier_free_trailing_empty_partitions():
    """n = 9 over P = 8: ceil(9/8) = 2, so parts 5..7 are empty and part 5 starts at min(n, 10) = 9."""
    rp, ci = G.path(9)
    csr = csr_of(rp, ci, num_parts=8)
    for s in (0, 4, 8):
        d, st = atos.bfs(csr, s, barrier_free=1)
        np.testing.assert_array_equal(as_u32(d), oracle.bfs(rp, ci, s))
        r, st = atos.pagerank(csr, 0.85, 1e-10, barrier_free=1)
        check_pr(rp, ci, r, st, 1e-10)


def test_barrier_free_device_deadline():
    """timeout_s is a device deadline: a run longer than it stops itself and the call reports TIMEOUT;
    the next call on the same handle is unaffected."""
    g = gen.rmat(16, 16, seed=7)
    rp, ci = g.numpy()
    csr = atos.CSR.from_graph(g.to(DEV), num_parts=4)
    with pytest.raises(RuntimeError, match="TIMEOUT"):
        atos.pagerank(csr, 0.85, 1e-14, barrier_free=1, timeout_s=1e-5)
    r, st = atos.pagerank(csr, 0.85, 1e-6, barrier_free=1)
    check_pr(rp, ci, r, st, 1e-6)
