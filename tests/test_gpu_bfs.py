"""GPU parity: atos_bfs (through the C ABI) vs the serial oracle, bit-exact (BASELINE north_star).

Covers the design space of the paper's Queues API (Listing 3):
worker size thread / warp / CTA, FETCH_SIZE, persistent vs discrete,
dedupe on/off, at sizes spanning many fetch chunks with ragged tails, plus
the degenerate cases (isolated source, directed chain, empty rows).
"""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_icpp_chenbpbyo22_b200 as atos
from paper_conf_icpp_chenbpbyo22_b200 import gen

import _graphs as G
from _gpu import DEV, as_u32, check_pr, csr_of

pytestmark = pytest.mark.gpu

KNOBS = [
    dict(worker=256, fetch_size=256, persistent=1),
    dict(worker=256, fetch_size=64, persistent=1),
    dict(worker=128, fetch_size=512, persistent=1),
    dict(worker=1024, fetch_size=1024, persistent=1),
    dict(worker=32, fetch_size=1, persistent=1),
    dict(worker=32, fetch_size=8, persistent=1),
    dict(worker=1, fetch_size=1, persistent=1),
    dict(worker=1, fetch_size=4, persistent=1),
    dict(worker=256, fetch_size=256, persistent=0),
    dict(worker=32, fetch_size=8, persistent=0),
    dict(worker=1, fetch_size=2, persistent=0),
    dict(worker=256, fetch_size=256, persistent=1, dedupe=0),
    dict(worker=32, fetch_size=4, persistent=1, dedupe=0),
    # hub assist (big tasks) stressed with tiny thresholds/chunks, and disabled
    dict(worker=256, fetch_size=256, big_threshold=64, big_chunk=16),
    dict(worker=32, fetch_size=8, big_threshold=32, big_chunk=8),
    dict(worker=128, fetch_size=32, big_threshold=8, big_chunk=1, dedupe=0),
    dict(worker=256, fetch_size=256, big_threshold=-1),
    # the u32 depth-word state (the byte state's fallback for depths >= 126) forced from the start
    dict(worker=256, fetch_size=256, depth_state=2),
    dict(worker=32, fetch_size=8, depth_state=2),
    dict(worker=1, fetch_size=2, persistent=0, depth_state=2),
    # the 64-register worker build at 256 threads (default there: the 48-register 5-CTA/SM build)
    dict(worker=256, fetch_size=256, engine_variant=1),
    dict(worker=256, fetch_size=256, persistent=0, engine_variant=1),
]


def kid(k):
    return "-".join(f"{a}{b}" for a, b in k.items())


@pytest.fixture(scope="module")
def rmat14():
    g = gen.rmat(14, 16, seed=7)
    rp, ci = g.numpy()
    return rp, ci, atos.CSR.from_graph(g.to(DEV))


@pytest.mark.parametrize("knobs", KNOBS, ids=kid)
def test_rmat_all_knobs(rmat14, knobs):
    rp, ci, csr = rmat14
    for s in (gen.pick_source(gen.Graph(len(rp) - 1, len(ci), torch.from_numpy(rp), torch.from_numpy(ci)), 3), 0, 1):
        d, st = atos.bfs(csr, s, **knobs)
        want = oracle.bfs(rp, ci, s)
        np.testing.assert_array_equal(as_u32(d), want)
        reached = int(np.sum(want != 0xFFFFFFFF))
        assert st["pops"] >= reached  # every reached vertex expanded at least once


@pytest.mark.parametrize("knobs", KNOBS[:1] + KNOBS[4:5] + KNOBS[8:9] + KNOBS[6:7] + KNOBS[-2:], ids=kid)
def test_mesh_closed_form(knobs):
    R, C = 300, 257
    g = gen.mesh(R, C)
    csr = atos.CSR.from_graph(g.to(DEV))
    r, c = np.divmod(np.arange(R * C), C)
    for (r0, c0) in ((0, 0), (R // 2, C // 2), (R - 1, 5)):
        d, st = atos.bfs(csr, r0 * C + c0, **knobs)
        np.testing.assert_array_equal(as_u32(d), np.abs(r - r0) + np.abs(c - c0))


def test_mesh_road_percolated():
    g = gen.mesh(200, 200, keep_prob=0.6, seed=2)
    rp, ci = g.numpy()
    csr = atos.CSR.from_graph(g.to(DEV))
    src = gen.mesh_centre_source(g, 200, 200)
    for knobs in (KNOBS[0], KNOBS[8], KNOBS[4]):
        d, _ = atos.bfs(csr, src, **knobs)
        np.testing.assert_array_equal(as_u32(d), oracle.bfs(rp, ci, src))


@pytest.mark.parametrize("name", ["path", "star", "disconnected", "dchain", "complete", "single_edge"])
def test_small_named(name):
    rp, ci = {
        "path": G.path(1000), "star": G.star(3000), "complete": G.complete(40),
        "disconnected": G.csr_from_edges(50, [(0, 1), (1, 2), (10, 11)], symmetric=True),
        "dchain": G.csr_from_edges(6, [(0, 1), (1, 2), (2, 3), (3, 4), (4, 5)]),
        "single_edge": G.csr_from_edges(2, [(0, 1)]),
    }[name]
    n = len(rp) - 1
    csr = csr_of(rp, ci)
    for knobs in KNOBS:
        for s in sorted({0, n - 1, n // 2}):
            d, _ = atos.bfs(csr, s, **knobs)
            np.testing.assert_array_equal(as_u32(d), oracle.bfs(rp, ci, s), err_msg=f"{name} s={s} {knobs}")


def test_isolated_source():
    rp, ci = G.csr_from_edges(10, [(1, 2), (2, 3)], symmetric=True)
    csr = csr_of(rp, ci)
    d, st = atos.bfs(csr, 0)
    want = np.full(10, 0xFFFFFFFF, dtype=np.uint32)
    want[0] = 0
    np.testing.assert_array_equal(as_u32(d), want)
    assert st["pops"] == 1


def test_host_input_and_output():
    g = gen.rmat(12, 8, seed=3)
    rp, ci = g.numpy()
    csr = csr_of(rp, ci, host=True)
    out = torch.empty(g.n, dtype=torch.int32).pin_memory()
    s = gen.pick_source(g, 1)
    d, _ = atos.bfs(csr, s, out=out)
    assert not d.is_cuda
    np.testing.assert_array_equal(d.numpy().view(np.uint32), oracle.bfs(rp, ci, s))


def test_repeat_calls_reuse_workspace():
    g = gen.rmat(13, 16, seed=5)
    rp, ci = g.numpy()
    csr = atos.CSR.from_graph(g.to(DEV))
    for s in range(0, 200, 17):
        d, _ = atos.bfs(csr, s)
        np.testing.assert_array_equal(as_u32(d), oracle.bfs(rp, ci, s))


def test_errors():
    g = gen.rmat(8, 4, seed=1)
    csr = atos.CSR.from_graph(g.to(DEV))
    with pytest.raises(RuntimeError, match="INVALID_ARG"):
        atos.bfs(csr, g.n)
    with pytest.raises(RuntimeError, match="INVALID_ARG"):
        atos.bfs(csr, 0, worker=48)
    with pytest.raises(RuntimeError, match="INVALID_ARG"):
        atos.bfs(csr, 0, fetch_size=0, worker=5)
    bad_rp = torch.tensor([0, 2, 1], dtype=torch.int64, device=DEV)
    with pytest.raises(RuntimeError, match="INVALID_ARG"):
        atos.CSR(bad_rp, torch.tensor([1, 0], dtype=torch.int32, device=DEV))
    with pytest.raises(RuntimeError, match="INVALID_ARG"):
        atos.CSR(torch.tensor([0, 1], dtype=torch.int64), torch.tensor([5], dtype=torch.int32))
    # host input: non-monotone offsets are caught while narrowing on the device, for one
    # partition and for loopback partitions (host check)
    bad_h = torch.tensor([0, 2, 1, 3], dtype=torch.int64)
    cols_h = torch.tensor([1, 2, 0], dtype=torch.int32)
    for parts in (1, 2):
        with pytest.raises(RuntimeError, match="INVALID_ARG"):
            atos.CSR(bad_h, cols_h, num_parts=parts)
    with pytest.raises(RuntimeError, match="INVALID_ARG"):
        atos.CSR(torch.tensor([0, 1, 3, 2], dtype=torch.int64), cols_h)  # row_ptr[n] != m
    with pytest.raises(RuntimeError, match="INVALID_ARG"):
        atos.CSR(torch.tensor([0, 4, 2, 3], dtype=torch.int64), cols_h)  # offset > m inside
    # rejected at conflict_policy outside 0..2 and depth_state outside {0, 2}
    with pytest.raises(RuntimeError, match="INVALID_ARG"):
        atos.color(csr, 1, conflict_policy=3)
    with pytest.raises(RuntimeError, match="INVALID_ARG"):
        atos.bfs(csr, 0, depth_state=1)


def test_small_queue_overflow_reports_error():
    # paper-literal (dedupe=0) with a tiny ring must fail loudly, never hang
    g = gen.rmat(12, 16, seed=2)
    csr = atos.CSR.from_graph(g.to(DEV))
    try:
        atos.bfs(csr, gen.pick_source(g, 1), dedupe=0, queue_capacity=64, timeout_s=2.0)
    except RuntimeError as e:
        assert "OVERFLOW" in str(e) or "TIMEOUT" in str(e)
    # the handle stays usable afterwards
    rp, ci = g.numpy()
    d, _ = atos.bfs(csr, 0)
    np.testing.assert_array_equal(as_u32(d), oracle.bfs(rp, ci, 0))


@pytest.mark.slow
def test_config_c1_bench_launch():
    """C1 (RMAT S16 EF16, seed 1, source seed 101) at the bench's launch configuration."""
    g = gen.make_config("C1", device=DEV)
    rp, ci = g.numpy()
    csr = atos.CSR.from_graph(g)
    src = gen.pick_source(g, 101)
    want = oracle.bfs(rp, ci, src)
    for knobs in (dict(), dict(worker=32), dict(persistent=0)):
        d, st = atos.bfs(csr, src, **knobs)
        np.testing.assert_array_equal(as_u32(d), want)


@pytest.mark.parametrize("n,deep", [(125, False), (126, True), (400, True)])
def test_byte_state_depth_boundary(n, deep):
    """Byte state encodes depths 0..125; a pop at depth 125 with edges re-runs with u32 words
    (stats flag bit 0).  Results are bit-exact either way."""
    rp, ci = G.path(n)
    csr = csr_of(rp, ci)
    want = oracle.bfs(rp, ci, 0)
    for i, knobs in enumerate((dict(), dict(worker=32, fetch_size=4), dict(persistent=0))):
        d, st = atos.bfs(csr, 0, **knobs)
        np.testing.assert_array_equal(as_u32(d), want)
        # the first deep call re-runs (bit 0); later calls on the same graph start with u32 words (bit 1)
        assert st["flags"] == (0 if not deep else (1 if i == 0 else 2))
        d2, st2 = atos.bfs(csr, 0, depth_state=2, **knobs)
        np.testing.assert_array_equal(as_u32(d2), want)
        assert st2["flags"] == 0


@pytest.mark.parametrize("src", [0, 1733, 2999])
def test_deep_path_thin_chain(src):
    """The thin-frontier chain of the low-degree builds (CAS-first u32 relax, warp-0 scan, single-CAS
    publish, lean completion, no assist without big rows) on a 3000-vertex path: one vertex per level, depths
    far past the u8 shadow's 254 -- closed form |i - src| for every worker / grid / dedupe / discrete mode."""
    n = 3000
    rp, ci = G.path(n)
    csr = csr_of(rp, ci)
    want = np.abs(np.arange(n) - src).astype(np.uint32)
    for knobs in (dict(), dict(num_blocks=1), dict(num_blocks=3), dict(dedupe=0), dict(worker=32, fetch_size=4),
                  dict(persistent=0), dict(depth_state=2), dict(worker=1024, fetch_size=1024)):
        d, _ = atos.bfs(csr, src, **knobs)
        np.testing.assert_array_equal(as_u32(d), want, err_msg=str(knobs))


def test_byte_state_word_neighbours():
    """Four consecutive vertex ids share one 32-bit state word: a 4-clique plus pendant chains
    exercises CAS retries on neighbouring bytes."""
    edges = [(a, b) for a in range(4) for b in range(4) if a != b]
    edges += [(k, 4 + k) for k in range(4)] + [(4 + k, 8 + k) for k in range(4)]
    rp, ci = G.csr_from_edges(12, edges, symmetric=True)
    csr = csr_of(rp, ci)
    for src in range(12):
        d, _ = atos.bfs(csr, src)
        np.testing.assert_array_equal(as_u32(d), oracle.bfs(rp, ci, src))


@pytest.mark.parametrize("layout", ["input", "auto", "degree"])
def test_layout_modes(layout):
    """The degree layout (default) is invisible: caller ids in, caller ids out, device and host outputs."""
    g = gen.rmat(13, 16, seed=5)
    rp, ci = g.numpy()
    csr = atos.CSR.from_graph(g.to(DEV), layout=layout)
    for s in (gen.pick_source(g, 9), 0, g.n - 1):
        want = oracle.bfs(rp, ci, s)
        d, _ = atos.bfs(csr, s)
        np.testing.assert_array_equal(as_u32(d), want)
        out = torch.empty(g.n, dtype=torch.int32)
        d, _ = atos.bfs(csr, s, out=out)
        np.testing.assert_array_equal(d.numpy().view(np.uint32), want)
        d, _ = atos.bfs_bsp(csr, s)
        np.testing.assert_array_equal(as_u32(d), want)


def test_layout_degree_mesh_closed_form():
    R, C = 300, 257
    g = gen.mesh(R, C)
    csr = atos.CSR.from_graph(g.to(DEV), layout="degree")
    r, c = np.divmod(np.arange(R * C), C)
    for (r0, c0) in ((0, 0), (R // 2, C // 2)):
        d, st = atos.bfs(csr, r0 * C + c0)
        np.testing.assert_array_equal(as_u32(d), np.abs(r - r0) + np.abs(c - c0))


def test_l2_persist_window_parity():
    """cfg.l2_persist = 1 (persisting access-policy window on the hot state; the queue counters carry
    evict_last hints on every access regardless): same exact depths / in-tolerance ranks."""
    g = gen.rmat(16, 16, seed=11)
    rp, ci = g.numpy()
    csr = atos.CSR.from_graph(g.to(DEV))
    src = gen.pick_source(g, 3)
    d, _ = atos.bfs(csr, src, l2_persist=1)
    np.testing.assert_array_equal(as_u32(d), oracle.bfs(rp, ci, src))
    r, st = atos.pagerank(csr, 0.85, 1e-6, l2_persist=1)
    check_pr(rp, ci, r, st, 1e-6)
