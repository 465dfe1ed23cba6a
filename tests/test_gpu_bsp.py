"""GPU parity of the bulk-synchronous baselines, through the C ABI:
atos_bfs_bsp (Alg.1) bit-exact vs the serial oracle; atos_pagerank_bsp
(Alg.3) within the north_star tolerances plus the one-sided band and
conservation (the BSP iteration keeps the same invariant x* = x + (I - aP^T)^-1 r,
r >= 0); atos_color_bsp (Alg.5) always a valid colouring."""
import numpy as np
import pytest

import oracle
import paper_conf_icpp_chenbpbyo22_b200 as atos
from paper_conf_icpp_chenbpbyo22_b200 import gen

import _graphs as G
from _gpu import DEV, as_u32, check_pr, csr_of

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def rmat14():
    g = gen.rmat(14, 16, seed=21)
    rp, ci = g.numpy()
    return g, rp, ci, atos.CSR.from_graph(g.to(DEV))


def test_bfs_bsp_rmat_sources(rmat14):
    g, rp, ci, csr = rmat14
    for sseed in range(6):
        src = gen.pick_source(g, 300 + sseed)
        d, st = atos.bfs_bsp(csr, src)
        want = oracle.bfs(rp, ci, src)
        np.testing.assert_array_equal(as_u32(d), want)
        assert st["rounds"] == int(want[want != 0xFFFFFFFF].max()) + 1  # one iteration per level
        assert st["pops"] == int(np.sum(want != 0xFFFFFFFF))            # each reached vertex once


def test_bfs_bsp_matches_async(rmat14):
    g, rp, ci, csr = rmat14
    src = gen.pick_source(g, 7)
    a, _ = atos.bfs(csr, src)
    b, _ = atos.bfs_bsp(csr, src)
    np.testing.assert_array_equal(as_u32(a), as_u32(b))


@pytest.mark.parametrize("shape", ["grid", "path", "star", "directed", "isolated"])
def test_bfs_bsp_shapes(shape):
    if shape == "grid":
        rp, ci = G.grid(97, 131)
        src = 97 * 131 // 2
    elif shape == "path":
        rp, ci = G.path(5000)
        src = 0
    elif shape == "star":
        rp, ci = G.star(20000)   # hub of degree 19999: one vertex spans many 2048-edge tiles
        src = 5
    elif shape == "directed":
        rp, ci = G.gnp(3000, 0.002, seed=5, directed=True)
        src = 1
    else:
        rp, ci = G.csr_from_edges(10, [(1, 2), (2, 3)], symmetric=True)
        src = 0
    csr = csr_of(rp, ci)
    d, _ = atos.bfs_bsp(csr, src)
    np.testing.assert_array_equal(as_u32(d), oracle.bfs(rp, ci, src))


def test_bfs_bsp_host_output(rmat14):
    g, rp, ci, csr = rmat14
    import torch
    src = gen.pick_source(g, 1)
    out = torch.empty(g.n, dtype=torch.int32).pin_memory()
    atos.bfs_bsp(csr, src, out=out)
    np.testing.assert_array_equal(out.numpy().view(np.uint32), oracle.bfs(rp, ci, src))


def test_bfs_bsp_zero_degree_frontier():
    # many zero-degree vertices inside one frontier (owner range wider than the staged tile)
    n = 9000
    edges = [(0, v) for v in range(1, n)] + [(n - 1, n - 2)]
    rp, ci = G.csr_from_edges(n, edges, symmetric=False)
    csr = csr_of(rp, ci)
    d, _ = atos.bfs_bsp(csr, 0)
    np.testing.assert_array_equal(as_u32(d), oracle.bfs(rp, ci, 0))


def test_pagerank_bsp_rmat(rmat14):
    g, rp, ci, csr = rmat14
    r, st = atos.pagerank_bsp(csr, 0.85, 1e-6)
    err = check_pr(rp, ci, r, st, 1e-6)
    assert abs(err) < 1e-9 * g.n
    assert st["rounds"] > 1


def test_pagerank_bsp_regular_and_dangling():
    for rp, ci in (G.torus(40, 50), G.cycle(3000), G.complete(60)):
        n = len(rp) - 1
        r, _ = atos.pagerank_bsp(csr_of(rp, ci), 0.85, 1e-8)
        x = r.cpu().numpy() * n
        assert np.all(x <= 1 + 1e-12) and np.all(1 - x <= 1e-8 / 0.15 * 1.0001)
    # directed graph with dangling vertices: one-sided band against the Jacobi oracle
    rp, ci = G.gnp(400, 0.01, seed=9, directed=True)
    r, st = atos.pagerank_bsp(csr_of(rp, ci), 0.85, 1e-7)
    ref, _, ok = oracle.pagerank_jacobi(rp, ci, 0.85)
    assert ok
    x, xs = r.cpu().numpy() * 400, ref * 400
    assert np.all(x <= xs * (1 + 1e-9) + 1e-12)
    assert np.all(xs - x <= 1e-7 * xs / 0.15 * (1 + 1e-6) + 1e-12)


def test_color_bsp_valid(rmat14):
    g, rp, ci, csr = rmat14
    for seed in (1, 2, 3):
        c, st = atos.color_bsp(csr, seed=seed)
        col = c.cpu().numpy()
        assert oracle.validate_color(rp, ci, col) == 0
        assert st["colors_used"] == col.max() + 1
        assert st["rounds"] >= 1


@pytest.mark.parametrize("shape", ["complete", "crown", "grid", "wheel"])
def test_color_bsp_shapes(shape):
    rp, ci = {"complete": lambda: G.complete(40), "crown": lambda: G.crown(30),
              "grid": lambda: G.grid(50, 70), "wheel": lambda: G.wheel(101)}[shape]()
    c, st = atos.color_bsp(csr_of(rp, ci), seed=5, validate=1)
    col = c.cpu().numpy()
    assert oracle.validate_color(rp, ci, col) == 0
    if shape == "complete":
        assert st["colors_used"] == 40


def test_color_bsp_literal_policy_terminates_or_times_out(rmat14):
    g, rp, ci, csr = rmat14
    try:
        c, _ = atos.color_bsp(csr, seed=1, conflict_policy=1, timeout_s=3.0)
        assert oracle.validate_color(rp, ci, c.cpu().numpy()) == 0
    except RuntimeError as e:
        assert "TIMEOUT" in str(e)


def test_color_bsp_rejects_asymmetric():
    rp, ci = G.csr_from_edges(4, [(0, 1), (1, 2)], symmetric=False)
    with pytest.raises(RuntimeError, match="SYMMETRIC"):
        atos.color_bsp(csr_of(rp, ci), seed=1, validate=1)


def test_bsp_rejects_partitions():
    rp, ci = G.grid(20, 20)
    csr = csr_of(rp, ci, num_parts=2)
    with pytest.raises(RuntimeError, match="UNSUPPORTED"):
        atos.bfs_bsp(csr, 0)
