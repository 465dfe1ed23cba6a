"""GPU parity: atos_pagerank vs the oracle's fixed point (BASELINE north_star tolerances:
every rank within 1e-4 relative, L1 <= 1e-5 at eps = 1e-6), plus the proven
one-sided band 0 <= x* - x <= eps x*/(1-a) and mass conservation
sum x + sum r/(1-a) = n - a #isolated (DESIGN.md R-PR-1/R-PR-6)."""
import numpy as np
import torch
import pytest

import oracle
import paper_conf_icpp_chenbpbyo22_b200 as atos
from paper_conf_icpp_chenbpbyo22_b200 import gen

import _graphs as G
from _gpu import DEV, check_pr, csr_of

pytestmark = pytest.mark.gpu

KNOBS = [
    dict(worker=256, fetch_size=256),
    dict(worker=512, fetch_size=128),
    dict(worker=32, fetch_size=8),
    dict(worker=32, fetch_size=1),
    dict(worker=1, fetch_size=1),
    dict(worker=256, fetch_size=256, persistent=0),
    dict(worker=32, fetch_size=4, persistent=0),
    dict(worker=256, fetch_size=256, check_size=1024),
    dict(worker=256, fetch_size=256, big_threshold=64, big_chunk=16),
    dict(worker=32, fetch_size=4, big_threshold=16, big_chunk=4),
    dict(worker=256, fetch_size=256, big_threshold=-1),
    dict(worker=256, fetch_size=256, engine_variant=1),
]


def kid(k):
    return "-".join(f"{a}{b}" for a, b in k.items())


@pytest.fixture(scope="module")
def rmat13():
    g = gen.rmat(13, 16, seed=11)
    rp, ci = g.numpy()
    ref, _, ok = oracle.pagerank_jacobi(rp, ci, 0.85)
    return rp, ci, ref, atos.CSR.from_graph(g.to(DEV))


@pytest.mark.parametrize("knobs", KNOBS, ids=kid)
def test_rmat_parity(rmat13, knobs):
    rp, ci, ref, csr = rmat13
    r, st = atos.pagerank(csr, 0.85, 1e-6, **knobs)
    err = check_pr(rp, ci, r, st, 1e-6, ref=ref)
    assert abs(err) < 1e-9 * len(ref)


def test_regular_graphs_uniform():
    for rp, ci in (G.torus(64, 80), G.cycle(5000), G.hypercube(10)):
        n = len(rp) - 1
        csr = csr_of(rp, ci)
        r, st = atos.pagerank(csr, 0.85, 1e-8)
        x = r.cpu().numpy() * n
        assert np.all(x <= 1 + 1e-12) and np.all(1 - x <= 1e-8 / 0.15 * 1.0001)


def test_star_closed_form():
    n = 20001
    rp, ci = G.star(n)
    csr = csr_of(rp, ci)
    r, st = atos.pagerank(csr, 0.85, 1e-10)
    a = 0.85
    xc = (1 + a * (n - 1)) / (1 + a)
    xl = (1 - a) + a * xc / (n - 1)
    x = r.cpu().numpy() * n
    np.testing.assert_allclose(x[0], xc, rtol=1e-8)
    np.testing.assert_allclose(x[1:], xl, rtol=1e-8)


def test_directed_dangling_and_multiedges():
    rng = np.random.default_rng(4)
    n = 3000
    src = rng.integers(0, n, 20000)
    dst = rng.integers(0, n // 2, 20000)  # half the vertices have no out-edges? no: in-edges only to low ids
    rp, ci = G.csr_from_edges(n, zip(src, dst), dedupe=False, keep_self_loops=True)
    csr = csr_of(rp, ci)
    for knobs in KNOBS[:5]:
        r, st = atos.pagerank(csr, 0.85, 1e-7, **knobs)
        check_pr(rp, ci, r, st, 1e-7)


def test_golden_three_vertex():
    rp, ci = G.csr_from_edges(3, [(0, 1), (0, 2), (1, 2)])
    csr = csr_of(rp, ci)
    r, st = atos.pagerank(csr, 0.85, 1e-13)
    np.testing.assert_allclose(r.cpu().numpy() * 3, [0.15, 0.21375, 0.3954375], rtol=1e-11)


def test_mesh_road():
    g = gen.mesh(150, 170, keep_prob=0.6, seed=2)
    rp, ci = g.numpy()
    csr = atos.CSR.from_graph(g.to(DEV))
    r, st = atos.pagerank(csr, 0.85, 1e-6)
    err = check_pr(rp, ci, r, st, 1e-6)
    assert abs(err) < 1e-9 * g.n


def test_bad_args():
    rp, ci = G.cycle(10)
    csr = csr_of(rp, ci)
    with pytest.raises(RuntimeError, match="INVALID_ARG"):
        atos.pagerank(csr, 1.0, 1e-6)
    with pytest.raises(RuntimeError, match="INVALID_ARG"):
        atos.pagerank(csr, 0.85, 0.0)


def test_layout_input_and_auto_agree(rmat13):
    rp, ci, ref, _ = rmat13
    g = gen.Graph(len(rp) - 1, len(ci), torch.from_numpy(rp), torch.from_numpy(ci))
    for layout in ("input", "auto", "degree"):
        csr = atos.CSR.from_graph(g.to(DEV), layout=layout)
        r, st = atos.pagerank(csr, 0.85, 1e-6)
        check_pr(rp, ci, r, st, 1e-6, ref=ref)


@pytest.fixture(scope="module")
def rmat13_degree(rmat13):
    rp, ci, ref, _ = rmat13
    g = gen.Graph(len(rp) - 1, len(ci), torch.from_numpy(rp), torch.from_numpy(ci))
    return rp, ci, ref, atos.CSR.from_graph(g.to(DEV), layout="degree")


@pytest.mark.parametrize("knobs", KNOBS, ids=kid)
def test_degree_layout_residue_slots(rmat13_degree, knobs):
    """Single-partition PageRank on a degree-layout graph keeps its residue and rank arrays in interleaved
    slots (apps.cuh res_slot): init, seed, relax, the Check_Size sweep and the finalize all go through the
    same bijection -- every worker mode stays in the north-star tolerance with conservation."""
    rp, ci, ref, csr = rmat13_degree
    r, st = atos.pagerank(csr, 0.85, 1e-6, **knobs)
    err = check_pr(rp, ci, r, st, 1e-6, ref=ref)
    assert abs(err) < 1e-9 * len(ref)


@pytest.mark.parametrize("slot_log", ["0", "1", "4"])
def test_degree_layout_slot_widths(rmat13_degree, slot_log, monkeypatch):
    """Other interleave widths (ATOS_PR_SLOT_LOG; 0 = plain addressing) give the same fixed point."""
    monkeypatch.setenv("ATOS_PR_SLOT_LOG", slot_log)
    rp, ci, ref, csr = rmat13_degree
    r, st = atos.pagerank(csr, 0.85, 1e-6)
    check_pr(rp, ci, r, st, 1e-6, ref=ref)


def test_degree_layout_tiny_graphs():
    """n below 32 (no room for an interleave) and a star (one hub) under the degree layout."""
    for rp, ci in (G.path(7), G.star(40), G.complete(12)):
        n = len(rp) - 1
        g = gen.Graph(n, len(ci), torch.from_numpy(rp), torch.from_numpy(ci))
        csr = atos.CSR.from_graph(g.to(DEV), layout="degree")
        r, st = atos.pagerank(csr, 0.85, 1e-8)
        check_pr(rp, ci, r, st, 1e-8)
