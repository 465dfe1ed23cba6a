"""GPU parity at BASELINE.json's full sizes, in the launch configuration bench.py
times (library defaults), checked against what the oracle / mathematics fix at
that size:

* C2  mesh 4900 x 4900 (24.0M vertices): BFS depth has the closed form
      |r - r0| + |c - c0| -> compared element by element, persistent AND discrete;
* C3  RMAT S22 PageRank: the oracle's Jacobi fixed point (fp64, ~1 min on one
      core) -> every rank within 1e-4 relative, L1 <= 1e-5, one-sided band,
      conservation;
* C4  Kronecker S20 EF64 colouring: oracle validator (proper, colour <= deg);
* C5  RMAT S26 BFS (2.1B edges): full oracle BFS from EVERY one of the 8 sources
      bench.py times (seeds 105..112), compared bit for bit, plus the Graph500
      validator;
* C5  RMAT S26 PageRank (the bench's pagerank_c5 line, degree layout): the
      residual certificate r = (1-a)1 + a P^T x - x computed by the oracle in one
      pass; 0 <= r <= eps elementwise implies 0 <= x* - x <= eps x*/(1-a) (the
      north-star 1e-4 relative / 1e-5 L1 tolerance with 15x / 1.5x margin)
      without ~185 Jacobi sweeps over 2.1B edges; plus conservation;
* S23 RMAT PageRank (the first scale where ATOS_LAYOUT_AUTO picks the degree
      layout): full Jacobi parity like C3.
Marked slow; they run in the -m gpu suite."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_icpp_chenbpbyo22_b200 as atos
from paper_conf_icpp_chenbpbyo22_b200 import gen

from _gpu import DEV, as_u32, check_pr

pytestmark = [pytest.mark.gpu, pytest.mark.slow]


@pytest.mark.parametrize("persistent", [1, 0], ids=["persistent", "discrete"])
def test_c2_mesh_closed_form(persistent):
    R = C = 4900
    g = gen.mesh(R, C, device=DEV)
    csr = atos.CSR.from_graph(g)
    src = gen.mesh_centre_source(g, R, C)
    r0, c0 = divmod(src, C)
    d, st = atos.bfs(csr, src, persistent=persistent, timeout_s=120.0)
    v = torch.arange(R * C, device=DEV, dtype=torch.int64)
    want = (torch.abs(v // C - r0) + torch.abs(v % C - c0)).to(torch.int32)
    assert torch.equal(d, want)
    if not persistent:
        assert st["rounds"] == int(want.max().item()) + 1  # one launch per BFS level (frontier)


def test_c2_road_persistent_vs_discrete():
    g = gen.mesh(4900, 4900, keep_prob=0.6, seed=2, device=DEV)
    csr = atos.CSR.from_graph(g)
    src = gen.mesh_centre_source(g, 4900, 4900)
    a, _ = atos.bfs(csr, src, timeout_s=120.0)
    b, _ = atos.bfs(csr, src, persistent=0, timeout_s=120.0)
    assert torch.equal(a, b)
    rp, ci = g.numpy()
    np.testing.assert_array_equal(as_u32(a), oracle.bfs(rp, ci, src))


def test_c3_pagerank_full():
    g = gen.make_config("C3", device=DEV)
    csr = atos.CSR.from_graph(g)
    r, st = atos.pagerank(csr, 0.85, 1e-6)
    rp, ci = g.numpy()
    ref, it, ok = oracle.pagerank_jacobi(rp, ci, 0.85)
    assert ok
    err = check_pr(rp, ci, r, st, 1e-6, ref=ref)
    assert abs(err) < 1e-9 * g.n


def test_c4_color_full():
    g = gen.make_config("C4", device=DEV)
    assert 100e6 <= g.m <= 120e6  # hollywood-shaped band
    csr = atos.CSR.from_graph(g)
    c, st = atos.color(csr, 1)
    rp, ci = g.numpy()
    assert oracle.validate_color(rp, ci, c.cpu().numpy()) == 0
    assert st["colors_used"] == int(c.max().item()) + 1


def test_s23_pagerank_degree_layout_jacobi():
    g = gen.rmat(23, 16, 3, device=DEV)
    csr = atos.CSR.from_graph(g)
    assert csr.layout == "degree"  # the auto rule's first degree-layout scale (n * 8 B > L2 / 2)
    r, st = atos.pagerank(csr, 0.85, 1e-6)
    rp, ci = g.numpy()
    ref, it, ok = oracle.pagerank_jacobi(rp, ci, 0.85)
    assert ok
    err = check_pr(rp, ci, r, st, 1e-6, ref=ref)
    assert abs(err) < 1e-9 * g.n


@pytest.fixture(scope="module")
def c5():
    g = gen.make_config("C5", device=DEV)
    rp, ci = g.numpy()
    sources = [gen.pick_source(g, 105 + i) for i in range(8)]  # the bench's timed sources
    csr = atos.CSR.from_graph(g)
    n = g.n
    del g
    torch.cuda.empty_cache()
    yield csr, rp, ci, n, sources
    csr.close()


def test_c5_bfs_full_all_bench_sources(c5):
    csr, rp, ci, n, sources = c5
    out = torch.empty(n, dtype=torch.int32, device=DEV)
    for src in sources:
        d, st = atos.bfs(csr, src, out=out)
        got = as_u32(d)
        assert oracle.validate_bfs(rp, ci, src, got) == 0, src
        np.testing.assert_array_equal(got, oracle.bfs(rp, ci, src), err_msg=f"source {src}")


def test_c5_pagerank_residual_certificate(c5):
    """C5 PageRank at eps = 1e-6 in the bench's launch configuration (library defaults: degree layout).
    x* - x = (I - a P^T)^{-1} r with r = (1-a)1 + a P^T x - x (Alg.4's residue), and
    (I - a P^T)^{-1} >= 0 with (I - a P^T)^{-1} 1 = x*/(1-a).  So
      -eta <= r <= eps + eta  elementwise   =>   -eta x*/(1-a) <= x* - x <= (eps + eta) x*/(1-a),
    i.e. every rank within (eps + eta)/(1-a) = 6.7e-6 relative and L1(x/n) <= 6.7e-6 (north star: 1e-4, 1e-5).
    eta = 1e-12 * max(1, x_w) absorbs the fp64 rounding of the ranks themselves (red.add accumulation)."""
    csr, rp, ci, n, _ = c5
    eps, alpha = 1e-6, 0.85
    assert csr.layout == "degree"
    r, st = atos.pagerank(csr, alpha, eps)
    x = r.cpu().numpy() * n  # n = 2^26: exact scaling
    res = oracle.pagerank_residual(rp, ci, x, alpha)
    eta = 1e-12 * np.maximum(1.0, x)
    assert np.all(res >= -eta), f"min residual {res.min()} (rank above the fixed point)"
    assert np.all(res <= eps + eta), f"max residual {res.max()} > eps"
    # the certificate's consequences, stated as the north-star tolerances
    rel_bound = (eps + eta.max()) / (1 - alpha)
    assert rel_bound < 1e-4
    assert rel_bound * (x.sum() + res.sum() / (1 - alpha)) / n < 1e-5  # L1(x/n) <= rel_bound * sum(x*)/n
    # conservation (symmetric graph): sum x + sum r/(1-a) = n - a #isolated, with the library's residues
    iso = int(np.sum(np.diff(rp) == 0))
    assert abs(x.sum() + st["residual_sum"] / (1 - alpha) - (n - alpha * iso)) < 1e-9 * n
    # and the library's residual sum agrees with the certificate's
    assert abs(st["residual_sum"] - res.sum()) < 1e-6 * n


@pytest.mark.parametrize("P", [2, 8])
def test_c5_partitioned_bfs_vs_oracle(c5, P):
    """The bench's partitioned C5 lines (exchange rounds and barrier-free over P loopback partitions) against
    the ORACLE, not only against the single-partition result."""
    csr, rp, ci, n, sources = c5
    src = sources[0]
    want = oracle.bfs(rp, ci, src)
    pc = atos.CSR(torch.from_numpy(rp), torch.from_numpy(ci), num_parts=P)
    out = torch.empty(n, dtype=torch.int32, device=DEV)
    d, st = atos.bfs(pc, src, out=out)
    np.testing.assert_array_equal(as_u32(d), want)
    d, st = atos.bfs(pc, src, out=out, barrier_free=1)
    np.testing.assert_array_equal(as_u32(d), want)
    pc.close()
