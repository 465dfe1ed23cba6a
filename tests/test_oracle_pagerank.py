"""Pins for oracle.pagerank_jacobi / oracle.pagerank_push (CPU).

Definition pinned (DESIGN.md R-PR-1): x = (1-a)1 + a P^T x, output x/n.
 * regular graphs (cycle, complete, hypercube, torus): x = 1  ->  rank = 1/n;
 * star S_n: x_c = (1 + a(n-1))/(1+a), x_leaf = (1-a) + a x_c/(n-1);
 * hand-solved 3-vertex graph with a dangling vertex (tests/golden);
 * dense LU solve (numpy.linalg.solve) of (I - a P^T) x = (1-a) 1 for n <= 200,
   with multi-edges and dangling vertices;
 * the serial push oracle (Alg.3 init + Alg.4) must land
   inside the proven one-sided band 0 <= x* - x <= eps x*/(1-a) and satisfy
   conservation  sum x + sum r/(1-a) = n - a * #isolated  on symmetric graphs.
"""
import json
import os

import numpy as np
import pytest

import oracle
import _graphs as G

A = 0.85
GOLD = os.path.join(os.path.dirname(__file__), "golden")


def dense_solve(rp, ci, alpha=A):
    n = len(rp) - 1
    Adj = G.to_dense(rp, ci)
    deg = Adj.sum(axis=1)
    P = np.zeros_like(Adj)
    nz = deg > 0
    P[nz] = Adj[nz] / deg[nz, None]
    x = np.linalg.solve(np.eye(n) - alpha * P.T, (1 - alpha) * np.ones(n))
    return x


@pytest.mark.parametrize("g", ["cycle", "complete", "hypercube", "torus"])
def test_regular_graphs_are_uniform(g):
    rp, ci = {"cycle": G.cycle(37), "complete": G.complete(12), "hypercube": G.hypercube(6),
              "torus": G.torus(9, 11)}[g]
    n = len(rp) - 1
    r, it, ok = oracle.pagerank_jacobi(rp, ci, A)
    assert ok
    np.testing.assert_allclose(r, 1.0 / n, rtol=1e-12)


@pytest.mark.parametrize("n", [2, 5, 50, 301])
def test_star_closed_form(n):
    rp, ci = G.star(n)
    r, it, ok = oracle.pagerank_jacobi(rp, ci, A)
    assert ok
    xc = (1 + A * (n - 1)) / (1 + A)
    xl = (1 - A) + A * xc / (n - 1)
    np.testing.assert_allclose(r[0] * n, xc, rtol=1e-11)
    np.testing.assert_allclose(r[1:] * n, xl, rtol=1e-11)


def test_golden_three_vertex_dangling():
    g = json.load(open(os.path.join(GOLD, "pr_3vertex_dangling.json")))
    rp, ci = G.csr_from_edges(g["n"], g["edges"])
    r, it, ok = oracle.pagerank_jacobi(rp, ci, g["alpha"])
    assert ok
    np.testing.assert_allclose(r * g["n"], g["x"], rtol=1e-12)
    p, res, pops = oracle.pagerank_push(rp, ci, g["alpha"], 1e-12)
    np.testing.assert_allclose(p * g["n"], g["x"], rtol=1e-10)


@pytest.mark.parametrize("seed", range(6))
def test_dense_lu(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(20, 200))
    m = int(n * rng.uniform(1.0, 5.0))
    src = rng.integers(0, n, m)
    dst = rng.integers(0, n, m)
    # keep multi-edges and self loops (R-PR-9); some vertices dangle
    rp, ci = G.csr_from_edges(n, zip(src, dst), dedupe=False, keep_self_loops=True)
    x = dense_solve(rp, ci)
    r, it, ok = oracle.pagerank_jacobi(rp, ci, A)
    assert ok
    np.testing.assert_allclose(r * n, x, rtol=1e-11, atol=0)


def test_iterates_monotone_bound():
    """Jacobi with a loose tol stays below x* and within tol*x*/(1-a) (R-PR-oracle)."""
    rp, ci = G.gnp(120, 0.05, seed=11)
    n = 120
    x = dense_solve(rp, ci)
    for tol in (1e-3, 1e-6, 1e-9):
        r, it, ok = oracle.pagerank_jacobi(rp, ci, A, tol=tol)
        gap = x - r * n
        assert np.all(gap >= -1e-12)
        assert np.all(gap <= tol * x / (1 - A) + 1e-12)


@pytest.mark.parametrize("seed", range(5))
@pytest.mark.parametrize("eps", [1e-3, 1e-6])
def test_push_oracle_band_and_conservation(seed, eps):
    rp, ci = G.gnp(150 + 10 * seed, 0.04, seed=20 + seed)
    n = len(rp) - 1
    deg = np.diff(rp)
    xstar = dense_solve(rp, ci)
    p, res, pops = oracle.pagerank_push(rp, ci, A, eps)
    x = p * n
    assert np.all(res >= 0) and np.all(res <= eps)
    gap = xstar - x
    assert np.all(gap >= -1e-10)
    assert np.all(gap <= eps * xstar / (1 - A) + 1e-10)
    iso = int(np.sum(deg == 0))
    assert abs(x.sum() + res.sum() / (1 - A) - (n - A * iso)) < 1e-9 * n


def test_push_matches_jacobi_on_regular():
    rp, ci = G.torus(20, 20)
    p, res, pops = oracle.pagerank_push(rp, ci, A, 1e-10)
    np.testing.assert_allclose(p * 400, 1.0, rtol=1e-8)
    # no vertex is ever pushed on a regular graph after init? no: every vertex starts with
    # residue a(1-a) > eps, so pops >= n
    assert pops >= 400


def test_bad_args():
    rp, ci = G.cycle(5)
    with pytest.raises(ValueError):
        oracle.pagerank_jacobi(rp, ci, 1.5)
    with pytest.raises(ValueError):
        oracle.pagerank_push(rp, ci, 0.85, 0.0)


# ---- oracle.pagerank_residual: r = (1-a)1 + a P^T x - x (the certificate used at C5 size) ----------

def test_residual_golden_hand_values():
    g = json.load(open(os.path.join(GOLD, "pr_residual_3vertex.json")))
    rp, ci = G.csr_from_edges(g["n"], g["edges"])
    r = oracle.pagerank_residual(rp, ci, g["x"], g["alpha"])
    np.testing.assert_allclose(r, g["r"], rtol=0, atol=1e-15)


def test_residual_zero_at_golden_fixed_point():
    g = json.load(open(os.path.join(GOLD, "pr_3vertex_dangling.json")))
    rp, ci = G.csr_from_edges(g["n"], g["edges"])
    r = oracle.pagerank_residual(rp, ci, g["x"], g["alpha"])
    np.testing.assert_allclose(r, 0.0, atol=1e-15)


@pytest.mark.parametrize("n", [3, 11, 200])
def test_residual_star_closed_form(n):
    """Star at x = 1: centre r = (1-a) + a(n-1) - 1 = a(n-2); leaf r = (1-a) + a/(n-1) - 1."""
    rp, ci = G.star(n)
    r = oracle.pagerank_residual(rp, ci, np.ones(n), A)
    np.testing.assert_allclose(r[0], A * (n - 2), rtol=1e-14)
    np.testing.assert_allclose(r[1:], A / (n - 1) - A, rtol=1e-13)


@pytest.mark.parametrize("seed", range(4))
def test_residual_vs_dense_and_push(seed):
    """Against the dense matrix (multi-edges, self loops, dangling rows) at a random x; at the LU
    solution r = 0; and the push oracle's own residue array equals the residual of its ranks
    (the invariant x* = x + (I - a P^T)^{-1} r that the GPU certificate relies on)."""
    rng = np.random.default_rng(100 + seed)
    n = int(rng.integers(20, 150))
    m = int(n * rng.uniform(1.0, 4.0))
    rp, ci = G.csr_from_edges(n, zip(rng.integers(0, n, m), rng.integers(0, n, m)), dedupe=False,
                              keep_self_loops=True)
    Adj = G.to_dense(rp, ci)
    deg = Adj.sum(axis=1)
    P = np.zeros_like(Adj)
    P[deg > 0] = Adj[deg > 0] / deg[deg > 0, None]
    x = rng.uniform(0.1, 3.0, n)
    want = (1 - A) + A * (P.T @ x) - x
    np.testing.assert_allclose(oracle.pagerank_residual(rp, ci, x, A), want, rtol=1e-12, atol=1e-13)
    xs = dense_solve(rp, ci)
    assert np.max(np.abs(oracle.pagerank_residual(rp, ci, xs, A))) < 1e-12
    p, res, pops = oracle.pagerank_push(rp, ci, A, 1e-6)
    np.testing.assert_allclose(oracle.pagerank_residual(rp, ci, p * n, A), res, rtol=0, atol=1e-12)


def test_residual_at_jacobi_result_is_below_tol():
    """Jacobi stops when |x^{k+1}-x^k|_inf <= tol; its last increment is the residual of x^k, and the residual of
    x^{k+1} is a P^T of that increment -- so 0 <= r <= tol elementwise (monotone iterates, R-PR-oracle)."""
    rp, ci = G.gnp(300, 0.03, seed=5)
    for tol in (1e-4, 1e-8):
        r_, it, ok = oracle.pagerank_jacobi(rp, ci, A, tol=tol)
        r = oracle.pagerank_residual(rp, ci, r_ * 300, A)
        assert np.all(r >= -1e-13) and np.all(r <= tol + 1e-13)


def test_residual_bad_args():
    rp, ci = G.cycle(5)
    with pytest.raises(ValueError):
        oracle.pagerank_residual(rp, ci, np.ones(4), A)
    with pytest.raises(ValueError):
        oracle.pagerank_residual(rp, ci, np.ones(5), 1.0)
