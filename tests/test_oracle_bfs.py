"""Pins for oracle.bfs / oracle.validate_bfs (CPU, no GPU).

The oracle's BFS is pinned against things other than itself:
 * Floyd-Warshall all-pairs shortest paths on every small graph (n <= 64),
   directed and undirected, connected and not;
 * closed forms: path |i-s|, cycle min(|i-s|, n-|i-s|), star, complete graph,
   R x C grid |r-r0| + |c-c0| (BFS depth = shortest-path length);
 * the Graph500-style validator must accept the oracle's answers and reject
   single-vertex perturbations (so a validator bug cannot hide an oracle bug).
"""
import numpy as np
import pytest

import oracle
import _graphs as G

U = 0xFFFFFFFF


def floyd_warshall(row_ptr, col):
    n = len(row_ptr) - 1
    INF = np.iinfo(np.int64).max // 4
    D = np.full((n, n), INF, dtype=np.int64)
    np.fill_diagonal(D, 0)
    for v in range(n):
        for e in range(row_ptr[v], row_ptr[v + 1]):
            if col[e] != v:
                D[v, col[e]] = 1
    for k in range(n):
        D = np.minimum(D, D[:, k:k + 1] + D[k:k + 1, :])
    out = np.where(D >= INF, U, D).astype(np.uint32)
    return out


def _small_graphs():
    gs = {
        "path9": G.path(9), "cycle10": G.cycle(10), "cycle11": G.cycle(11), "star7": G.star(7),
        "K6": G.complete(6), "grid5x7": G.grid(5, 7), "petersen": G.petersen(), "Q4": G.hypercube(4),
        "grotzsch": G.grotzsch(), "wheel8": G.wheel(8),
    }
    for s in range(6):
        gs[f"gnp_u{s}"] = G.gnp(40 + s * 4, 0.06, seed=s)
        gs[f"gnp_d{s}"] = G.gnp(30 + s * 6, 0.05, seed=100 + s, directed=True)
    # two disjoint components + isolated vertices
    gs["disconnected"] = G.csr_from_edges(12, [(0, 1), (1, 2), (2, 0), (5, 6), (6, 7)], symmetric=True)
    # directed chain: only forward reachability
    gs["dchain"] = G.csr_from_edges(6, [(0, 1), (1, 2), (2, 3), (3, 4), (4, 5)])
    # multi-edges and self-loops kept: must be harmless (R-BFS-4)
    gs["multi"] = G.csr_from_edges(5, [(0, 1), (0, 1), (1, 1), (1, 2), (2, 3), (3, 3), (3, 4)],
                                   dedupe=False, keep_self_loops=True)
    return gs


@pytest.mark.parametrize("name", list(_small_graphs().keys()))
def test_bfs_matches_floyd_warshall(name):
    rp, ci = _small_graphs()[name]
    n = len(rp) - 1
    D = floyd_warshall(rp, ci)
    for s in range(n):
        d = oracle.bfs(rp, ci, s)
        np.testing.assert_array_equal(d, D[s], err_msg=f"{name} src={s}")
        assert oracle.validate_bfs(rp, ci, s, d) == 0


def test_closed_forms():
    n = 50
    rp, ci = G.path(n)
    for s in (0, 17, 49):
        np.testing.assert_array_equal(oracle.bfs(rp, ci, s), np.abs(np.arange(n) - s))
    rp, ci = G.cycle(n)
    for s in (0, 13):
        k = np.abs(np.arange(n) - s)
        np.testing.assert_array_equal(oracle.bfs(rp, ci, s), np.minimum(k, n - k))
    rp, ci = G.star(20)
    d = oracle.bfs(rp, ci, 0)
    assert d[0] == 0 and np.all(d[1:] == 1)
    d = oracle.bfs(rp, ci, 5)
    assert d[5] == 0 and d[0] == 1 and np.all(np.delete(d, [0, 5]) == 2)
    rp, ci = G.complete(9)
    d = oracle.bfs(rp, ci, 3)
    assert d[3] == 0 and np.all(np.delete(d, 3) == 1)


@pytest.mark.parametrize("R,C,r0,c0", [(30, 40, 0, 0), (31, 17, 15, 8), (1, 60, 0, 33), (64, 64, 63, 0)])
def test_grid_closed_form(R, C, r0, c0):
    rp, ci = G.grid(R, C)
    d = oracle.bfs(rp, ci, r0 * C + c0)
    r, c = np.divmod(np.arange(R * C), C)
    np.testing.assert_array_equal(d, np.abs(r - r0) + np.abs(c - c0))


def test_validator_rejects_perturbations():
    rng = np.random.default_rng(7)
    rp, ci = G.gnp(60, 0.08, seed=3)
    d = oracle.bfs(rp, ci, 0)
    reached = np.flatnonzero((d != U) & (np.arange(60) != 0))
    assert len(reached) > 10
    for _ in range(20):
        v = rng.choice(reached)
        for delta in (+1, -1):
            bad = d.copy()
            bad[v] = int(bad[v]) + delta
            assert oracle.validate_bfs(rp, ci, 0, bad) != 0
        bad = d.copy()
        bad[v] = U
        assert oracle.validate_bfs(rp, ci, 0, bad) != 0
    bad = d.copy()
    bad[0] = 1
    assert oracle.validate_bfs(rp, ci, 0, bad) != 0


def test_empty_and_single():
    rp = np.zeros(2, dtype=np.int64)
    ci = np.zeros(0, dtype=np.int32)
    np.testing.assert_array_equal(oracle.bfs(rp, ci, 0), [0])
    with pytest.raises(ValueError):
        oracle.bfs(rp, ci, 1)
