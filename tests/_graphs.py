"""Tiny named graphs for oracle pins, built from explicit edge lists (numpy only).

These fixtures are independent of both the oracle and the product path: each
graph is written out from its textbook definition so closed forms can be
checked against it.
"""
from __future__ import annotations

import itertools

import numpy as np


def csr_from_edges(n, edges, symmetric=False, dedupe=True, keep_self_loops=False):
    """CSR (int64 row_ptr, int32 col) with rows sorted by neighbour id."""
    e = np.asarray(list(edges), dtype=np.int64).reshape(-1, 2)
    if symmetric and len(e):
        e = np.concatenate([e, e[:, ::-1]], axis=0)
    if not keep_self_loops and len(e):
        e = e[e[:, 0] != e[:, 1]]
    if dedupe and len(e):
        e = np.unique(e, axis=0)
    elif len(e):
        e = e[np.lexsort((e[:, 1], e[:, 0]))]
    counts = np.bincount(e[:, 0], minlength=n) if len(e) else np.zeros(n, dtype=np.int64)
    row_ptr = np.zeros(n + 1, dtype=np.int64)
    row_ptr[1:] = np.cumsum(counts)
    col = e[:, 1].astype(np.int32) if len(e) else np.zeros(0, dtype=np.int32)
    return row_ptr, col


def path(n):
    return csr_from_edges(n, [(i, i + 1) for i in range(n - 1)], symmetric=True)


def cycle(n):
    return csr_from_edges(n, [(i, (i + 1) % n) for i in range(n)], symmetric=True)


def star(n):
    """centre 0, leaves 1..n-1"""
    return csr_from_edges(n, [(0, i) for i in range(1, n)], symmetric=True)


def complete(n):
    return csr_from_edges(n, [(i, j) for i in range(n) for j in range(n) if i != j])


def grid(R, C):
    """4-neighbour R x C grid, row-major ids v = r*C + c."""
    edges = []
    for r in range(R):
        for c in range(C):
            v = r * C + c
            if c + 1 < C:
                edges.append((v, v + 1))
            if r + 1 < R:
                edges.append((v, v + C))
    return csr_from_edges(R * C, edges, symmetric=True)


def torus(R, C):
    edges = []
    for r in range(R):
        for c in range(C):
            v = r * C + c
            edges.append((v, r * C + (c + 1) % C))
            edges.append((v, ((r + 1) % R) * C + c))
    return csr_from_edges(R * C, edges, symmetric=True)


def hypercube(d):
    n = 1 << d
    return csr_from_edges(n, [(v, v ^ (1 << b)) for v in range(n) for b in range(d)])


def petersen():
    outer = [(i, (i + 1) % 5) for i in range(5)]
    spokes = [(i, i + 5) for i in range(5)]
    inner = [(5 + i, 5 + (i + 2) % 5) for i in range(5)]
    return csr_from_edges(10, outer + spokes + inner, symmetric=True)


def wheel(rim):
    """hub 0 + cycle on 1..rim"""
    edges = [(0, i) for i in range(1, rim + 1)] + [(i, i % rim + 1) for i in range(1, rim + 1)]
    return csr_from_edges(rim + 1, edges, symmetric=True)


def grotzsch():
    """Mycielskian of C5: 11 vertices, triangle-free, chromatic number 4."""
    c5 = [(i, (i + 1) % 5) for i in range(5)]
    edges = list(c5)
    for (a, b) in c5:  # u_i adjacent to neighbours of v_i
        edges.append((5 + a, b))
        edges.append((5 + b, a))
    edges += [(10, 5 + i) for i in range(5)]
    return csr_from_edges(11, edges, symmetric=True)


def crown(k):
    """K_{k,k} minus a perfect matching: u_i = 2i, v_i = 2i+1 (interleaved ids)."""
    edges = [(2 * i, 2 * j + 1) for i in range(k) for j in range(k) if i != j]
    return csr_from_edges(2 * k, edges, symmetric=True)


def gnp(n, p, seed, directed=False):
    rng = np.random.default_rng(seed)
    if directed:
        edges = [(i, j) for i in range(n) for j in range(n) if i != j and rng.random() < p]
        return csr_from_edges(n, edges)
    edges = [(i, j) for i, j in itertools.combinations(range(n), 2) if rng.random() < p]
    return csr_from_edges(n, edges, symmetric=True)


def to_dense(row_ptr, col):
    n = len(row_ptr) - 1
    A = np.zeros((n, n), dtype=np.float64)
    for v in range(n):
        for e in range(row_ptr[v], row_ptr[v + 1]):
            A[v, col[e]] += 1.0
    return A
