"""Pins for the colouring oracle (CPU).

 * brute-force chromatic number (backtracking, n <= 11) of textbook graphs must
   equal the golden values (tests/golden/chromatic_numbers.json), and every
   oracle colouring uses >= chi colours and passes the validator;
 * greedy on complete graphs uses n colours; on a row-major bipartite grid
   exactly 2 (every vertex's earlier neighbours sit on the other parity class);
 * crown graph: interleaved order forces k colours, sides-first order 2
   (classic worst case of first-fit);
 * Jones-Plassmann by priority order == literal round-based JP simulation;
 * the validator rejects conflicts and uncoloured vertices.
The GPU colour count is parity-unpinned (any proper colouring is valid).
"""
import json
import os

import numpy as np
import pytest

import oracle
import _graphs as G

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def chromatic_number(rp, ci):
    n = len(rp) - 1
    adj = [set(int(w) for w in ci[rp[v]:rp[v + 1]] if w != v) for v in range(n)]
    order = sorted(range(n), key=lambda v: -len(adj[v]))

    def colourable(k):
        col = [-1] * n

        def bt(i):
            if i == n:
                return True
            v = order[i]
            used = {col[w] for w in adj[v]}
            for c in range(k):
                if c not in used:
                    col[v] = c
                    if bt(i + 1):
                        return True
            col[v] = -1
            return False
        return bt(0)

    k = 1
    while not colourable(k):
        k += 1
    return k


NAMED = {
    "K5": lambda: G.complete(5), "K7": lambda: G.complete(7), "C8": lambda: G.cycle(8),
    "C9": lambda: G.cycle(9), "petersen": G.petersen, "wheel6": lambda: G.wheel(6),
    "wheel7": lambda: G.wheel(7), "grotzsch": G.grotzsch,
}


@pytest.mark.parametrize("name", list(NAMED))
def test_bruteforce_chi_and_oracle(name):
    gold = json.load(open(os.path.join(GOLD, "chromatic_numbers.json")))["graphs"]
    rp, ci = NAMED[name]()
    chi = chromatic_number(rp, ci)
    assert chi == gold[name]
    c, k = oracle.color_greedy(rp, ci)
    assert oracle.validate_color(rp, ci, c) == 0
    assert k >= chi and k == c.max() + 1
    c, k = oracle.color_jp(rp, ci, seed=5)
    assert oracle.validate_color(rp, ci, c) == 0 and k >= chi


@pytest.mark.parametrize("seed", range(4))
def test_random_gnp10(seed):
    rp, ci = G.gnp(10, 0.5, seed=seed)
    chi = chromatic_number(rp, ci)
    for order_seed in range(3):
        order = np.random.default_rng(order_seed).permutation(10)
        c, k = oracle.color_greedy(rp, ci, order)
        assert oracle.validate_color(rp, ci, c) == 0 and k >= chi


def test_complete_and_grid():
    rp, ci = G.complete(13)
    c, k = oracle.color_greedy(rp, ci)
    assert k == 13 and sorted(c.tolist()) == list(range(13))
    rp, ci = G.grid(20, 33)
    c, k = oracle.color_greedy(rp, ci)
    r, cc = np.divmod(np.arange(20 * 33), 33)
    np.testing.assert_array_equal(c, (r + cc) % 2)
    assert k == 2


def test_crown_worst_case():
    k = 9
    rp, ci = G.crown(k)
    c, ncol = oracle.color_greedy(rp, ci)  # interleaved u0 v0 u1 v1 ...
    assert ncol == k
    order = np.concatenate([np.arange(0, 2 * k, 2), np.arange(1, 2 * k, 2)])
    c, ncol = oracle.color_greedy(rp, ci, order)
    assert ncol == 2


@pytest.mark.parametrize("seed", range(6))
def test_jp_equals_rounds(seed):
    rp, ci = G.gnp(60, 0.1, seed=40 + seed)
    a, ka = oracle.color_jp(rp, ci, seed)
    b, kb = oracle.color_jp_rounds(rp, ci, seed)
    np.testing.assert_array_equal(a, b)
    assert ka == kb
    assert oracle.validate_color(rp, ci, a) == 0


def test_splitmix64_reference_values():
    # splitmix64 outputs for state increments from seed 0 (Vigna's reference
    # sequence: next() with x=0 returns 0xE220A8397B1DCDAF, then 0x6E789E6AA1B965F4).
    assert oracle.splitmix64(0) == 0xE220A8397B1DCDAF
    assert oracle.splitmix64(0x9E3779B97F4A7C15) == 0x6E789E6AA1B965F4


def test_validator_rejects():
    rp, ci = G.petersen()
    c, k = oracle.color_greedy(rp, ci)
    bad = c.copy()
    w = ci[rp[0]]
    bad[0] = bad[w]
    assert oracle.validate_color(rp, ci, bad) == 2 or oracle.validate_color(rp, ci, bad) == 1
    bad = c.copy()
    bad[3] = -1
    assert oracle.validate_color(rp, ci, bad) == 1
    bad = c.copy()
    bad[4] = 1000
    assert oracle.validate_color(rp, ci, bad) == 1
