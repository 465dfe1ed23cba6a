"""GPU: atos_color must always return a valid colouring (BASELINE north_star) --
every vertex coloured, no edge u != w with equal colours, color[v] <= deg(v).
The colour COUNT is parity-unpinned (the method is a speculative heuristic,
P:689-717); it is compared loosely with the oracle's greedy / JP counts."""
import numpy as np
import pytest

import oracle
import paper_conf_icpp_chenbpbyo22_b200 as atos
from paper_conf_icpp_chenbpbyo22_b200 import gen

import _graphs as G
from _gpu import DEV, csr_of

pytestmark = pytest.mark.gpu

KNOBS = [
    dict(worker=32, fetch_size=1),
    dict(worker=32, fetch_size=8),
    dict(worker=256, fetch_size=256),
    dict(worker=512, fetch_size=64),
    dict(worker=1, fetch_size=1),
    dict(worker=1, fetch_size=2),
    dict(worker=32, fetch_size=4, persistent=0),
    dict(worker=256, fetch_size=256, persistent=0),
    dict(worker=1, fetch_size=1, persistent=0),
    dict(worker=32, fetch_size=8, permute_init=1),
    dict(worker=256, fetch_size=128, permute_init=1),
    dict(worker=1024, fetch_size=128, conflict_policy=2),  # hash-only priority
    dict(worker=32, fetch_size=8, conflict_policy=2),
]


def kid(k):
    return "-".join(f"{a}{b}" for a, b in k.items())


def check_color(rp, ci, c, st):
    col = c.cpu().numpy()
    assert oracle.validate_color(rp, ci, col) == 0
    assert st["colors_used"] == col.max() + 1
    return int(col.max() + 1)


@pytest.fixture(scope="module")
def rmat13():
    g = gen.rmat(13, 32, seed=4)
    rp, ci = g.numpy()
    return rp, ci, atos.CSR.from_graph(g.to(DEV))


@pytest.mark.parametrize("knobs", KNOBS, ids=kid)
def test_rmat_valid(rmat13, knobs):
    rp, ci, csr = rmat13
    c, st = atos.color(csr, seed=1, **knobs)
    k = check_color(rp, ci, c, st)
    _, kg = oracle.color_greedy(rp, ci)
    assert k <= np.diff(rp).max() + 1
    assert st["pops"] >= 2 * (len(rp) - 1)  # one assign + one check per vertex at least
    print(f"colours gpu={k} greedy={kg} tasks/n={st['pops'] / (len(rp) - 1):.3f}")


@pytest.mark.parametrize("name", ["K40", "petersen", "grid", "star", "crown", "cycle_odd", "empty_rows"])
def test_named(name):
    rp, ci = {
        "K40": G.complete(40), "petersen": G.petersen(), "grid": G.grid(60, 70), "star": G.star(5000),
        "crown": G.crown(30), "cycle_odd": G.cycle(10001),
        "empty_rows": G.csr_from_edges(100, [(3, 4), (4, 5)], symmetric=True),
    }[name]
    csr = csr_of(rp, ci)
    for knobs in KNOBS:
        c, st = atos.color(csr, seed=3, **knobs)
        k = check_color(rp, ci, c, st)
        if name == "K40":
            assert k == 40


def test_literal_policy():
    """Paper-literal policy (both endpoints re-queue themselves) may
    livelock when two adjacent vertices keep recolouring in lock step (DESIGN.md
    R-GC-2); it must then stop with ATOS_ERR_TIMEOUT, never hang, and a result it
    does return must be valid."""
    g = gen.rmat(12, 16, seed=8)
    rp, ci = g.numpy()
    csr = atos.CSR.from_graph(g.to(DEV))
    for knobs in (dict(worker=32), dict(worker=256), dict(worker=1)):
        try:
            c, st = atos.color(csr, seed=1, conflict_policy=1, timeout_s=3.0, **knobs)
        except RuntimeError as e:
            assert "TIMEOUT" in str(e)
            continue
        check_color(rp, ci, c, st)
    # the handle stays usable after a timeout
    c, st = atos.color(csr, seed=1)
    check_color(rp, ci, c, st)


def test_mesh_road():
    g = gen.mesh(300, 300, keep_prob=0.6, seed=2)
    rp, ci = g.numpy()
    csr = atos.CSR.from_graph(g.to(DEV))
    for knobs in KNOBS[:3]:
        c, st = atos.color(csr, seed=2, **knobs)
        assert check_color(rp, ci, c, st) <= 5


def test_not_symmetric_rejected():
    rp, ci = G.csr_from_edges(4, [(0, 1), (1, 2)])
    csr = csr_of(rp, ci)
    with pytest.raises(RuntimeError, match="NOT_SYMMETRIC"):
        atos.color(csr, seed=1, validate=1)


def test_host_output():
    import torch
    g = gen.rmat(11, 16, seed=9)
    rp, ci = g.numpy()
    csr = atos.CSR.from_graph(g.to(DEV))
    out = torch.empty(g.n, dtype=torch.int32)
    c, st = atos.color(csr, seed=5, out=out)
    check_color(rp, ci, c, st)


@pytest.mark.parametrize("layout", ["input", "auto", "degree"])
def test_layout_modes_valid(layout):
    g = gen.rmat(12, 32, seed=8)
    rp, ci = g.numpy()
    csr = atos.CSR.from_graph(g.to(DEV), layout=layout)
    for knobs in (dict(), dict(permute_init=1), dict(worker=32, fetch_size=8)):
        c, st = atos.color(csr, seed=3, **knobs)
        check_color(rp, ci, c, st)
        c, st = atos.color_bsp(csr, seed=3)
        check_color(rp, ci, c, st)


@pytest.mark.parametrize("spread", [2, 8, 64])
def test_recolor_spread_valid(rmat13, spread):
    """cfg.recolor_spread (R-GC-10): still a proper colouring with colour <= deg(v) for every vertex (the
    j-th free colour is taken among [0, deg(v)]); the dense Kronecker core exercises repeated recolours."""
    rp, ci, csr = rmat13
    for seed in (1, 2):
        c, st = atos.color(csr, seed, recolor_spread=spread)
        assert oracle.validate_color(rp, ci, c.cpu().numpy()) == 0
        assert st["colors_used"] == int(c.max().item()) + 1
    with pytest.raises(RuntimeError, match="INVALID_ARG"):
        atos.color(csr, 1, recolor_spread=65)
