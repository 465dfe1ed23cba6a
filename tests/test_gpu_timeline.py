"""cfg.timeline (the progress samples behind Figs. 1-3): the samples are monotone in time and in
the done / tail / head counters, done never exceeds tail, and the final sample's done equals the run's
task count -- so the normalized throughput (analysis.normalized_throughput) integrates to the real work."""
import numpy as np
import pytest
import torch

import paper_conf_icpp_chenbpbyo22_b200 as atos
from paper_conf_icpp_chenbpbyo22_b200 import analysis, gen

from _gpu import DEV

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("app", ["bfs", "pr", "gc"])
def test_timeline_samples(app):
    g = gen.rmat(18, 16, seed=3, device=DEV)
    csr = atos.CSR.from_graph(g)
    cap = 1 << 14
    tl = torch.zeros(4 * cap, dtype=torch.int64, device=DEV)
    knobs = dict(timeline=tl, timeline_interval_ns=2000)
    if app == "bfs":
        _, st = atos.bfs(csr, gen.pick_source(g, 1), **knobs)
        _, sb = atos.bfs_bsp(csr, gen.pick_source(g, 1))
    elif app == "pr":
        _, st = atos.pagerank(csr, 0.85, 1e-6, **knobs)
        _, sb = atos.pagerank_bsp(csr, 0.85, 1e-6)
    else:
        _, st = atos.color(csr, 1, **knobs)
        sb = None
    assert 2 <= st["timeline_len"] <= cap
    tab = atos.timeline_table(tl, st).numpy()
    # samplers race only at interval boundaries: rows are time-ordered up to rare swaps, and each row's
    # three counters are relaxed reads taken one after another -- so check the series in time order, with
    # a small allowance for those swaps, and the exact closing sample
    tab = tab[np.argsort(tab[:, 0], kind="stable")]
    t, done, tail, head = tab[:, 0], tab[:, 1], tab[:, 2], tab[:, 3]
    for series in (done, tail, head):
        assert np.mean(np.diff(series) < 0) <= 0.02
    assert done[-1] == done.max() and tail[-1] == tail.max()
    assert np.all(done <= tail)
    # every task of the run completes before the last worker exits; the last sample is taken at exit
    # (Worker::complete samples after each batch), so it sees all of them relative to the first sample
    first_done = done[0]
    assert done[-1] - first_done <= st["pops"]
    assert done[-1] - first_done >= 0.95 * st["pops"]
    ow = analysis.overwork_factor(app, st["pops"], bsp_pops=sb["pops"] if sb else None, n=g.n)
    tt, nt = analysis.normalized_throughput(tab, ow)
    assert np.mean(nt < 0) <= 0.02
    dt_us = np.diff(t)[np.diff(t) > 0] / 1e3
    # the normalized series integrates back to the tasks done between the first and last sample
    assert abs(np.sum(nt * dt_us) * ow - (done[-1] - done[0])) < 1e-6 * max(1, done[-1])
