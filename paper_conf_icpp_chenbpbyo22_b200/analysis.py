"""Analysis helpers for the paper's design-space study (host-side; not on the hot path).

Normalized throughput (the y axis of Figs. 1-3): "the measured throughput divided by
the overwork factors in Table 4" -- the overwork factor being the workload relative to the BSP
implementation for BFS and PageRank, and relative to |V| for colouring (Table 4).  Here
the workload unit is the task (a popped vertex, stats.pops), the BSP workload comes from the
in-framework BSP baselines (atos_*_bsp, stats.pops = frontier items processed), and the throughput
over time comes from the cfg.timeline samples (globaltimer ns, tasks done, queue tail, queue head)
the workers take every timeline_interval_ns.
"""
from __future__ import annotations

import numpy as np


def overwork_factor(app: str, pops: int, bsp_pops: int | None = None, n: int | None = None) -> float:
    """Table 4's ratio: Atos tasks / BSP tasks (BFS, PageRank) or tasks / |V| (colouring)."""
    if app in ("bfs", "pr", "pagerank"):
        if not bsp_pops:
            raise ValueError("BFS / PageRank overwork needs the BSP baseline's task count")
        return pops / bsp_pops
    if app in ("gc", "color"):
        if not n:
            raise ValueError("colouring overwork needs |V|")
        return pops / n
    raise ValueError(f"unknown app {app!r}")


def throughput_series(table) -> tuple[np.ndarray, np.ndarray]:
    """(t_us at interval mid-points, tasks completed per microsecond) from a timeline table
    (rows: globaltimer ns since the first sample, done, tail, head -- see timeline_table())."""
    tab = np.asarray(table, dtype=np.float64)
    tab = tab[np.argsort(tab[:, 0], kind="stable")]  # samplers of adjacent intervals can land out of order
    t = tab[:, 0] / 1e3
    done = tab[:, 1]
    if t.size < 2:
        return np.zeros(0), np.zeros(0)
    dt = np.diff(t)
    keep = dt > 0
    mid = (t[1:] + t[:-1]) / 2
    return mid[keep], np.diff(done)[keep] / dt[keep]


def normalized_throughput(table, overwork: float) -> tuple[np.ndarray, np.ndarray]:
    """Figs. 1-3: measured throughput / overwork factor, over time."""
    if overwork <= 0:
        raise ValueError("overwork factor must be positive")
    t, tp = throughput_series(table)
    return t, tp / overwork
