"""Normalized throughput of Figs. 1-3 from a timeline table -- CPU checks of the arithmetic."""
import numpy as np
import pytest

from paper_conf_icpp_chenbpbyo22_b200 import analysis


def test_throughput_series_constant_rate():
    t = np.arange(0, 100, 5.0)
    done = 3.0 * t  # 3 tasks per microsecond
    tab = np.stack([t * 1e3, done, done + 10, done], axis=1)  # timeline rows carry nanoseconds
    mid, tp = analysis.throughput_series(tab)
    np.testing.assert_allclose(mid, t[1:] - 2.5)
    np.testing.assert_allclose(tp, 3.0)
    # integrating the throughput recovers the tasks done between the first and last sample
    assert abs(np.sum(tp * np.diff(t)) - (done[-1] - done[0])) < 1e-9


def test_normalized_divides_by_overwork_and_skips_repeated_timestamps():
    tab = np.array([[0, 0, 0, 0], [10e3, 100, 0, 0], [10e3, 100, 0, 0], [30e3, 300, 0, 0]], dtype=np.float64)
    t, nt = analysis.normalized_throughput(tab, 2.0)
    np.testing.assert_allclose(t, [5.0, 20.0])
    np.testing.assert_allclose(nt, [5.0, 5.0])


def test_overwork_factor_definitions():
    assert analysis.overwork_factor("bfs", 150, bsp_pops=100) == 1.5  # Table 4 upper: vs BSP
    assert analysis.overwork_factor("gc", 2_000, n=1_000) == 2.0     # Table 4 lower: vs |V|
    with pytest.raises(ValueError):
        analysis.overwork_factor("pr", 10)
    with pytest.raises(ValueError):
        analysis.normalized_throughput(np.zeros((3, 4)), 0.0)
