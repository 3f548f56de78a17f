"""Host logic of the paced online validation (SURVEY.md §8(d) "sustained 30-FPS streams"): the verdict that decides
whether a stream count is sustained. CPU only."""
import numpy as np

from paper_conf_icpp_zhangcjzly18_b200.online import sustained_verdict


def _flat(S, seconds=30.0, level=2.0, slope=0.0, dt=0.025):
    t = np.arange(0.0, seconds, dt)
    return t, S * level + slope * t


def test_steady_run_is_sustained():
    t, v = _flat(1000)
    r = sustained_verdict(10000, 10000, 0.2, t, v, 1000, 30.0)
    assert r["sustained"] and r["decided_fraction_of_window"] == 1.0 and abs(r["backlog_slope_frames_per_s"]) < 1e-6


def test_latency_over_budget_fails():
    t, v = _flat(10)
    assert not sustained_verdict(100, 100, 1.5, t, v, 10, 30.0)["sustained"]


def test_undecided_frames_fail_at_99_percent():
    t, v = _flat(10)
    assert sustained_verdict(1000, 990, 0.1, t, v, 10, 30.0)["sustained"]       # exactly 99 %
    assert not sustained_verdict(1000, 989, 0.1, t, v, 10, 30.0)["sustained"]   # a runtime at 98.9 % of the load


def test_growing_backlog_fails_even_when_latency_and_decisions_pass():
    S = 1000
    # 0.1 frame per stream per second of growth over the last 10 s (1 frame per stream in 10 s): not sustained
    t, v = _flat(S, slope=0.1 * S)
    r = sustained_verdict(100000, 100000, 0.3, t, v, S, 30.0)
    assert not r["sustained"] and abs(r["backlog_slope_per_stream"] - 0.1) < 1e-6
    # growth only before the last 10 s does not count
    t = np.arange(0.0, 30.0, 0.025)
    v = np.where(t < 15.0, S * 0.2 * t, S * 3.0)
    assert sustained_verdict(100000, 100000, 0.3, t, v, S, 30.0)["sustained"]


def test_short_rung_uses_half_the_run():
    t, v = _flat(100, seconds=4.0)
    r = sustained_verdict(100, 100, 0.1, t, v, 100, 4.0)
    assert r["tail_seconds"] == 2.0 and r["sustained"]
