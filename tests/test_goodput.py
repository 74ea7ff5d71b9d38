"""The goodput simulation (f4) against the paper's Eq 4 recovery bound (oracle/manager_model)."""
import pytest

from oracle.manager_model import recovery_bound
from tools.goodput import simulate


@pytest.mark.parametrize("f,tw,N", [(10, 0.02, 2), (1, 0.05, 2), (5, 0.3, 1), (20, 0.5, 4)])
def test_lost_iterations_within_eq4(f, tw, N):
    t = 0.017
    r = simulate(t, f, tw, l=0.0, rate=1 / 20.0, horizon=2000.0, n_inflight=N, seed=3)
    assert r["failures"] > 10
    # Eq 4 bounds the redone time (l = 0 here): f*t + t*min(N*f, Tw/t), plus the iteration in progress
    bound_iters = recovery_bound(0.0, t, f, N, tw) / t + 1
    assert r["max_lost_iters"] <= bound_iters + 1e-9


def test_no_failures_is_ideal_minus_slowdown():
    r = simulate(0.01, 10, 0.02, 0.1, rate=0.0, horizon=100.0, slowdown_pct=2.0)
    assert r["failures"] == 0
    assert abs(r["useful_iters"] - 100.0 / (0.01 * 1.02)) <= 2
