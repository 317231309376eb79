"""Pins of the oracle's closed loop under gain mismatch (NEXT-4, §4.4)
against the closed-form pole analysis of tests/stability.py: the oracle must
converge to the predicted equilibrium p* within the rigorous delta-sigma
disturbance bound when |rho(g)| < 1, and must NOT settle when |rho(g)| > 1.
A wrong sign, a dropped c_0, a mis-scaled R, a plant gain applied to the model
instead of the plant, or a set point outside the true range fails one of them."""
import numpy as np
import pytest

from gen import configs
from tests import stability as ST

K = 300
W = 60


@pytest.fixture(scope="module", params=[(0.1, 1.0), (0.02, 0.25), (1e-3, 1.0)], ids=["r0.1q1", "r0.02q.25", "r1e-3q1"])
def sweep(oracle_mod, request):
    r0, q = request.param
    d = configs.stability_sweep(n_servers=6, n_gains=24, periods=K, r0=r0)
    d["controller"]["q"] = q
    o = oracle_mod.Oracle(d)
    ng = d["workload"]["n_caps"]
    out = o.simulate(np.arange(6 * ng), periods=K)
    return d, o, out


def test_identification_exact_when_noiseless(sweep):
    d, o, _ = sweep
    for s in range(6):
        A0, C0, r2 = o.identify_server(s)
        gs = o.gen_server(s)
        np.testing.assert_allclose(A0, gs["a_true"], rtol=1e-12)
        assert abs(C0 - gs["c_true"]) <= 1e-9 * abs(gs["c_true"])
        assert r2 == pytest.approx(1.0, abs=1e-12)


def test_set_point_inside_true_range(sweep):
    """P:230 feasibility: P_s = mid-range of the TRUE plant C + g a.f."""
    d, o, out = sweep
    fmin, fmax, _, _ = ST.knob_arrays(d)
    gains = ST.gains(d)
    ng = len(gains)
    for s in range(6):
        gs = o.gen_server(s)
        for c, g in enumerate(gains):
            lo = gs["c_true"] + g * (gs["a_true"] @ fmin)
            hi = gs["c_true"] + g * (gs["a_true"] @ fmax)
            assert out["cap"][0, s * ng + c] == pytest.approx(0.5 * (lo + hi), rel=1e-12)


def test_pole_analysis_stable_and_unstable(sweep):
    d, o, out = sweep
    gains = ST.gains(d)
    ng = len(gains)
    fmin, fmax, _, _ = ST.knob_arrays(d)
    n_stable = n_unstable = 0
    for s in range(6):
        gs = o.gen_server(s)
        a, C = gs["a_true"], gs["c_true"]
        for c, g in enumerate(gains):
            i = s * ng + c
            info = ST.analyse(d, a, C, out["cap"][-1, i], g)
            win = out["p"][-W:, i]
            dev = np.max(np.abs(win - info["p_star"]))
            if abs(info["rho"]) <= 0.9:
                assert info["interior"], (s, g)
                u0 = out["u"][-W:, i, 0, :]
                assert np.all(u0 > fmin) and np.all(u0 < fmax), (s, g)
                assert dev <= info["dev_bound"] + 1e-6, (s, g, dev, info["dev_bound"])
                mb = ST.mean_bound(info, g, W)
                assert abs(win.mean() - info["p_star"]) <= mb + 1e-6, (s, g, win.mean() - info["p_star"], mb)
                n_stable += 1
            elif abs(info["rho"]) >= 1.1:
                assert dev >= 0.25 * info["p_range"], (s, g, dev, info["p_range"])
                n_unstable += 1
    assert n_stable >= 40 and n_unstable >= 40


def test_one_step_pole(sweep):
    """Every period whose applied u(k) is strictly inside the box obeys the
    closed-loop recursion |(p(k+1) - p*) - rho (p(k) - p*)| <= g E (sign and
    size of the pole), stable and unstable gains alike."""
    d, o, out = sweep
    gains = ST.gains(d)
    ng = len(gains)
    fmin, fmax, _, _ = ST.knob_arrays(d)
    checked = 0
    for s in range(6):
        gs = o.gen_server(s)
        for c, g in enumerate(gains):
            i = s * ng + c
            info = ST.analyse(d, gs["a_true"], gs["c_true"], out["cap"][-1, i], g)
            dp = out["p"][:, i] - info["p_star"]
            u0 = out["u"][:-1, i, 0, :]
            inside = np.all((u0 > fmin) & (u0 < fmax), axis=1)
            r = np.abs(dp[1:] - info["rho"] * dp[:-1])[inside]
            assert np.all(r <= g * info["E"] * (1 + 1e-9) + 1e-7), (s, g, r.max(), g * info["E"])
            checked += int(np.count_nonzero(inside & (np.abs(dp[:-1]) > 10 * g * info["E"])))
    assert checked >= 100  # enough large-deviation steps that the sign of rho matters


def test_deadbeat_at_nominal_gain(oracle_mod):
    """g = 1: rho = 0, so after the first control period p(k) - p* is only the
    delta-sigma error of one period, |p - p*| <= E (the special case where the
    model is exact, P:221 step 1)."""
    d = configs.stability_sweep(n_servers=4, n_gains=2, g_lo=1.0, g_hi=2.0, periods=40)
    o = oracle_mod.Oracle(d)
    out = o.simulate(np.array([0, 2, 4, 6]), periods=40)
    for col, s in enumerate(range(4)):
        gs = o.gen_server(s)
        info = ST.analyse(d, gs["a_true"], gs["c_true"], out["cap"][-1, col], 1.0)
        assert info["rho"] == 0.0
        assert np.max(np.abs(out["p"][2:, col] - info["p_star"])) <= info["E"] + 1e-9
