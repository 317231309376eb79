"""Pins of the oracle's S2 weights, S4 plant (delta-sigma), the closed loop and
the S5 budget (DESIGN.md §4 P5-P8, P11, P12).  P:NNN = /root/reference/PAPER.md line."""
import json
import os

import numpy as np
import pytest

from tests.inputs import desc_for

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


# ---------------------------------------------------------------- S2 (P11)

def test_p11_weights_and_stable_ranks(oracle_mod):
    """theta = clamp(thr/thr_max, theta_min, 1), R = r0/theta,
    rank = stable descending sort (ties -> lower knob index); numpy's stable
    argsort is the independent reference."""
    d = desc_for(8)
    o = oracle_mod.Oracle(d)
    rng = np.random.default_rng(31)
    n = o.n
    for it in range(500):
        thr_max = 40 + 160 * rng.random(n)
        frac = rng.random(n) * 1.2
        if it % 3 == 0:  # force ties at the clamps and exact duplicates
            frac[rng.integers(0, n, 3)] = 1.3
            frac[rng.integers(0, n, 2)] = 0.0
        thr = thr_max * frac
        th, R, rk = o.weights(thr, thr_max)
        th_ref = np.clip(thr / thr_max, 0.05, 1.0)
        assert np.array_equal(th, th_ref)
        assert np.array_equal(R, 1e-4 / th_ref)
        order = np.argsort(-th_ref, kind="stable")
        rk_ref = np.empty(n, dtype=np.int8); rk_ref[order] = np.arange(n)
        assert np.array_equal(rk, rk_ref)


# ---------------------------------------------------------------- S4 (P7, P8)

def test_p8_golden_delta_sigma_example(oracle_mod):
    """target 2.4 between the two nearest levels {2, 3} (units GHz).  The
    paper's listed pattern 2,2,2,3 averages 2.25 (inconsistent); the first-order
    modulator gives 2,3,2,3,2, whose mean is exactly 2.4 (golden fixture)."""
    with open(os.path.join(GOLDEN, "delta_sigma_p242.json")) as fh:
        gold = json.load(fh)
    d = desc_for(0, noise_std=0.0)
    d["knobs"] = [dict(f_min=gold["levels"][0], f_max=gold["levels"][1], n_levels=2, sweep_base=0)]
    d["controller"]["substeps"] = 1
    o = oracle_mod.Oracle(d)
    acc = np.zeros(1)
    seen = []
    for _ in range(len(gold["pattern"])):
        fbar, p, thr, acc, lv = o.plant_step([0.0], 0.0, [1.0], [1.0], 0.0, [gold["target"]], acc)
        seen.append(float(fbar[0]))
    assert seen == gold["pattern"]
    assert abs(np.mean(seen) - gold["target"]) < 1e-12


@pytest.mark.parametrize("knob", [0, 1])
def test_p7_p8_delta_sigma_bounds(oracle_mod, knob):
    """|sum_{s<n} (level_s - u)| <= step/2 for a constant command, level index in
    [0, L-1], |acc| <= step/2 (first-order error feedback)."""
    d = desc_for(1)
    o = oracle_mod.Oracle(d)
    lv, mid, g = o.levels(knob)
    step = lv[1] - lv[0]
    rng = np.random.default_rng(32 + knob)
    for _ in range(50):
        u = lv[0] + (lv[-1] - lv[0]) * rng.random()
        uvec = np.array([u, u]) if knob == 0 else np.array([1100.0, u])
        acc = np.zeros(2)
        err = 0.0
        for k in range(200):
            fbar, p, thr, acc, levels = o.plant_step([0.0, 0.0], 0.0, [1.0, 1.0], [1.0, 1.0], 0.0, uvec, acc)
            assert np.all(levels[:, knob] <= len(lv) - 1)
            assert abs(acc[knob]) <= step / 2 + 1e-9
            err += (fbar[knob] - u) * o.S
            assert abs(err) <= step / 2 + 1e-7


def test_plant_levels_are_nearest_with_feedback(oracle_mod):
    """Level index = #midpoints strictly below v (ties -> lower), Q15."""
    d = desc_for(1)
    o = oracle_mod.Oracle(d)
    lv, mid, g = o.levels(1)
    for tgt, expect in [(mid[3], 3), (np.nextafter(mid[3], np.inf), 4), (lv[0], 0), (lv[-1], len(lv) - 1)]:
        acc = np.zeros(2)
        fbar, p, thr, acc, levels = o.plant_step([0, 0], 0.0, [1, 1], [1, 1], 0.0, [1100.0, tgt], acc)
        assert levels[0, 1] == expect


# ---------------------------------------------------------------- closed loop

def test_p5_deadbeat_steady_state_continuous(oracle_mod):
    """P5: exact plant = model, no noise, frozen model, continuous actuator,
    M >= 2, interior: deadbeat and p_inf = P_s + (P_min - P_s)/(1 + Q sum a^2/R)."""
    d = desc_for(2, P=8, M=2)
    o = oracle_mod.Oracle(d)
    n = o.n
    a = np.array([0.05, 0.21, 0.18]); c0 = 300.0
    lo, hi, m = np.array([1100.0, 435, 435]), np.array([2400.0, 1350, 1350]), np.array([1100.0, 435, 435])
    R = np.full(n, 1e-4)
    pmin, pmax = c0 + a @ lo, c0 + a @ hi
    Ps = pmin + 0.6 * (pmax - pmin)
    f = lo.copy(); p = c0 + a @ f
    ps = []
    for k in range(20):
        beta = p - a @ f - Ps
        u, act, *_ = o.mpc(a, R, beta, lo, hi, m)
        assert np.all(act == 0)
        f = u[0]; p = c0 + a @ f
        ps.append(p)
    expect = Ps + (pmin - Ps) / (1 + np.sum(a * a / R))
    assert abs(ps[0] - expect) <= 1e-9 and abs(ps[-1] - expect) <= 1e-9


def test_p5_steady_state_with_delta_sigma(oracle_mod):
    """P5 through the full oracle loop (identify -> S1..S4) with the quantising
    actuator: theta_min = 1 (all weights 1), no noise, frozen model (huge rho).
    The window mean of p is within the delta-sigma averaging bound
    sum_j a_j step_j / (2 * substeps_in_window) of the closed form."""
    d = desc_for(2, P=8, M=2, noise_std=0.0, rho=1e20, theta_min=1.0, periods=400)
    d["workload"]["demand_kind"] = 0
    o = oracle_mod.Oracle(d)
    out = o.simulate([0])
    g = o.gen_server(0)
    a, c0 = g["a_true"], g["c_true"]
    lo = np.array([k["f_min"] for k in d["knobs"]]); hi = np.array([k["f_max"] for k in d["knobs"]])
    pmin, pmax = c0 + a @ lo, c0 + a @ hi
    Ps = pmin + 0.6 * (pmax - pmin)
    expect = Ps + (pmin - Ps) / (1 + np.sum(a * a / 1e-4))
    s = out["summary"]
    mean = s["sum_p"][0] / s["n_window"][0]
    steps = np.array([(k["f_max"] - k["f_min"]) / (k["n_levels"] - 1) for k in d["knobs"]])
    bound = np.sum(a * steps) / (2 * s["n_window"][0] * 4) * 2 + 1e-9
    assert abs(mean - expect) <= bound, (mean, expect, bound)


@pytest.mark.parametrize("g", [0.5, 1.5, 1.9])
def test_p6_pole_under_gain_mismatch(oracle_mod, g):
    """P6 / §4.4: frozen Ahat = A0, true gains g*A0: the single
    closed-loop pole is -(g - 1) Q kappa / (1 + Q kappa), kappa = sum A0^2/R."""
    d = desc_for(2, P=8, M=2)
    o = oracle_mod.Oracle(d)
    n = o.n
    A0 = np.array([0.05, 0.2, 0.17]); R = np.full(n, 1e-3); c0 = 300.0
    big = 1e7
    lo, hi, m = np.full(n, -big), np.full(n, big), np.array([1100.0, 435, 435])
    Ps = 900.0
    kappa = np.sum(A0 * A0 / R)
    pole = -(g - 1) * kappa / (1 + kappa)
    f = m.copy(); p = c0 + g * A0 @ f
    ss = []
    for k in range(12):
        beta = p - A0 @ f - Ps
        u, *_ = o.mpc(A0, R, beta, lo, hi, m)
        ss.append(beta + A0 @ u[0])  # s(k)
        f = u[0]; p = c0 + g * A0 @ f
    ss = np.array(ss)
    # s(k) - s* decays geometrically with ratio = pole
    dif = np.diff(ss)
    ratios = dif[1:] / dif[:-1]
    np.testing.assert_allclose(ratios[:6], pole, rtol=1e-6)


def test_p6_stability_bound(oracle_mod):
    """P6: converges iff 0 < g < 2 + 1/(Q kappa)."""
    d = desc_for(2, P=8, M=2)
    o = oracle_mod.Oracle(d)
    n = o.n
    A0 = np.array([0.05, 0.2, 0.17]); R = np.full(n, 5e-2); c0 = 300.0
    kappa = np.sum(A0 * A0 / R)
    gcrit = 2 + 1 / kappa
    big = 1e9
    lo, hi, m = np.full(n, -big), np.full(n, big), np.array([1100.0, 435, 435])
    for g, conv in [(gcrit * 0.995, True), (gcrit * 1.005, False)]:
        f = m.copy(); p = c0 + g * A0 @ f
        errs = []
        for k in range(3000):
            beta = p - A0 @ f - 900.0
            u, *_ = o.mpc(A0, R, beta, lo, hi, m)
            f = u[0]; pn = c0 + g * A0 @ f
            errs.append(abs(pn - p)); p = pn
        assert (errs[-1] < errs[10]) == conv


def test_p7_bounds_every_period(oracle_mod):
    """P7: l <= u_t <= h and 0 <= level <= L-1 every period of a noisy bursty run."""
    d = desc_for(4, P=8, M=2, periods=300)
    o = oracle_mod.Oracle(d)
    out = o.simulate(np.arange(6))
    lo = np.array([k["f_min"] for k in d["knobs"]]); hi = np.array([k["f_max"] for k in d["knobs"]])
    L = np.array([k["n_levels"] for k in d["knobs"]])
    assert np.all(out["u"] >= lo) and np.all(out["u"] <= hi)
    assert np.all(out["levels"] <= L - 1)
    assert np.all(out["status"] & oracle_mod.ST_SOLVER_CAP == 0)


def test_p9_closed_loop_modes_agree(oracle_mod):
    """P9 in closed loop: recursive (Welford) and definition (two-pass history)
    model updates give the same traces (cfg 1, 200 periods)."""
    o = oracle_mod.oracle_for(1)
    a = o.simulate([0], definition_mode=False)
    b = o.simulate([0], definition_mode=True)
    np.testing.assert_allclose(a["ahat"], b["ahat"], rtol=1e-10)
    np.testing.assert_allclose(a["p"], b["p"], rtol=0, atol=1e-8)
    assert np.array_equal(a["levels"], b["levels"])


# ---------------------------------------------------------------- S5 (P12)

def test_p12_budget_conservation(oracle_mod):
    """P12: sum_i cap_i = B_c when no rack limit binds; a binding rack gets exactly
    its limit; caps are >= P_min and proportional to w inside a rack."""
    o = oracle_mod.oracle_for(4)
    rng = np.random.default_rng(33)
    n, rack = 256, 16
    pmin = 900 + 200 * rng.random(n)
    pmax = pmin + 1000 + 500 * rng.random(n)
    w = 0.05 + 0.95 * rng.random(n)
    W = w.sum()
    Bc = pmin.sum() + 0.55 * (pmax.sum() - pmin.sum())
    Brack = 0.9 * pmax.reshape(-1, rack).sum(axis=1)
    cap = o.budget_caps(pmin, w, W, Bc, pmin.sum(), np.full(n // rack, 1e12), rack)
    assert abs(cap.sum() - Bc) <= 1e-9 * Bc
    assert np.all(cap >= pmin)
    r0 = (cap[:rack] - pmin[:rack]) / w[:rack]
    np.testing.assert_allclose(r0, r0[0], rtol=1e-12)
    Brack[3] = pmin[48:64].sum() + 1.0  # force rack 3 to bind
    cap = o.budget_caps(pmin, w, W, Bc, pmin.sum(), Brack, rack)
    assert abs(cap[48:64].sum() - Brack[3]) <= 1e-9 * Brack[3]
