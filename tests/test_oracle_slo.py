"""Pins of the oracle's SLO schedule (NEXT-1: §6.4, Eq. 10b-c P:205-208;
DESIGN.md Q29-Q31).  P:NNN = /root/reference/PAPER.md line.

What fixes the answer independently of the oracle's own formulas:
  * the latency model itself, evaluated FORWARD (e = e_min (f_max/f)^gamma,
    Eq. 10b, Q14) at the grid levels: the SLO level must be the lowest level
    whose latency meets the SLO (the oracle inverts the model instead);
  * P15: e(f_req) = SLO for the continuous bound;
  * schedule edges (step schedule, same convention as the cap schedule);
  * closed-loop invariants: u_t >= l(k) every period and block, and a loose SLO
    (level 0) reproduces the SLO-free run bit for bit;
  * the miss count against a recount of the level trace, and non-zero misses
    for the SLO-blind controller on the same plant (the metric is not vacuous).
"""
import numpy as np
import pytest

from gen import configs


def _o(oracle_mod, **kw):
    return oracle_mod.Oracle(configs.slo_schedule(**kw))


@pytest.mark.parametrize("gamma", [0.91, 0.5, 1.7])
def test_slo_level_is_lowest_level_meeting_the_latency(oracle_mod, gamma):
    d = configs.slo_schedule(n_servers=1)
    d["controller"]["gamma"] = gamma
    o = oracle_mod.Oracle(d)
    rng = np.random.default_rng(7)
    for j in (0, 1):
        lv, _, _ = o.levels(j)
        fmax = d["knobs"][j]["f_max"]
        lat = (fmax / lv) ** gamma  # e / e_min at every level (Eq. 10b, forward)
        for ratio in list(rng.uniform(0.8, 4.0, 200)) + [1.0, 1.15, 1.35, 1.6]:
            q, f_req = o.slo_level(j, ratio)
            # P15: the continuous bound has latency exactly SLO
            assert abs((fmax / f_req) ** gamma - ratio) <= 1e-12 * ratio
            if q < len(lv):
                assert lat[q] <= ratio * (1 + 1e-12)
            else:
                assert ratio < 1.0  # even f_max misses
            if q > 0:
                assert lat[q - 1] > ratio * (1 - 1e-12)


def test_slo_bounds_follow_the_schedule(oracle_mod):
    o = _o(oracle_mod, n_servers=1, periods=400)
    lv_gpu, _, _ = o.levels(1)
    qa = o.slo_level(1, configs.SLO_TAIL[50])[0]
    q30 = o.slo_level(1, configs.SLO_TAIL[30])[0]
    q80 = o.slo_level(1, configs.SLO_TAIL[80])[0]
    assert q30 > qa > q80  # tighter SLO -> higher level
    for k in range(400):
        lo, q, st = o.slo_bounds(k)
        b = 14 <= k % 200 < 114
        exp_q = [0, q30, q80, q80] if b else [0, qa, qa, qa]
        assert list(q) == exp_q, k
        assert lo[0] == 1100.0  # the CPU task has no SLO
        assert np.array_equal(lo[1:], lv_gpu[exp_q[1:]])
        assert st == 0


def test_slo_infeasible_sets_status_and_pins_fmax(oracle_mod):
    d = configs.slo_schedule(n_servers=1, periods=30)
    d["workload"]["slo_a"] = [0.0, 0.9, 1.35, 1.35]  # 0.9 < 1: faster than f_max allows
    o = oracle_mod.Oracle(d)
    lo, q, st = o.slo_bounds(0)
    assert st == oracle_mod.ST_SLO_INFEASIBLE and q[1] == 11 and lo[1] == 1350.0
    out = o.simulate([0])
    assert np.all(out["status"][:14] & oracle_mod.ST_SLO_INFEASIBLE)
    assert not np.any(out["status"][14:] & oracle_mod.ST_SLO_INFEASIBLE)  # phase B is feasible
    # every sub-step of the infeasible knob misses while phase A is in force
    assert np.all(out["levels"][:14, 0, :, 1] < 11)


def test_slo_closed_loop_bounds_and_misses(oracle_mod):
    K = 300
    o = _o(oracle_mod, n_servers=12, periods=K)
    out = o.simulate(list(range(12)))
    lo_k = np.array([o.slo_bounds(k)[0] for k in range(K)])
    q_k = np.array([o.slo_bounds(k)[1] for k in range(K)])
    u = out["u"]  # [K][inst][M][N]
    assert np.all(u >= lo_k[:, None, None, :])  # Eq. 10a + 10c at every block, every period
    assert np.all(u <= np.array([k["f_max"] for k in o.desc["knobs"]]))
    miss = (out["levels"] < q_k[:, None, None, :])  # [K][inst][S][N]
    kw = K - (4 * K) // 5
    assert np.array_equal(out["summary"]["n_miss"], miss[kw:].sum(axis=(0, 2, 3)))
    # with the SLO bound in the MPC, the delta-sigma levels never fall below it
    assert miss.sum() == 0
    # the phase switch acts at the switch instant itself (Q17-style indexing)
    assert np.all(u[14, :, 0, 1] >= o.slo_bounds(14)[0][1])


def test_slo_blind_controller_misses(oracle_mod):
    """Same plant, SLO-free MPC: the sub-step levels fall below the SLO levels
    (so the miss metric measures something the SLO constraint fixes)."""
    K = 200
    o_slo = _o(oracle_mod, n_servers=12, periods=K)
    d = configs.slo_schedule(n_servers=12, periods=K)
    d["workload"].update(slo_period=0, slo_a=None, slo_b=None)
    blind = oracle_mod.Oracle(d).simulate(list(range(12)))
    q_k = np.array([o_slo.slo_bounds(k)[1] for k in range(K)])
    assert (blind["levels"] < q_k[:, None, None, :]).sum() > 100


def test_loose_slo_reproduces_slo_free_run(oracle_mod):
    """An SLO every level meets (q = 0, l = f_min) changes nothing: bitwise."""
    K = 150
    d1 = configs.slo_schedule(n_servers=4, periods=K)
    d1["workload"].update(slo_a=[0.0, 50.0, 50.0, 50.0], slo_b=[50.0, 0.0, 50.0, 0.0])
    d0 = configs.slo_schedule(n_servers=4, periods=K)
    d0["workload"].update(slo_period=0, slo_a=None, slo_b=None)
    a = oracle_mod.Oracle(d1).simulate(list(range(4)))
    b = oracle_mod.Oracle(d0).simulate(list(range(4)))
    for key in ("p", "u", "levels", "active", "status"):
        assert np.array_equal(a[key], b[key]), key
    assert a["summary"]["n_miss"].sum() == 0
