"""Pins of the oracle's NEXT-3 reference trajectory (the controller
"comprises a least squares solver, a cost function, a reference trajectory,
and a system model"; Q37).  Prediction step i tracks

    r(k+i|k) = P_s - alpha^i (P_s - p(k)),   alpha = exp(-T / T_ref) in [0, 1),

instead of P_s, so Eq. 9's tracking term becomes
sum_i Q (p(k+i|k) - r(k+i|k))^2 with p(k+i|k) = p(k) + A.(u_{min(i,M)-1} - f(k)).

Independent of the oracle's dense H, g:
  * the cost is typed here from that definition;
  * P2-style KKT with the typed cost's central finite-difference gradient
    (literal Eq. 9 blocks and the move-suppressed coupled QP);
  * P3-style brute force over all 3^(MN) active sets;
  * P1-style closed form of the first block when no bound is active
    (Sherman-Morrison with the row-1 target);
  * alpha = 0 reproduces the literal Eq. 9 bitwise;
  * Q11 still holds: u_0 sees only row 1 (alpha), not P;
  * closed loop on an exact continuous plant: the error decays geometrically
    with ratio gamma * alpha, gamma = Q kappa / (1 + Q kappa), around the fixed
    point p_inf = (P_min - gamma (P_min - P_s) - gamma alpha P_s) / (1 - gamma alpha).
"""
import numpy as np
import pytest

from tests.inputs import desc_for, mpc_problem


def _V(u, pr, P, M, alpha, W=0.0, q=1.0):
    """Eq. 9 with the reference trajectory, typed from the definition."""
    p, f, cap, a = pr["p"], pr["f"], pr["cap"], pr["ahat"]
    V = 0.0
    for i in range(1, P + 1):
        t = min(i, M) - 1
        pred = p + a @ (u[t] - f)
        r = cap - alpha ** i * (cap - p)
        V += q * (pred - r) ** 2
    for t in range(M):
        V += np.sum(pr["R"] * (u[t] - pr["m"]) ** 2)
        if W > 0:
            d = u[t] - (f if t == 0 else u[t - 1])
            V += W * np.sum(d * d)
    return V


def _o(oracle_mod, n_gpus, P, M, alpha, W=0.0):
    d = desc_for(n_gpus, P=P, M=M)
    d["controller"]["ref_alpha"] = alpha
    d["controller"]["wmove"] = W
    return oracle_mod.Oracle(d), d


def _solve(o, pr, W):
    dref = pr["cap"] - pr["p"]
    if W > 0:
        return o.mpc_move(pr["ahat"], pr["R"], pr["beta"], pr["f"], pr["lo"], pr["hi"], pr["m"], dref=dref)
    return o.mpc(pr["ahat"], pr["R"], pr["beta"], pr["lo"], pr["hi"], pr["m"], dref=dref)


@pytest.mark.parametrize("n_gpus,P,M,alpha,W", [(1, 8, 2, 0.6, 0.0), (3, 8, 2, 0.3, 0.0), (2, 8, 3, 0.85, 0.0),
                                                (8, 8, 3, 0.5, 0.0), (3, 6, 4, 0.7, 0.0), (1, 8, 1, 0.5, 0.0),
                                                (3, 8, 2, 0.6, 3e-4), (2, 8, 3, 0.4, 1e-3)])
def test_ref_kkt_and_cost(oracle_mod, n_gpus, P, M, alpha, W):
    o, d = _o(oracle_mod, n_gpus, P, M, alpha, W)
    rng = np.random.default_rng(300 + 7 * n_gpus + M)
    n_act = 0
    for _ in range(60):
        pr = mpc_problem(rng, d)
        u, act, tie, st, _ = _solve(o, pr, W)
        assert st == 0
        assert np.all(u >= pr["lo"]) and np.all(u <= pr["hi"])
        if W == 0:
            Vo = o.mpc_cost(pr["ahat"], pr["R"], pr["beta"], pr["m"], u, dref=pr["cap"] - pr["p"])
            Vt = _V(u, pr, P, M, alpha)
            assert abs(Vo - Vt) <= 1e-9 * max(1.0, abs(Vt))
        h = 1e-3
        g = np.zeros_like(u)
        for t in range(M):
            for j in range(o.n):
                up = u.copy(); up[t, j] += h
                um = u.copy(); um[t, j] -= h
                g[t, j] = (_V(up, pr, P, M, alpha, W) - _V(um, pr, P, M, alpha, W)) / (2 * h)
        scale = 1e-6 * max(1.0, np.max(np.abs(g)))
        for t in range(M):
            for j in range(o.n):
                if u[t, j] == pr["lo"][j]:
                    assert g[t, j] >= -scale
                    n_act += 1
                elif u[t, j] == pr["hi"][j]:
                    assert g[t, j] <= scale
                    n_act += 1
                else:
                    assert abs(g[t, j]) <= scale
    assert n_act > 10


@pytest.mark.parametrize("n_gpus,M,W", [(1, 2, 0.0), (2, 2, 0.0), (1, 3, 0.0), (3, 2, 0.0), (2, 2, 2e-4),
                                        (1, 4, 5e-4)])
def test_ref_bruteforce(oracle_mod, n_gpus, M, W):
    o, d = _o(oracle_mod, n_gpus, 8, M, 0.55, W)
    rng = np.random.default_rng(41 + 10 * n_gpus + M)
    for _ in range(50):
        pr = mpc_problem(rng, d)
        u, *_ = _solve(o, pr, W)
        ub = o.mpc_bruteforce(pr["ahat"], pr["R"], pr["beta"], pr["lo"], pr["hi"], pr["m"],
                              dref=pr["cap"] - pr["p"], fbar=pr["f"] if W > 0 else None)
        np.testing.assert_allclose(u, ub, rtol=1e-11, atol=1e-9)


def test_ref_first_block_closed_form(oracle_mod):
    """No bound active: block 0 minimises Q (beta_0 + A.u)^2 + sum R (u - m)^2
    with beta_0 = beta + alpha dref (row 1 only), so
    u = m - Q s R^-1 A,  s = (beta_0 + A.m) / (1 + Q sum A^2/R)."""
    alpha = 0.7
    o, d = _o(oracle_mod, 3, 8, 2, alpha)
    rng = np.random.default_rng(17)
    done = 0
    for _ in range(300):
        pr = mpc_problem(rng, d, active_mix=False)
        u, act, *_ = _solve(o, pr, 0.0)
        if act[0] != 0:
            continue
        a, R, m = pr["ahat"], pr["R"], pr["m"]
        b0 = pr["beta"] + alpha * (pr["cap"] - pr["p"])
        s = (b0 + a @ m) / (1 + np.sum(a * a / R))
        np.testing.assert_allclose(u[0], m - s * a / R, rtol=1e-12)
        done += 1
        if done >= 20:
            break
    assert done >= 20


def test_ref_alpha_zero_is_literal(oracle_mod):
    o0, d = _o(oracle_mod, 3, 8, 3, 0.0)
    rng = np.random.default_rng(23)
    for _ in range(40):
        pr = mpc_problem(rng, d)
        ul, al, *_ = o0.mpc(pr["ahat"], pr["R"], pr["beta"], pr["lo"], pr["hi"], pr["m"])
        ur, ar, *_ = o0.mpc(pr["ahat"], pr["R"], pr["beta"], pr["lo"], pr["hi"], pr["m"], dref=pr["cap"] - pr["p"])
        assert np.array_equal(ul, ur) and np.array_equal(al, ar)


def test_ref_u0_sees_alpha_not_P(oracle_mod):
    """Q11 with the reference trajectory: block 0 holds only prediction row 1,
    so u_0 depends on alpha but not on P; the last block sees P."""
    rng = np.random.default_rng(29)
    dP = dA = dlast = 0.0
    for _ in range(30):
        o8, d = _o(oracle_mod, 2, 8, 2, 0.6)
        o12, _ = _o(oracle_mod, 2, 12, 2, 0.6)
        o8b, _ = _o(oracle_mod, 2, 8, 2, 0.3)
        pr = mpc_problem(rng, d, active_mix=False)
        u8, u12, u8b = _solve(o8, pr, 0)[0], _solve(o12, pr, 0)[0], _solve(o8b, pr, 0)[0]
        dP = max(dP, np.max(np.abs(u8[0] - u12[0])))
        dlast = max(dlast, np.max(np.abs(u8[1] - u12[1])))
        dA = max(dA, np.max(np.abs(u8[0] - u8b[0])))
    assert dP <= 1e-9 and dlast > 1e-3 and dA > 1e-3


@pytest.mark.parametrize("alpha", [0.0, 0.4, 0.8])
def test_ref_closed_loop_pole(oracle_mod, alpha):
    """Exact continuous plant p = C + a.f, frozen exact model, interior: the
    error to p_inf shrinks by gamma * alpha per period (deadbeat at alpha = 0)."""
    o, d = _o(oracle_mod, 2, 8, 2, alpha)
    a = np.array([0.05, 0.21, 0.18]); c0 = 300.0
    lo, hi, m = np.array([1100.0, 435, 435]), np.array([2400.0, 1350, 1350]), np.array([1100.0, 435, 435])
    R = np.full(o.n, 1e-4)
    pmin, pmax = c0 + a @ lo, c0 + a @ hi
    Ps = pmin + 0.6 * (pmax - pmin)
    gam = np.sum(a * a / R) / (1 + np.sum(a * a / R))
    p_inf = (pmin - gam * (pmin - Ps) - gam * alpha * Ps) / (1 - gam * alpha)
    f = lo.copy(); p = c0 + a @ f
    errs = [p - p_inf]
    for k in range(12):
        beta = p - a @ f - Ps
        u, act, *_ = o.mpc(a, R, beta, lo, hi, m, dref=Ps - p)
        assert np.all(act == 0)
        f = u[0]; p = c0 + a @ f
        errs.append(p - p_inf)
    errs = np.array(errs)
    if alpha == 0.0:
        assert np.all(np.abs(errs[1:]) <= 1e-9)
    else:
        np.testing.assert_allclose(errs[1:6] / errs[0:5], gam * alpha, rtol=1e-7)


def test_ref_simulate_bounds_and_slower_approach(oracle_mod):
    """Full oracle loop (S1-S4) with the reference trajectory: bounds every
    period (P7), and a step change in the cap is approached more slowly than
    with the literal Eq. 9 (the first-period move is scaled by 1 - alpha)."""
    from gen import configs
    d0 = configs.get(2, n_servers=8, periods=120)
    d1 = configs.get(2, n_servers=8, periods=120)
    d1["controller"]["ref_alpha"] = 0.8
    r0 = oracle_mod.Oracle(d0).simulate([0, 3], periods=120)
    r1 = oracle_mod.Oracle(d1).simulate([0, 3], periods=120)
    lo = np.array([k.get("f_lo", k["f_min"]) for k in d1["knobs"]])
    hi = np.array([k["f_max"] for k in d1["knobs"]])
    u = r1["u"]  # [periods][inst][M][N]
    assert np.all(u >= lo - 1e-9) and np.all(u <= hi + 1e-9)
    # applied-frequency moves are smaller with the reference trajectory
    mv0 = np.abs(np.diff(r0["u"][:, :, 0], axis=0)).sum()
    mv1 = np.abs(np.diff(r1["u"][:, :, 0], axis=0)).sum()
    assert mv1 < mv0
