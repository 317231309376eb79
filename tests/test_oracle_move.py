"""Pins of the oracle's NEXT-3 horizon-active MPC: Eq. 9 plus a
move-suppression term sum_{t<M} W |d(k+t|k)|^2 (Q36), which couples
the control-horizon blocks so that P and M change the applied u_0.

Independent of the oracle's dense H, g:
  * the cost is typed here from the definition in the increments d
    (p(k+i|k) = p(k) + A sum_{tau<min(i,M)} d_tau, d_t = u_t - u_{t-1}, u_{-1} = f(k));
  * P2-style KKT with that cost's central finite-difference gradient;
  * P3-style brute force over all 3^(MN) active sets (MN <= 8);
  * the unconstrained minimiser from a finite-difference Hessian of the typed
    cost (numpy solve), for a problem with no bound active;
  * W = 0 reproduces the literal (decoupled) Eq. 9 solve, W -> inf freezes
    the frequencies at f(k) (clamped to the box);
  * W > 0 makes u_0 depend on the prediction horizon P, W = 0 does not (Q11).
"""
import numpy as np
import pytest

from tests.inputs import desc_for, mpc_problem


def _V(u, ahat, R, beta, m, P, M, W, f, q=1.0):
    V = 0.0
    for i in range(1, P + 1):
        t = min(i, M) - 1
        V += q * (beta + ahat @ u[t]) ** 2
    for t in range(M):
        V += np.sum(R * (u[t] - m) ** 2)
        d = u[t] - (f if t == 0 else u[t - 1])
        V += W * np.sum(d * d)
    return V


def _o(oracle_mod, n_gpus, P, M, W):
    d = desc_for(n_gpus, P=P, M=M)
    d["controller"]["wmove"] = W
    return oracle_mod.Oracle(d), d


@pytest.mark.parametrize("n_gpus,P,M,W", [(1, 8, 2, 1e-4), (3, 8, 2, 3e-4), (2, 8, 3, 1e-3), (8, 8, 3, 2e-4),
                                          (3, 6, 4, 5e-5)])
def test_move_kkt(oracle_mod, n_gpus, P, M, W):
    o, d = _o(oracle_mod, n_gpus, P, M, W)
    rng = np.random.default_rng(100 + n_gpus + M)
    n_act = 0
    for _ in range(80):
        pr = mpc_problem(rng, d)
        u, act, tie, st, _ = o.mpc_move(pr["ahat"], pr["R"], pr["beta"], pr["f"], pr["lo"], pr["hi"], pr["m"])
        assert st == 0
        assert np.all(u >= pr["lo"]) and np.all(u <= pr["hi"])
        assert abs(o.mpc_move_cost(pr["ahat"], pr["R"], pr["beta"], pr["f"], pr["m"], u)
                   - _V(u, pr["ahat"], pr["R"], pr["beta"], pr["m"], P, M, W, pr["f"])) <= 1e-9 * max(1.0, abs(
                       _V(u, pr["ahat"], pr["R"], pr["beta"], pr["m"], P, M, W, pr["f"])))
        h = 1e-3
        g = np.zeros_like(u)
        for t in range(M):
            for j in range(o.n):
                up = u.copy(); up[t, j] += h
                um = u.copy(); um[t, j] -= h
                g[t, j] = (_V(up, pr["ahat"], pr["R"], pr["beta"], pr["m"], P, M, W, pr["f"])
                           - _V(um, pr["ahat"], pr["R"], pr["beta"], pr["m"], P, M, W, pr["f"])) / (2 * h)
        scale = 1e-6 * max(1.0, np.max(np.abs(g)))
        for t in range(M):
            code = (act[t] >> (2 * np.arange(o.n))) & 3
            for j in range(o.n):
                if u[t, j] == pr["lo"][j]:
                    assert g[t, j] >= -scale and code[j] == 1
                    n_act += 1
                elif u[t, j] == pr["hi"][j]:
                    assert g[t, j] <= scale and code[j] == 2
                    n_act += 1
                else:
                    assert abs(g[t, j]) <= scale and code[j] == 0
    assert n_act > 20


@pytest.mark.parametrize("n_gpus,M", [(1, 2), (2, 2), (3, 2), (1, 3), (1, 4)])
def test_move_bruteforce(oracle_mod, n_gpus, M):
    o, d = _o(oracle_mod, n_gpus, 8, M, 2e-4)
    rng = np.random.default_rng(7 + 10 * n_gpus + M)
    for _ in range(60):
        pr = mpc_problem(rng, d)
        u, *_ = o.mpc_move(pr["ahat"], pr["R"], pr["beta"], pr["f"], pr["lo"], pr["hi"], pr["m"])
        ub = o.mpc_move_bruteforce(pr["ahat"], pr["R"], pr["beta"], pr["f"], pr["lo"], pr["hi"], pr["m"])
        np.testing.assert_allclose(u, ub, rtol=1e-11, atol=1e-9)


def test_move_unconstrained_closed_form(oracle_mod):
    """No bound active: u = -H^-1 g with H, g from finite differences of the
    typed cost (exact for a quadratic up to rounding)."""
    o, d = _o(oracle_mod, 2, 8, 3, 4e-4)
    rng = np.random.default_rng(5)
    done = 0
    for _ in range(200):
        pr = mpc_problem(rng, d, active_mix=False)
        u, act, *_ = o.mpc_move(pr["ahat"], pr["R"], pr["beta"], pr["f"], pr["lo"], pr["hi"], pr["m"])
        if np.any(act):
            continue
        n, M = o.n, o.M
        V = lambda x: _V(x.reshape(M, n), pr["ahat"], pr["R"], pr["beta"], pr["m"], 8, M, 4e-4, pr["f"])  # noqa
        x0 = u.reshape(-1)
        h = 1.0
        nv = n * M
        Hm = np.zeros((nv, nv)); gv = np.zeros(nv)
        for a in range(nv):
            ea = np.zeros(nv); ea[a] = h
            gv[a] = (V(x0 + ea) - V(x0 - ea)) / (2 * h)
            for b in range(nv):
                eb = np.zeros(nv); eb[b] = h
                Hm[a, b] = (V(x0 + ea + eb) - V(x0 + ea - eb) - V(x0 - ea + eb) + V(x0 - ea - eb)) / (4 * h * h)
        xs = x0 - np.linalg.solve(Hm, gv)  # one Newton step from u lands on the minimiser
        np.testing.assert_allclose(u.reshape(-1), xs, rtol=1e-9, atol=1e-6)
        done += 1
        if done >= 10:
            break
    assert done >= 10


def test_move_limits(oracle_mod):
    rng = np.random.default_rng(9)
    o0, d = _o(oracle_mod, 3, 8, 3, 0.0)
    ow, _ = _o(oracle_mod, 3, 8, 3, 1e9)
    for _ in range(40):
        pr = mpc_problem(rng, d)
        a = (pr["ahat"], pr["R"], pr["beta"])
        u0, *_ = o0.mpc(*a, pr["lo"], pr["hi"], pr["m"])
        um, *_ = o0.mpc_move(*a, pr["f"], pr["lo"], pr["hi"], pr["m"])
        np.testing.assert_allclose(um, u0, rtol=1e-12, atol=1e-9)  # W = 0: the literal Eq. 9
        uw, *_ = ow.mpc_move(*a, pr["f"], pr["lo"], pr["hi"], pr["m"])
        np.testing.assert_allclose(uw, np.tile(np.clip(pr["f"], pr["lo"], pr["hi"]), (3, 1)), rtol=0, atol=1e-3)


def test_move_makes_the_horizon_matter(oracle_mod):
    rng = np.random.default_rng(11)
    diff_w, diff_0 = 0.0, 0.0
    for _ in range(30):
        o8, d = _o(oracle_mod, 2, 8, 2, 3e-3)
        o4, _ = _o(oracle_mod, 2, 4, 2, 3e-3)
        p8, _ = _o(oracle_mod, 2, 8, 2, 0.0)
        p4, _ = _o(oracle_mod, 2, 4, 2, 0.0)
        pr = mpc_problem(rng, d, active_mix=False)
        a = (pr["ahat"], pr["R"], pr["beta"], pr["f"], pr["lo"], pr["hi"], pr["m"])
        diff_w = max(diff_w, np.max(np.abs(o8.mpc_move(*a)[0][0] - o4.mpc_move(*a)[0][0])))
        diff_0 = max(diff_0, np.max(np.abs(p8.mpc_move(*a)[0][0] - p4.mpc_move(*a)[0][0])))
    assert diff_0 == 0.0  # Q11: u_0 of the literal Eq. 9 does not see P
    assert diff_w > 1e-3  # MHz: with the move term it does (exactly 0 without)
