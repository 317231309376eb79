"""Pins of the oracle's S3 MPC solve (Eq. 9-10a) against things other
than itself: closed forms, KKT conditions, brute force, a grid search, an
independent library least-squares solver (scipy bvls) and the paper's own
solver family (SLSQP on Eq. 9 written in the increments d).  DESIGN.md §4 P1-P4, P13.
"""
import numpy as np
import pytest
from scipy.optimize import lsq_linear, minimize

from tests.inputs import desc_for, mpc_problem


def _c_blocks(P, M, q=1.0):
    # weight of block t = Q * #{i in 1..P : min(i, M) - 1 == t}   (Eq. 9 + Eq. 7)
    c = np.zeros(M)
    for i in range(1, P + 1):
        c[min(i, M) - 1] += q
    return c


def _V(u, ahat, R, beta, m, P, M, q=1.0):
    """Eq. 9 typed from the paper in the increments d: p(k+i|k) = p(k) + A sum_{tau<min(i,M)} d."""
    V = 0.0
    for i in range(1, P + 1):
        t = min(i, M) - 1
        V += q * (beta + ahat @ u[t]) ** 2
    for t in range(M):
        V += np.sum(R * (u[t] - m) ** 2)
    return V


@pytest.mark.parametrize("n_gpus,P,M", [(1, 4, 2), (2, 8, 2), (4, 8, 2), (8, 8, 3), (3, 8, 1)])
def test_p1_closed_form_interior(oracle_mod, n_gpus, P, M):
    """P1: no bound active -> Sherman-Morrison closed form of
    (c A'A + R) u = R m - c beta A' for every block."""
    d = desc_for(n_gpus, P=P, M=M)
    o = oracle_mod.Oracle(d)
    rng = np.random.default_rng(11)
    ct = _c_blocks(P, M)
    np.testing.assert_array_equal(o.block_weights(), ct)
    checked = 0
    for _ in range(200):
        pr = mpc_problem(rng, d, active_mix=False)
        lo = np.full(o.n, -1e6); hi = np.full(o.n, 1e6)  # bounds far away
        u, act, tie, st, _ = o.mpc(pr["ahat"], pr["R"], pr["beta"], lo, hi, pr["m"])
        assert st == 0
        a, R, m, beta = pr["ahat"], pr["R"], pr["m"], pr["beta"]
        for t in range(M):
            s = (beta + a @ m) / (1.0 + ct[t] * np.sum(a * a / R))
            u_cf = m - ct[t] * s * a / R
            # forward error of a dense solve ~ cond(H) eps, cond(H) <~ 1e4 here
            np.testing.assert_allclose(u[t], u_cf, rtol=1e-11, atol=1e-9)
        assert np.all(act == 0)
        checked += 1
    assert checked == 200


@pytest.mark.parametrize("n_gpus,P,M", [(1, 4, 2), (2, 8, 2), (4, 8, 2), (8, 8, 3)])
def test_p2_kkt(oracle_mod, n_gpus, P, M):
    """P2: KKT of the box-constrained Eq. 9 with the gradient of V taken by
    central finite differences of the literal cost (independent of the oracle's
    H, g): free |grad| small, lower grad >= 0, upper grad <= 0, primal feasible."""
    d = desc_for(n_gpus, P=P, M=M)
    o = oracle_mod.Oracle(d)
    rng = np.random.default_rng(12)
    n_act = 0
    for _ in range(150):
        pr = mpc_problem(rng, d)
        u, act, tie, st, _ = o.mpc(pr["ahat"], pr["R"], pr["beta"], pr["lo"], pr["hi"], pr["m"])
        assert st == 0
        assert np.all(u >= pr["lo"]) and np.all(u <= pr["hi"])
        # analytic-from-definition gradient via finite differences of V
        h = 1e-3
        g = np.zeros_like(u)
        for t in range(M):
            for j in range(o.n):
                up = u.copy(); up[t, j] += h
                um = u.copy(); um[t, j] -= h
                g[t, j] = (_V(up, pr["ahat"], pr["R"], pr["beta"], pr["m"], P, M)
                           - _V(um, pr["ahat"], pr["R"], pr["beta"], pr["m"], P, M)) / (2 * h)
        scale = 1e-6 * max(1.0, np.max(np.abs(g)))
        for t in range(M):
            for j in range(o.n):
                at_lo = u[t, j] == pr["lo"][j]
                at_hi = u[t, j] == pr["hi"][j]
                if at_lo:
                    assert g[t, j] >= -scale
                    n_act += 1
                elif at_hi:
                    assert g[t, j] <= scale
                    n_act += 1
                else:
                    assert abs(g[t, j]) <= scale
    assert n_act > 20  # the draw exercises active bounds


@pytest.mark.parametrize("n_gpus,M", [(1, 2), (2, 2), (3, 2), (1, 3), (1, 4), (4, 1), (7, 1)])
def test_p3_bruteforce(oracle_mod, n_gpus, M):
    """P3: 3^(MN) active-set enumeration agrees with the active-set solve."""
    d = desc_for(n_gpus, P=8, M=M)
    o = oracle_mod.Oracle(d)
    rng = np.random.default_rng(13)
    for _ in range(60):
        pr = mpc_problem(rng, d)
        u, *_ = o.mpc(pr["ahat"], pr["R"], pr["beta"], pr["lo"], pr["hi"], pr["m"])
        ub = o.mpc_bruteforce(pr["ahat"], pr["R"], pr["beta"], pr["lo"], pr["hi"], pr["m"])
        np.testing.assert_allclose(u, ub, rtol=1e-11, atol=1e-8)


@pytest.mark.parametrize("n_gpus,P,M", [(1, 4, 2), (2, 8, 2), (4, 8, 2), (8, 8, 3), (8, 64, 8)])
def test_bvls_library(oracle_mod, n_gpus, P, M):
    """Eq. 9 is a box-constrained linear least-squares problem ("least squares
    solver"): V = ||G u + beta||_Q^2 + ||R^(1/2)(u - m)||^2.  scipy's
    bounded-variable LS (exact active-set, independent library) must agree."""
    d = desc_for(n_gpus, P=P, M=M)
    o = oracle_mod.Oracle(d)
    rng = np.random.default_rng(14)
    n = o.n
    for _ in range(40):
        pr = mpc_problem(rng, d)
        a, R, beta, m = pr["ahat"], pr["R"], pr["beta"], pr["m"]
        rows, rhs = [], []
        for i in range(1, P + 1):
            t = min(i, M) - 1
            r = np.zeros(M * n); r[t * n:(t + 1) * n] = a
            rows.append(r); rhs.append(-beta)
        for t in range(M):
            for j in range(n):
                r = np.zeros(M * n); r[t * n + j] = np.sqrt(R[j])
                rows.append(r); rhs.append(np.sqrt(R[j]) * m[j])
        res = lsq_linear(np.array(rows), np.array(rhs), bounds=(np.tile(pr["lo"], M), np.tile(pr["hi"], M)),
                         method="bvls", tol=1e-14, lsmr_tol=None)
        u, *_ = o.mpc(a, R, beta, pr["lo"], pr["hi"], m)
        Vo = _V(u, a, R, beta, m, P, M)
        Vs = _V(res.x.reshape(M, n), a, R, beta, m, P, M)
        assert Vo <= Vs * (1 + 1e-12) + 1e-9
        np.testing.assert_allclose(u.ravel(), res.x, rtol=1e-8, atol=1e-6)


def test_slsqp_increment_form(oracle_mod):
    """Eq. 9 / 10a solved literally in the increments d(k+i|k) with the paper's
    solver family (SLSQP): cumulative constraints f_min <= f + sum d <= f_max."""
    d = desc_for(2, P=8, M=2)
    o = oracle_mod.Oracle(d)
    rng = np.random.default_rng(15)
    n, M, P = o.n, 2, 8
    for _ in range(15):
        pr = mpc_problem(rng, d)
        f, a, R, m, lo, hi = pr["f"], pr["ahat"], pr["R"], pr["m"], pr["lo"], pr["hi"]
        p0 = pr["p"]; Ps = pr["cap"]

        def V(dv):
            dd = dv.reshape(M, n)
            tot = 0.0
            for i in range(1, P + 1):
                cum = dd[:min(i, M)].sum(axis=0)
                tot += (p0 + a @ cum - Ps) ** 2
            fk = f.copy()
            for t in range(M):
                tot += np.sum(R * (dd[t] + fk - m) ** 2)
                fk = fk + dd[t]
            return tot

        cons = []
        for t in range(M):
            cons.append(dict(type="ineq", fun=lambda dv, t=t: f + dv.reshape(M, n)[:t + 1].sum(axis=0) - lo))
            cons.append(dict(type="ineq", fun=lambda dv, t=t: hi - f - dv.reshape(M, n)[:t + 1].sum(axis=0)))
        res = minimize(V, np.zeros(M * n), method="SLSQP", constraints=cons,
                       options=dict(ftol=1e-14, maxiter=500))
        u, *_ = o.mpc(a, R, pr["beta"], lo, hi, m)
        d_o = np.diff(np.vstack([f, u]), axis=0)
        assert V(d_o.ravel()) <= res.fun * (1 + 1e-9) + 1e-9
        np.testing.assert_allclose(d_o.ravel(), res.x, atol=5e-2)


@pytest.mark.parametrize("n_gpus,step", [(1, 1.0), (2, 5.0)])
def test_p4_grid_search(oracle_mod, n_gpus, step):
    """P4: exhaustive grid over the box (1 MHz for 1 CPU + 1 GPU, 5 MHz for
    1 CPU + 2 GPUs), single block M = 1: J(u*) <= J_grid <= J(u*) + 1/2 lmax(H) N (h/2)^2."""
    d = desc_for(n_gpus, P=4, M=1)
    o = oracle_mod.Oracle(d)
    rng = np.random.default_rng(16)
    n = o.n
    for _ in range(4):
        pr = mpc_problem(rng, d)
        a, R, beta, m, lo, hi = pr["ahat"], pr["R"], pr["beta"], pr["m"], pr["lo"], pr["hi"]
        axes = [np.arange(lo[j], hi[j] + 1e-9, step) for j in range(n)]
        grids = np.meshgrid(*axes, indexing="ij")
        U = np.stack([g.ravel() for g in grids], axis=1)
        J = 4.0 * (beta + U @ a) ** 2 + ((U - m) ** 2 * R).sum(axis=1)
        jg = J.min()
        u, *_ = o.mpc(a, R, beta, lo, hi, m)
        js = o.mpc_cost(a, R, beta, m, u)
        H = 2 * (4.0 * np.outer(a, a) + np.diag(R))
        lmax = np.linalg.eigvalsh(H).max()
        assert js <= jg * (1 + 1e-12) + 1e-9
        assert jg <= js + 0.5 * lmax * n * (step / 2) ** 2 + 1e-9


@pytest.mark.parametrize("n_gpus,P,M", [(2, 8, 2), (4, 8, 2), (8, 8, 3)])
def test_p13_stacked_equals_blocks(oracle_mod, n_gpus, P, M):
    """P13: the stacked problem decouples per control step; each block t solved
    alone (scipy bvls on c_t (beta + A.u)^2 + sum R (u - m)^2) equals the
    oracle's stacked solve.  This is the fact the CUDA path relies on (Q11)."""
    d = desc_for(n_gpus, P=P, M=M)
    o = oracle_mod.Oracle(d)
    rng = np.random.default_rng(17)
    ct = _c_blocks(P, M)
    n = o.n
    for _ in range(40):
        pr = mpc_problem(rng, d)
        a, R, beta, m = pr["ahat"], pr["R"], pr["beta"], pr["m"]
        u, *_ = o.mpc(a, R, beta, pr["lo"], pr["hi"], m)
        for t in range(M):
            A = np.vstack([np.sqrt(ct[t]) * a[None, :], np.diag(np.sqrt(R))])
            b = np.concatenate([[-np.sqrt(ct[t]) * beta], np.sqrt(R) * m])
            res = lsq_linear(A, b, bounds=(pr["lo"], pr["hi"]), method="bvls", tol=1e-14)
            np.testing.assert_allclose(u[t], res.x, rtol=1e-8, atol=1e-6)


def test_active_set_classification(oracle_mod):
    """Q19: the 2-bit active codes agree with where the solution sits."""
    d = desc_for(4, P=8, M=2)
    o = oracle_mod.Oracle(d)
    rng = np.random.default_rng(18)
    for _ in range(200):
        pr = mpc_problem(rng, d)
        u, act, tie, st, _ = o.mpc(pr["ahat"], pr["R"], pr["beta"], pr["lo"], pr["hi"], pr["m"])
        for t in range(o.M):
            for j in range(o.n):
                code = (int(act[t]) >> (2 * j)) & 3
                if (int(tie[t]) >> (2 * j)) & 3:
                    continue
                if code == 1:
                    assert u[t, j] == pr["lo"][j]
                elif code == 2:
                    assert u[t, j] == pr["hi"][j]
                else:
                    assert pr["lo"][j] < u[t, j] < pr["hi"][j]
