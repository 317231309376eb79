"""Pins of the oracle's S0 identification and S1 online model update
(DESIGN.md §4 P9, P10).  P:NNN = /root/reference/PAPER.md line."""
import numpy as np
import pytest

from tests.inputs import desc_for


@pytest.mark.parametrize("n_gpus", [1, 2, 4, 8])
def test_p10_noiseless_sweep_exact(oracle_mod, n_gpus):
    """P10: the paper's sweep on a noiseless linear plant
    recovers (A, C) exactly and R^2 = 1."""
    d = desc_for(n_gpus, noise_std=0.0)
    o = oracle_mod.Oracle(d)
    for server in range(20):
        g = o.gen_server(server)
        A, Cc, r2 = o.identify_server(server)
        np.testing.assert_allclose(A, g["a_true"], rtol=1e-11)
        assert abs(Cc - g["c_true"]) <= 1e-9 * g["c_true"]
        assert abs(r2 - 1.0) <= 1e-12


@pytest.mark.parametrize("n_gpus", [1, 4, 8])
def test_identify_vs_numpy_lstsq(oracle_mod, n_gpus):
    """Independent library: numpy's SVD least squares on the same sweep rows."""
    d = desc_for(n_gpus)
    o = oracle_mod.Oracle(d)
    for server in range(10):
        F, p = o.sweep_rows(server)
        rows = F.shape[0]
        assert rows == sum(k["n_levels"] for k in d["knobs"])
        X = np.hstack([F, np.ones((rows, 1))])
        x, *_ = np.linalg.lstsq(X, p, rcond=None)
        A, Cc, r2 = o.identify_ls(F, p)
        np.testing.assert_allclose(A, x[:-1], rtol=1e-10, atol=1e-12)
        assert abs(Cc - x[-1]) <= 1e-9 * abs(x[-1])
        r2_np = 1 - np.sum((p - X @ x) ** 2) / np.sum((p - p.mean()) ** 2)
        assert abs(r2 - r2_np) <= 1e-12


def test_p10_r2_calibration(oracle_mod):
    """P10: with meter noise sigma = 11 W the paper's 1 CPU + 1 GPU sweep gives
    R^2 ~ 0.96 (P:183 reports 0.96): mean over servers within +-0.02."""
    o = oracle_mod.Oracle(desc_for(1))
    r2 = np.array([o.identify_server(s)[2] for s in range(1000)])
    assert abs(r2.mean() - 0.96) <= 0.02


def _random_history(rng, n, K, a, c0, noise=0.0):
    F = np.empty((K, n))
    lo = np.array([1100.0] + [435.0] * (n - 1)); hi = np.array([2400.0] + [1350.0] * (n - 1))
    for k in range(K):
        F[k] = lo + (hi - lo) * rng.random(n)
    p = c0 + F @ a + noise * rng.standard_normal(K)
    return F, p


@pytest.mark.parametrize("n_gpus", [1, 2, 4, 8])
def test_p9_recursive_equals_definition(oracle_mod, n_gpus):
    """P9: the recursive weighted-Welford state equals the two-pass definition
    (lambda-weighted centred LS with ridge toward A0) up to rounding."""
    d = desc_for(n_gpus)
    o = oracle_mod.Oracle(d)
    n = o.n
    rng = np.random.default_rng(21)
    a = np.where(np.arange(n) == 0, 0.05, 0.2)
    A0 = a * (1 + 0.2 * rng.standard_normal(n))
    A0 = np.abs(A0)
    F, p = _random_history(rng, n, 120, a, 300.0, noise=11.0)
    m = o.model_new()
    for k in range(len(p)):
        o.model_push(m, F[k], p[k])
        rec = o.model_solve(m, A0)
        dfn = o.model_definition(F[:k + 1], p[:k + 1], A0)
        np.testing.assert_allclose(rec, dfn, rtol=1e-11, atol=1e-15)


def test_p9_noiseless_excited_recovers_truth(oracle_mod):
    """P9: noiseless, persistently excited, rho -> 0, no clamp: Ahat -> a_true
    (the level form of Eq. 5 with a free intercept)."""
    d = desc_for(4, rho=1e-12, a_lo=-1e9, a_hi=1e9, lam=0.95)
    o = oracle_mod.Oracle(d)
    n = o.n
    rng = np.random.default_rng(22)
    a = np.array([0.05, 0.2, 0.17, 0.22, 0.19])
    F, p = _random_history(rng, n, 60, a, 280.0)
    m = o.model_new()
    for k in range(len(p)):
        o.model_push(m, F[k], p[k])
    est = o.model_solve(m, np.ones(n))
    np.testing.assert_allclose(est, a, rtol=1e-10)


def test_p9_zero_excitation_keeps_prior(oracle_mod):
    """P9: with no excitation (the same z pushed every period) the centred
    scatter stays exactly zero and Ahat = A0 (to the rounding of rho*A0/rho)."""
    d = desc_for(8, rho=100.0)
    o = oracle_mod.Oracle(d)
    n = o.n
    A0 = np.linspace(0.04, 0.3, n)
    m = o.model_new()
    f = np.array([1400.0] + [700.0] * (n - 1))
    for _ in range(50):
        o.model_push(m, f, 1234.5)
        est = o.model_solve(m, A0)
        assert np.all(np.abs(est - A0) <= 2 * np.spacing(A0))
    assert np.all(np.array(m.S_ff)[:n, :n] == 0.0) and np.all(np.array(m.S_fp)[:n] == 0.0)


def test_model_clamp(oracle_mod):
    """Q4: Ahat is clamped to [a_lo, a_hi] * A0 knob by knob."""
    d = desc_for(2, rho=1e-9)
    o = oracle_mod.Oracle(d)
    n = o.n
    rng = np.random.default_rng(23)
    a = np.array([0.05, 0.2, 0.2])
    F, p = _random_history(rng, n, 40, a, 300.0)
    m = o.model_new()
    for k in range(len(p)):
        o.model_push(m, F[k], p[k])
    A0 = np.array([0.01, 0.4, 0.1])  # truth lies outside [0.25, 4] x A0 for knob 0
    est = o.model_solve(m, A0)
    assert est[0] == 4.0 * A0[0]
    np.testing.assert_allclose(est[1:], a[1:], rtol=1e-6)
