"""GPU parity of the NEXT-3 explicit (multi-parametric) MPC (an offline
part and an online part evaluated as a piecewise linear function) through the
C ABI: the tabulated law u_0(beta) against the oracle's dense stacked active
set QP of Eq. 9 (block 0) with the same model and weights -- u within 1e-9
relative, block-0 codes exact except oracle-flagged ties -- over parameters that
sweep every critical region, and across consecutive online steps on one table."""
import numpy as np
import pytest

from tests.inputs import desc_for
from tests.test_gpu_parity import G, H, T, active_equal  # noqa: F401

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("n_gpus,P,M", [(1, 4, 2), (3, 8, 2), (8, 8, 3), (4, 8, 1)])
def test_explicit_law_matches_qp(G, oracle_mod, n_gpus, P, M):
    d = desc_for(n_gpus, P=P, M=M)
    o = oracle_mod.Oracle(d)
    N = o.n
    n = 257
    rng = np.random.default_rng(97 + N + M)
    g = G.CapGPU.from_config(d, n_servers=n)
    A0 = np.abs(np.where(np.arange(N)[:, None] == 0, 0.05, 0.2) * (1 + 0.2 * rng.standard_normal((N, n)))) + 1e-3
    g.set_prior(T(A0))
    lo, hi, m = (np.array([k[x] for k in d["knobs"]]) for x in ("f_min", "f_max", "f_min"))
    tm = 40 + 160 * rng.random((N, n))
    a_true = np.where(np.arange(N)[:, None] == 0, 0.05, 0.2)
    # a few control steps give the model state a history (the table is built from it)
    for _ in range(6):
        f = lo[:, None] + (hi - lo)[:, None] * rng.random((N, n))
        p = 300 + np.sum(a_true * f, axis=0) + rng.normal(0, 11, n)
        cap = 300 + a_true[:, 0] @ lo + rng.random(n) * (a_true[:, 0] @ (hi - lo))
        out = g.control_step(T(p), T(f), T(tm * rng.random((N, n))), T(tm), T(cap))
    ahat = H(out["ahat"])
    thr = tm * rng.random((N, n)) * 1.1
    g.explicit_build(T(thr), T(tm))
    pmin = 300 + a_true[:, 0] @ lo
    pmax = 300 + a_true[:, 0] @ hi
    n_tie = 0
    regions = set()
    for step in range(8):  # online steps on the same table
        f = lo[:, None] + (hi - lo)[:, None] * rng.random((N, n))
        p = 300 + np.sum(a_true * f, axis=0) + rng.normal(0, 11, n)
        cap = pmin + rng.uniform(-0.2, 1.2, n) * (pmax - pmin)  # every region, both infeasible sides
        ex = g.explicit_step(T(p), T(f), T(cap))
        u, act, st = H(ex["u"]), H(ex["active"]), H(ex["status"])
        for s in range(n):
            _, R, _ = o.weights(thr[:, s], tm[:, s])
            beta = p[s] - cap[s] - ahat[:, s] @ f[:, s]
            uo, acto, tie, _, _ = o.mpc(ahat[:, s], R, beta, lo, hi, m)
            np.testing.assert_allclose(u[:, s], uo[0], rtol=1e-9, atol=1e-9)
            bad, ties = active_equal(act[s:s + 1], acto[:1], tie[:1])
            assert bad == 0, (step, s, act[s], acto[0])
            n_tie += ties
            regions.add(int(np.sum(uo[0] >= hi - 1e-9)))
            smin = beta + ahat[:, s] @ lo
            smax = beta + ahat[:, s] @ hi
            assert bool(st[s] & 1) == (smin > 0 or smax < 0)
    assert n_tie == 0
    assert len(regions) >= min(N, 3)  # several critical regions were visited


def test_explicit_order_and_scope(G):
    d = desc_for(2)
    g = G.CapGPU.from_config(d, n_servers=4)
    z = T(np.ones(4))
    f = T(np.full((3, 4), 1000.0))
    with pytest.raises(G.CapGPUError, match="call order"):
        g.explicit_build(f, f)  # no prior yet
    g.set_prior(T(np.full((3, 4), 0.1)))
    with pytest.raises(G.CapGPUError, match="call order"):
        g.explicit_step(z, f, z)  # no table yet
    d2 = desc_for(2)
    d2["knobs"][1]["f_lo"] = 700.0  # an SLO-style lower bound: not the convex law
    g2 = G.CapGPU.from_config(d2, n_servers=4)
    g2.set_prior(T(np.full((3, 4), 0.1)))
    with pytest.raises(G.CapGPUError, match="unsupported"):
        g2.explicit_build(f, f)
