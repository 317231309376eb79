"""GPU parity of the NEXT-3 reference trajectory (Q37) through
the C ABI against the oracle's dense stacked QP with the per-row targets
r(k+i|k) = P_s - alpha^i (P_s - p(k)): u within 1e-9 relative, p within 1e-6 W,
level indices and ranks exact, active codes exact except oracle-flagged ties.
Covers the literal blocks (general exact block solve), the move-suppressed
coupled QP, chunked calls and the hierarchical per-period kernel."""
import numpy as np
import pytest

from gen import configs
from tests.inputs import desc_for
from tests.test_gpu_parity import G, H, _sim_compare  # noqa: F401  (fixture + helpers)

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("n_gpus,P,M,alpha", [(2, 8, 2, 0.6), (4, 8, 3, 0.3), (8, 8, 3, 0.8), (3, 8, 1, 0.5),
                                              (1, 6, 4, 0.7)])
def test_ref_closed_loop_parity(G, oracle_mod, n_gpus, P, M, alpha):
    d = desc_for(n_gpus, P=P, M=M, periods=250)
    d["workload"].update(demand_kind=1, cap_frac0=0.2, cap_frac_rand=0.7)
    d["controller"]["ref_alpha"] = alpha
    g, gp, ref = _sim_compare(G, oracle_mod, d, 97, np.array([0, 41, 96]), periods=250)
    sample = np.arange(0, 97, 4)
    r2 = oracle_mod.Oracle(d).simulate(sample, periods=250, traces=False)["summary"]
    np.testing.assert_allclose(g_sum := gp["sum_p"][sample], r2["sum_p"], rtol=0, atol=1e-6 * 250)
    assert np.array_equal(gp["n_viol"][sample], r2["n_viol"]) and g_sum.size == sample.size


def test_ref_cfg2_step_caps_chunked(G, oracle_mod):
    """cfg 2's step schedule of caps (Fig. 10 analogue) with the reference
    trajectory, state carried over three calls."""
    d = configs.get(2, n_servers=128, periods=240)
    d["controller"]["ref_alpha"] = 0.6
    _sim_compare(G, oracle_mod, d, 128, np.array([0, 77, 127]), periods=240, chunks=[80, 80, 80])


@pytest.mark.parametrize("n_gpus,M,W", [(3, 2, 2e-4), (2, 3, 5e-4)])
def test_ref_with_move_suppression(G, oracle_mod, n_gpus, M, W):
    d = configs.move_suppression(n_servers=96, periods=200, wmove=W, n_gpus=n_gpus, P=8, M=M)
    d["controller"]["ref_alpha"] = 0.5
    g, gp, ref = _sim_compare(G, oracle_mod, d, 96, np.array([0, 50, 95]), periods=200)
    assert np.all(gp["tr_status"] & G.ST_SOLVER_CAP == 0)


def test_ref_alpha_out_of_range(G):
    d = configs.get(1)
    d["controller"]["ref_alpha"] = 1.0
    with pytest.raises(G.CapGPUError, match="ref_alpha"):
        G.CapGPU.from_config(d)
