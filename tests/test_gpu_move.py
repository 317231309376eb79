"""GPU parity of the NEXT-3 horizon-active MPC (Eq. 9 + move suppression,
DESIGN.md Q36) through the C ABI against the oracle's generic dense active set:
u within 1e-9 relative, p within 1e-6 W, level indices exact, active codes exact
except oracle-flagged ties."""
import numpy as np
import pytest

from gen import configs
from tests.test_gpu_parity import G, H, _sim_compare  # noqa: F401  (fixture + helpers)

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("n_gpus,P,M,W", [(3, 8, 2, 2e-4), (2, 8, 3, 5e-4), (1, 6, 4, 1e-4), (4, 8, 2, 3e-3),
                                          (1, 8, 1, 2e-4), (8, 8, 3, 2e-4), (8, 8, 3, 2e-3), (5, 8, 4, 5e-4)])
def test_move_closed_loop_parity(G, oracle_mod, n_gpus, P, M, W):
    d = configs.move_suppression(n_servers=160, periods=300, wmove=W, n_gpus=n_gpus, P=P, M=M)
    g, gp, ref = _sim_compare(G, oracle_mod, d, 160, np.array([0, 33, 159]), periods=300)
    assert np.all(gp["tr_status"] & G.ST_SOLVER_CAP == 0)
    sample = np.arange(0, 160, 5)
    r2 = oracle_mod.Oracle(d).simulate(sample, periods=300, traces=False)["summary"]
    np.testing.assert_allclose(gp["sum_p"][sample], r2["sum_p"], rtol=0, atol=1e-6 * 300)
    assert np.array_equal(gp["n_viol"][sample], r2["n_viol"])


def test_move_chunked(G, oracle_mod):
    d = configs.move_suppression(n_servers=64, periods=150)
    _sim_compare(G, oracle_mod, d, 64, np.array([0, 63]), periods=150, chunks=[50, 50, 50])


def test_move_survey_scale_kkt(G, oracle_mod):
    """SURVEY §8(f) NEXT-3 at its scale: the 1 CPU + 8 GPU server with M = 3
    (27 coupled variables; 3^27 brute force is out of reach): the structured
    active set's u against the oracle's dense generic active set element by
    element over a closed loop, bound feasibility every period, and no
    solver-cap status."""
    d = configs.move_suppression(n_servers=256, periods=200, wmove=5e-4, n_gpus=8, P=8, M=3)
    g, gp, ref = _sim_compare(G, oracle_mod, d, 256, np.array([0, 100, 255]), periods=200)
    assert np.all(gp["tr_status"] & G.ST_SOLVER_CAP == 0)
    lo = np.array([k["f_min"] for k in d["knobs"]]); hi = np.array([k["f_max"] for k in d["knobs"]])
    u = gp["tr_u"]  # [K][M][N][n_trace]
    assert np.all(u >= lo[None, None, :, None]) and np.all(u <= hi[None, None, :, None])


def test_move_unsupported_shapes(G):
    """Stacks beyond M N = 36 (e.g. 1 CPU + 15 GPUs at M = 4: 64 variables) are rejected at create."""
    d = configs.move_suppression(n_servers=8, n_gpus=15, M=4)
    with pytest.raises(G.CapGPUError, match="unsupported"):
        G.CapGPU.from_config(d)
