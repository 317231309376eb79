"""GPU parity of the NEXT-1 SLO schedule (§6.4, Eq. 10b-c; DESIGN.md
Q29-Q31) through the C ABI against the oracle: traces element by element
(u within 1e-9 relative, p within 1e-6 W, level indices / active sets / status
bits exact) and the per-instance deadline-miss counts exactly."""
import numpy as np
import pytest

from gen import configs
from tests.test_gpu_parity import G, H, _sim_compare  # noqa: F401  (fixture + helpers)

pytestmark = pytest.mark.gpu


def _miss_and_status(G, oracle_mod, d, n, tr, periods):
    g, gp, ref = _sim_compare(G, oracle_mod, d, n, tr, periods=periods)
    assert np.array_equal(gp["tr_status"], ref["status"])  # CAP_ and SLO_INFEASIBLE bits
    sample = np.unique(np.concatenate([tr, np.arange(0, n, max(1, n // 64))]))
    r2 = oracle_mod.Oracle(d).simulate(sample, periods=periods, traces=False)["summary"]
    assert np.array_equal(gp["n_miss"][sample], r2["n_miss"])
    assert np.array_equal(gp["n_viol"][sample], r2["n_viol"])
    np.testing.assert_allclose(gp["sum_p"][sample], r2["sum_p"], rtol=0, atol=1e-6 * periods)
    return gp, ref


def test_slo_schedule_parity(G, oracle_mod):
    """The §6.4 schedule (switch at 14, back at 114, period 200) on 1 CPU + 3 GPUs."""
    d = configs.slo_schedule(n_servers=300, periods=420)
    gp, ref = _miss_and_status(G, oracle_mod, d, 300, np.array([0, 7, 150, 299]), 420)
    assert ref["summary"]["n_miss"].sum() == 0  # feasible SLOs are met


def test_slo_infeasible_and_blind_knobs(G, oracle_mod):
    """An unreachable SLO in phase A (ratio < 1 -> bound f_max, SLO_INFEASIBLE,
    misses every sub-step), a tight CPU SLO in phase B, N = 5."""
    d = configs.slo_schedule(n_servers=200, periods=260, slo_period=100, slo_lo=30, slo_hi=70)
    d["n_gpus"] = 4
    d["knobs"] = configs.knobs(4)
    d["workload"].update(slo_a=[0.0, 0.95, 1.35, 0.0, 1.6], slo_b=[1.1, 1.15, 0.0, 1.35, 1.35])
    gp, ref = _miss_and_status(G, oracle_mod, d, 200, np.array([0, 99, 199]), 260)
    assert np.any(ref["status"] & 2) and gp["n_miss"].sum() > 0


@pytest.mark.parametrize("n_gpus,M", [(8, 3), (2, 1)])
def test_slo_shapes(G, oracle_mod, n_gpus, M):
    """N = 9 with M = 3 (the cfg 3 shape) and N = 3 with M = 1, ragged counts."""
    d = configs.slo_schedule(n_servers=97, periods=230)
    d["n_gpus"], d["M"] = n_gpus, M
    d["knobs"] = configs.knobs(n_gpus)
    d["workload"].update(slo_a=[0.0] + [1.35] * n_gpus, slo_b=[0.0] + [1.15, 1.6] * (n_gpus // 2) + [1.6] * (n_gpus % 2))
    _miss_and_status(G, oracle_mod, d, 97, np.array([0, 50, 96]), 230)


def test_slo_chunked_calls_keep_the_phase(G, oracle_mod):
    """The phase is a function of the global period index: 3 calls of 60 == 180."""
    d = configs.slo_schedule(n_servers=64, periods=180, slo_period=50, slo_lo=14, slo_hi=33)
    _sim_compare(G, oracle_mod, d, 64, np.array([0, 63]), periods=180, chunks=[60, 60, 60])


def test_slo_off_is_the_default_path(G, oracle_mod):
    """All-zero SLO ratios: the library takes the SLO-free (convex) path and the
    miss counter stays 0."""
    d = configs.slo_schedule(n_servers=64, periods=100)
    d["workload"].update(slo_period=0, slo_a=None, slo_b=None)
    g, gp, ref = _sim_compare(G, oracle_mod, d, 64, np.array([0, 63]), periods=100)
    assert gp["n_miss"].sum() == 0


@pytest.mark.slow
def test_slo_bench_size_sampled(G, oracle_mod):
    """The bench workload (1,048,576 servers x 1,000 periods) in the bench's
    launch configuration; 16 sampled servers element by element."""
    d = configs.by_name("slo")
    tr = np.linspace(0, d["n_servers"] - 1, 16).astype(np.int64)
    g, gp, ref = _sim_compare(G, oracle_mod, d, d["n_servers"], tr)
    assert np.array_equal(gp["tr_status"], ref["status"])
    assert np.array_equal(gp["n_miss"][tr], ref["summary"]["n_miss"])
