"""GPU parity of the NEXT-2 baseline controllers (§6.1; DESIGN.md
Q32-Q35) through the C ABI against the oracle: commands within 1e-9 relative,
p within 1e-6 W, delta-sigma levels / weights / violation and miss counts exact
(the Fixed-step choice is an integer decision on IEEE weights)."""
import numpy as np
import pytest

from gen import configs
from tests.test_gpu_parity import G, H  # noqa: F401  (fixture + helpers)

pytestmark = pytest.mark.gpu


def _compare(G, oracle_mod, d, n, tr, periods, chunks=None):
    g = G.CapGPU.from_config(d, n_servers=n)
    wl = G.workload_from(d)
    if chunks is None:
        gp = {k: H(v) for k, v in g.simulate(periods, wl, trace_inst=tr).items()}
    else:
        parts = [{k: H(v) for k, v in g.simulate(c, wl, trace_inst=tr).items()} for c in chunks]
        gp = {k: np.concatenate([pp[k] for pp in parts], axis=0) for k in parts[0] if k.startswith("tr_")}
        gp.update({k: parts[-1][k] for k in ("final_p",)})
    o = oracle_mod.Oracle(d)
    ref = o.simulate_baseline(tr, periods=periods)
    np.testing.assert_allclose(gp["tr_p"], ref["p"], rtol=0, atol=1e-6)
    np.testing.assert_allclose(gp["tr_cap"], ref["cap"], rtol=1e-12)
    np.testing.assert_allclose(gp["tr_u"][:, 0], np.transpose(ref["u"], (0, 2, 1)), rtol=1e-9, atol=1e-9)
    assert np.array_equal(gp["tr_levels"], np.transpose(ref["levels"], (0, 2, 3, 1)))
    assert np.array_equal(gp["tr_theta"], np.transpose(ref["theta"], (0, 2, 1)))
    np.testing.assert_allclose(gp["final_p"][tr], ref["final_p"], rtol=0, atol=1e-6)
    if chunks is None:
        sample = np.unique(np.concatenate([tr, np.arange(0, n, max(1, n // 48))]))
        r2 = o.simulate_baseline(sample, periods=periods, traces=False)["summary"]
        np.testing.assert_allclose(gp["sum_p"][sample], r2["sum_p"], rtol=0, atol=1e-6 * periods)
        assert np.array_equal(gp["n_viol"][sample], r2["n_viol"])
        assert np.array_equal(gp["n_miss"][sample], r2["n_miss"])
        np.testing.assert_allclose(gp["sum_theta"][sample], r2["sum_theta"], rtol=1e-12)
    return gp, ref


@pytest.mark.parametrize("kind,steps", [("fixed", 1), ("fixed", 5), ("safe", 1), ("gpuonly", 1), ("cpuonly", 1)])
def test_baseline_parity(G, oracle_mod, kind, steps):
    d = configs.baseline(kind, n_servers=300, periods=400, fs_levels=steps)
    _compare(G, oracle_mod, d, 300, np.array([0, 77, 299]), 400)


def test_baseline_with_slo_misses(G, oracle_mod):
    d = configs.baseline("gpuonly", n_servers=128, periods=300, slo=True)
    gp, _ = _compare(G, oracle_mod, d, 128, np.array([0, 127]), 300)
    assert gp["n_miss"].sum() > 0


@pytest.mark.parametrize("n_gpus", [1, 8, 15])
def test_baseline_shapes_and_chunks(G, oracle_mod, n_gpus):
    d = configs.baseline("fixed", n_servers=97, periods=180, fs_levels=2)
    d["n_gpus"] = n_gpus
    d["knobs"] = configs.knobs(n_gpus)
    _compare(G, oracle_mod, d, 97, np.array([0, 50, 96]), 180, chunks=[60, 60, 60])


def test_baseline_controller_is_fixed_per_simulation(G):
    d = configs.baseline("fixed", n_servers=8, periods=10)
    g = G.CapGPU.from_config(d, n_servers=8)
    g.simulate(10, G.workload_from(d))
    d2 = configs.baseline("gpuonly", n_servers=8, periods=10)
    with pytest.raises(G.CapGPUError, match="call order"):
        g.simulate(10, G.workload_from(d2))
    g.sim_reset()
    g.simulate(10, G.workload_from(d2))


@pytest.mark.parametrize("share,n_gpus", [(0.5, 4), (0.6, 4), (0.82, 4), (0.8, 1), (0.85, 8)])
def test_cpu_gpu_parity(G, oracle_mod, share, n_gpus):
    """CPU+GPU (Q39): two loops on separately metered CPU and GPU power,
    the paper's 50/50 and 60/40 splits and splits where both loops act;
    chunked calls carry both loop commands and recompute the CPU meter."""
    d = configs.baseline("cpugpu", n_servers=150, periods=240, gpu_share=share)
    d["n_gpus"] = n_gpus
    d["knobs"] = configs.knobs(n_gpus)
    _compare(G, oracle_mod, d, 150, np.array([0, 70, 149]), 240, chunks=[80, 80, 80])


def test_cpu_gpu_share_validated(G):
    d = configs.baseline("cpugpu", n_servers=8, periods=10, gpu_share=1.0)
    g = G.CapGPU.from_config(d, n_servers=8)
    with pytest.raises(G.CapGPUError, match="gpu_share"):
        g.simulate(10, G.workload_from(d))
