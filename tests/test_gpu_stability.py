"""NEXT-4 on the GPU: the batched gain-mismatch sweep (§4.4).
(1) Parity with the oracle element by element on traced instances spanning the
stable and the unstable side of g*; (2) at scale (16,384 servers x 24 gains x
1,000 periods, `bench.py --config stab`) the per-instance summaries obey the
closed-form pole analysis of tests/stability.py."""
import numpy as np
import pytest

from gen import configs
from tests import stability as ST
from tests.test_gpu_parity import G, H, _sim_compare  # noqa: F401  (G is a fixture)

pytestmark = pytest.mark.gpu


def test_stability_sweep_parity(G, oracle_mod):  # noqa: F811
    d = configs.stability_sweep(n_servers=37, n_gains=24, periods=300)
    ng = 24
    tr = np.concatenate([np.arange(0, ng), 36 * ng + np.arange(0, ng, 3), [17 * ng + 11]]).astype(np.int64)
    _sim_compare(G, oracle_mod, d, 37, tr, periods=300)


def test_stability_sweep_chunked(G, oracle_mod):  # noqa: F811
    d = configs.stability_sweep(n_servers=8, n_gains=24, periods=240)
    _sim_compare(G, oracle_mod, d, 8, np.arange(0, 8 * 24, 5).astype(np.int64), periods=240, chunks=[100, 140])


def test_stability_sweep_closed_form_at_scale(G, oracle_mod):  # noqa: F811
    d = configs.by_name("stab")  # bench size and launch
    K, ns = d["periods"], d["n_servers"]
    gains = ST.gains(d)
    ng = len(gains)
    g = G.CapGPU.from_config(d)
    out = {k: H(v) for k, v in g.simulate(K, G.workload_from(d)).items()}
    o = oracle_mod.Oracle(d)
    fmin, fmax, _, _ = ST.knob_arrays(d)
    W = int(out["n_window"][0])
    assert W == K - (K - (4 * K) // 5)
    n_stable = n_unstable = 0
    for s in range(0, ns, 7):
        gs = o.gen_server(s)
        a, C = gs["a_true"], gs["c_true"]
        for c, gn in enumerate(gains):
            i = s * ng + c
            cap = 0.5 * ((C + gn * (a @ fmin)) + (C + gn * (a @ fmax)))
            info = ST.analyse(d, a, C, cap, gn)
            mean = out["sum_p"][i] / W
            var = max(out["sumsq_p"][i] / W - mean * mean, 0.0)
            if abs(info["rho"]) <= 0.9:
                assert abs(mean - info["p_star"]) <= ST.mean_bound(info, gn, W) + 1e-6, (s, gn)
                assert out["max_p"][i] - info["p_star"] <= info["dev_bound"] + 1e-6, (s, gn)
                assert out["n_viol"][i] <= W
                n_stable += 1
            elif abs(info["rho"]) >= 1.1:
                assert np.sqrt(var) >= 0.1 * info["p_range"], (s, gn, np.sqrt(var))
                n_unstable += 1
    assert n_stable > 5000 and n_unstable > 5000
