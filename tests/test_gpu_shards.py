"""Shard invariance of the independent-server configs ("1/2/4/8-GPU
outputs are bitwise identical"): one context holding the whole global problem
against 2, 4 and 8 contexts holding contiguous 1024-aligned sub-ranges (the
strong-scaling shards bench.py gives each GPU), on one GPU.  Every per-instance
summary, final power and plant state must agree BITWISE: the per-instance
arithmetic depends only on the global server id, and neither the launch
schedule (chunked or not, 32- or 128-wide CTAs) nor the shard boundary
changes its rounding."""
import numpy as np
import pytest

from gen import configs
from tests.test_gpu_parity import G, H  # noqa: F401  (fixture + helper)

pytestmark = pytest.mark.gpu

KEYS = ("final_p", "sum_p", "sumsq_p", "max_p", "sum_theta", "n_viol", "n_window", "act_count")


def _run(G, d, n, begin, K):
    g = G.CapGPU.from_config(d, n_servers=n, srv_begin=begin, n_servers_global=d["n_servers"])
    out = {k: H(v) for k, v in g.simulate(K, G.workload_from(d)).items()}
    st = {k: H(v) for k, v in g.sim_state().items()}
    del g
    return out, st


@pytest.mark.parametrize("cfg,n,K", [(3, 49152, 300), (5, 4096, 200), (2, 4096, 300)])
@pytest.mark.parametrize("shards", [2, 4, 8])
def test_subrange_shards_bitwise(G, cfg, n, K, shards):
    d = configs.get(cfg, n_servers=n)
    caps = d["workload"]["n_caps"]
    one, one_st = _run(G, d, n, 0, K)
    per = n // shards
    assert per % 1024 == 0 or n < 1024 * shards
    for r in range(shards):
        part, part_st = _run(G, d, per, r * per, K)
        sl = slice(r * per * caps, (r + 1) * per * caps)
        for k in KEYS:
            a = one[k][..., sl] if one[k].ndim > 1 else one[k][sl]
            assert np.array_equal(part[k], a), (cfg, shards, r, k)
        for k in one_st:
            a = one_st[k][..., sl] if one_st[k].ndim > 1 else one_st[k][sl]
            assert np.array_equal(part_st[k], a), (cfg, shards, r, k)
