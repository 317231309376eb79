"""cfg 4 hierarchical rack/cluster budget (S5, Q16) on the GPU: parity with
the oracle's lock-step cluster simulation, and shard invariance (1 context vs
2, 4 and 8 loopback shards on one GPU -- the 8-GPU shard logic: bitwise identical)."""
import numpy as np
import pytest
import torch

from gen import configs
from tests.test_gpu_parity import H, active_equal

pytestmark = pytest.mark.gpu

N_SRV, K = 2048, 60


@pytest.fixture(scope="module")
def G():
    from paper_conf_icpp_masw25_b200 import build as B
    B.build()
    from paper_conf_icpp_masw25_b200 import capgpu
    return capgpu


def _desc(periods=K):
    return configs.get(4, periods=periods)


@pytest.mark.parametrize("ref_alpha", [0.0, 0.6])
def test_hierarchical_vs_oracle(G, oracle_mod, ref_alpha):
    """ref_alpha > 0: the NEXT-3 reference trajectory (Q37) on the per-period kernel."""
    d = _desc()
    d["controller"]["ref_alpha"] = ref_alpha
    trs = np.array([0, 17, 1023, 1024, 2047])
    g = G.CapGPU.from_config(d, n_servers=N_SRV, n_servers_global=N_SRV)
    out = {k: H(v) for k, v in g.simulate(K, G.workload_from(d), trace_inst=trs).items()}
    ref = oracle_mod.Oracle(d).simulate_hier(N_SRV, trs, periods=K)
    np.testing.assert_allclose(out["agg_W"], ref["agg_W"], rtol=1e-12)
    np.testing.assert_allclose(out["agg_P"], ref["agg_P"], rtol=1e-12)
    np.testing.assert_allclose(out["tr_cap"], ref["cap"], rtol=1e-10)
    np.testing.assert_allclose(out["tr_p"], ref["p"], rtol=0, atol=1e-6)
    np.testing.assert_allclose(out["tr_u"], np.transpose(ref["u"], (0, 2, 3, 1)), rtol=1e-9, atol=1e-9)
    assert np.array_equal(out["tr_levels"], np.transpose(ref["levels"], (0, 2, 3, 1)))
    bad, _ = active_equal(out["tr_active"], np.transpose(ref["active"], (0, 2, 1)), np.transpose(ref["tie"], (0, 2, 1)))
    assert bad == 0
    np.testing.assert_allclose(out["final_p"], ref["final_p"], rtol=0, atol=1e-6)


@pytest.mark.parametrize("n", [1040, 1041])
def test_hierarchical_ragged_and_odd(G, oracle_mod, n):
    """Server counts off the 32-server warp grid: 1040 (even: the last warp's
    TMA boxes run past n_srv and are zero-filled, those lanes store nothing)
    and 1041 with racks of one server (odd: 8-byte rows are not 16-byte
    aligned, so k_period stages with per-thread cp.async instead of tensor
    maps) -- both against the oracle.  A server count that is not a whole
    number of racks is rejected before any launch."""
    d = _desc(40)
    if n % 16:
        with pytest.raises(G.CapGPUError, match="rack"):
            G.CapGPU.from_config(d, n_servers=n, n_servers_global=n).simulate(1, G.workload_from(d))
        d["workload"]["rack"] = 1
    trs = np.array([0, n // 2, n - 1])
    g = G.CapGPU.from_config(d, n_servers=n, n_servers_global=n)
    out = {k: H(v) for k, v in g.simulate(40, G.workload_from(d), trace_inst=trs).items()}
    ref = oracle_mod.Oracle(d).simulate_hier(n, trs, periods=40)
    np.testing.assert_allclose(out["agg_W"], ref["agg_W"], rtol=1e-12)
    np.testing.assert_allclose(out["agg_P"], ref["agg_P"], rtol=1e-12)
    np.testing.assert_allclose(out["tr_cap"], ref["cap"], rtol=1e-10)
    np.testing.assert_allclose(out["tr_p"], ref["p"], rtol=0, atol=1e-6)
    assert np.array_equal(out["tr_levels"], np.transpose(ref["levels"], (0, 2, 3, 1)))
    np.testing.assert_allclose(out["final_p"], ref["final_p"], rtol=0, atol=1e-6)


def test_nccl_one_rank_bitwise(G):
    """The library's NCCL path on one GPU: a one-rank communicator created by
    capgpu_create from capgpu_nccl_unique_id (ncclCommInitRank) and the
    per-period ncclAllReduce of the padded block vector (inside the CUDA graph
    of the period loop) give results bitwise identical to the communicator-free
    identity reduction."""
    import os
    os.environ.setdefault("NCCL_SOCKET_IFNAME", "lo")  # the bootstrap needs no network for one rank
    d = _desc(40)
    wl = G.workload_from(d)
    n = 2048
    trs = np.array([3, 1500])
    plain = G.CapGPU.from_config(d, n_servers=n, n_servers_global=n)
    o1 = {k: H(v) for k, v in plain.simulate(40, wl, trace_inst=trs).items()}
    nc = G.CapGPU.from_config(d, n_servers=n, n_servers_global=n, world=1, rank=0, nccl_id=G.nccl_unique_id())
    o2 = {k: H(v) for k, v in nc.simulate(40, wl, trace_inst=trs).items()}
    for k in ("agg_W", "agg_P", "tr_p", "tr_cap", "final_p", "sum_p"):
        assert np.array_equal(o1[k], o2[k]), k
    nc.close()
    plain.close()


@pytest.mark.parametrize("shards", [2, 4, 8])
def test_shard_invariance_bitwise(G, shards):
    """1 GPU holding all servers == `shards` loopback shards (same device):
    cluster aggregates, sampled traces and final powers bitwise identical."""
    n = 1024 * shards
    d = _desc(40)
    wl = G.workload_from(d)
    one = G.CapGPU.from_config(d, n_servers=n, n_servers_global=n)
    trs = np.array([5, n // 2 + 3, n - 1])
    o1 = {k: H(v) for k, v in one.simulate(40, wl, trace_inst=trs).items()}
    per = n // shards
    ctxs = [G.CapGPU.from_config(d, n_servers=per, srv_begin=r * per, world=shards, rank=r, n_servers_global=n)
            for r in range(shards)]
    tloc = [np.array([t - r * per for t in trs if r * per <= t < (r + 1) * per]) for r in range(shards)]
    tloc = [t if len(t) else None for t in tloc]
    outs = [{k: H(v) for k, v in o.items()} for o in G.simulate_group(ctxs, 40, wl, trace_insts=tloc)]
    for r in range(shards):
        assert np.array_equal(outs[r]["agg_W"], o1["agg_W"])
        assert np.array_equal(outs[r]["agg_P"], o1["agg_P"])
        assert np.array_equal(outs[r]["final_p"], o1["final_p"][r * per:(r + 1) * per])
    # traced servers
    for q, t in enumerate(trs):
        r = t // per
        j = list(tloc[r]).index(t - r * per)
        assert np.array_equal(outs[r]["tr_p"][:, j], o1["tr_p"][:, q])
        assert np.array_equal(outs[r]["tr_cap"][:, j], o1["tr_cap"][:, q])


def _rack_budgets(d, o, n_total, theta_tr, agg_W, rack=16):
    """B_r of the traced racks recomputed from the Q16 rule: the rack's weights
    of instant max(k-1, 0) (w_i = mean_j theta_ij, traced on the GPU), the
    cluster sum W of that instant (GPU all-reduce + tree) and the generator's
    true models over the whole cluster."""
    wl = d["workload"]
    fmin = np.array([k["f_min"] for k in d["knobs"]])
    fmax = np.array([k["f_max"] for k in d["knobs"]])
    pmin, pmax = np.zeros(n_total), np.zeros(n_total)
    for i in range(n_total):
        g = o.gen_server(i)
        pmin[i] = g["c_true"] + g["a_true"] @ fmin
        pmax[i] = g["c_true"] + g["a_true"] @ fmax
    Bc = pmin.sum() + wl["cluster_frac"] * (pmax.sum() - pmin.sum())
    nt = theta_tr.shape[1]
    Pr = pmin[:nt].reshape(-1, rack).sum(axis=1)
    Brack = wl["rack_frac"] * pmax[:nt].reshape(-1, rack).sum(axis=1)
    w = theta_tr.mean(axis=2)  # [K][nt]
    K = w.shape[0]
    Br = np.zeros((K, nt // rack))
    for k in range(K):
        kp = max(k - 1, 0)  # instant 0 uses the initial weights, whose cluster sum equals agg_W[0]
        Wr = w[kp].reshape(-1, rack).sum(axis=1)
        Br[k] = np.minimum(Brack, Pr + (Bc - pmin.sum()) * Wr / agg_W[kp])
    return Br


def test_hierarchical_replay_at_scale(G, oracle_mod):
    """Sampled racks of a larger cluster (16 racks x
    1,000 periods in replay mode): one GPU shard of cfg 4 (131,072 servers);
    the oracle takes the GPU's cluster sums W(k) (checked against a full oracle
    run above) and recomputes the first 16 racks' caps and closed loops.  Each
    traced rack's caps sum to its budget B_r recomputed from the Q16 rule."""
    n, K2 = 131072, 1000
    d = _desc(K2)
    g = G.CapGPU.from_config(d, n_servers=n, n_servers_global=n)
    trs = np.arange(256)  # racks 0..15
    out = {k: H(v) for k, v in g.simulate(K2, G.workload_from(d), trace_inst=trs).items()}
    W = out["agg_W"]
    o = oracle_mod.Oracle(d)
    ref = o.simulate_hier(256, trs, periods=K2, W_replay=W, W0_replay=W[0], n_total=n)
    np.testing.assert_allclose(out["tr_cap"], ref["cap"], rtol=1e-10)
    np.testing.assert_allclose(out["tr_p"], ref["p"], rtol=0, atol=1e-6)
    np.testing.assert_allclose(out["tr_u"], np.transpose(ref["u"], (0, 2, 3, 1)), rtol=1e-9, atol=1e-9)
    assert np.array_equal(out["tr_levels"], np.transpose(ref["levels"], (0, 2, 3, 1)))
    np.testing.assert_allclose(out["tr_theta"], np.transpose(ref["theta"], (0, 2, 1)), rtol=1e-12)
    # per-rack conservation (Q16): each rack's caps sum to its budget B_r
    Br = _rack_budgets(d, o, n, np.transpose(out["tr_theta"], (0, 2, 1)), W)
    caps = out["tr_cap"].reshape(K2, 16, 16).sum(axis=2)
    np.testing.assert_allclose(caps, Br, rtol=1e-10)
