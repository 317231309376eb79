"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle on the
same seeded inputs.  Bars (north star / SURVEY §8(c.4)): FP64 frequencies and
powers within 1e-9 relative, closed-loop power traces within 1e-6 W, integer
outputs (active sets, level indices, ranks) bit-exact except oracle-flagged
ties (Q19)."""
import numpy as np
import pytest
import torch

from gen import configs
from tests.inputs import desc_for, mpc_problem

pytestmark = pytest.mark.gpu

RTOL = 1e-9


@pytest.fixture(scope="module")
def G():
    from paper_conf_icpp_masw25_b200 import build as B
    B.build()
    from paper_conf_icpp_masw25_b200 import capgpu
    assert torch.cuda.is_available()
    return capgpu


def T(x, dtype=torch.float64):
    return torch.as_tensor(np.ascontiguousarray(x), dtype=dtype, device="cuda")


def H(t):
    torch.cuda.synchronize()
    return t.cpu().numpy()


def active_equal(a_gpu, a_ora, tie):
    """bit-exact 2-bit codes except where the oracle flags a near-tie (Q19)."""
    a_gpu = a_gpu.astype(np.uint32); a_ora = a_ora.astype(np.uint32); tie = tie.astype(np.uint32)
    diff = (a_gpu ^ a_ora) & ~tie
    return int(np.count_nonzero(diff)), int(np.count_nonzero((a_gpu ^ a_ora) & tie))


# ------------------------------------------------------------------ generator

@pytest.mark.parametrize("cfg", [2, 3, 5])
def test_device_generator_bit_identical(G, oracle_mod, cfg):
    d = configs.get(cfg)
    o = oracle_mod.Oracle(d)
    n = 300
    g = G.CapGPU.from_config(d, n_servers=n)
    for k in (0, 1, 9, 10, 137, 1999):
        out = {k2: H(v) for k2, v in g.debug_gen(k, d["workload"]["demand_kind"], d["workload"]["demand_frac"]).items()}
        for s in range(0, n, 7):
            gs = o.gen_server(s)
            assert np.array_equal(out["a_true"][:, s], gs["a_true"])
            assert np.array_equal(out["thr_max"][:, s], gs["thr_max"])
            assert out["c_true"][s] == gs["c_true"]
            assert np.array_equal(out["dem"][:, s], o.gen_demand(s, k))
            assert out["noise"][s] == o.gen_noise(s, k)


# ------------------------------------------------------------------ S0

@pytest.mark.parametrize("n_gpus", [1, 2, 4, 8, 15])
def test_identify_synthetic_sweep(G, oracle_mod, n_gpus):
    d = desc_for(n_gpus, P=8, M=2)
    o = oracle_mod.Oracle(d)
    n = 77
    g = G.CapGPU.from_config(d, n_servers=n)
    A, Cc, r2 = (H(x) for x in g.identify())
    for s in range(n):
        F, p = o.sweep_rows(s)
        Ao, Co, r2o = o.identify_ls(F, p)
        np.testing.assert_allclose(A[:, s], Ao, rtol=RTOL, atol=1e-12)
        assert abs(Cc[s] - Co) <= RTOL * abs(Co)
        assert abs(r2[s] - r2o) <= 1e-10


def test_identify_user_rows(G, oracle_mod):
    d = desc_for(4)
    o = oracle_mod.Oracle(d)
    n, rows = 50, 40
    rng = np.random.default_rng(41)
    lo = np.array([k["f_min"] for k in d["knobs"]]); hi = np.array([k["f_max"] for k in d["knobs"]])
    F = lo[None, :, None] + (hi - lo)[None, :, None] * rng.random((rows, 5, n))
    a = 0.05 + 0.2 * rng.random((5, n))
    p = 300 + np.einsum("rjn,jn->rn", F, a) + rng.normal(0, 11, (rows, n))
    g = G.CapGPU.from_config(d, n_servers=n)
    A, Cc, r2 = (H(x) for x in g.identify(T(F), T(p)))
    for s in range(n):
        Ao, Co, r2o = o.identify_ls(F[:, :, s], p[:, s])
        np.testing.assert_allclose(A[:, s], Ao, rtol=RTOL, atol=1e-12)
        assert abs(Cc[s] - Co) <= RTOL * abs(Co)
        assert abs(r2[s] - r2o) <= 1e-10


# ------------------------------------------------------------------ S2

def test_assign_weights_bit_exact(G, oracle_mod):
    d = desc_for(8)
    o = oracle_mod.Oracle(d)
    n = 4099  # ragged tail
    rng = np.random.default_rng(42)
    tm = 40 + 160 * rng.random((9, n))
    frac = rng.random((9, n)) * 1.2
    frac[:, ::3] = np.where(rng.random((9, n))[:, ::3] < 0.4, 1.3, frac[:, ::3])  # ties at theta = 1
    frac[:, 1::5] = np.where(rng.random((9, n))[:, 1::5] < 0.4, 0.0, frac[:, 1::5])  # ties at theta_min
    thr = tm * frac
    g = G.CapGPU.from_config(d, n_servers=n)
    th, R, rk = (H(x) for x in g.assign_weights(T(thr), T(tm)))
    for s in range(n):
        tho, Ro, rko = o.weights(thr[:, s], tm[:, s])
        assert np.array_equal(th[:, s], tho)
        assert np.array_equal(R[:, s], Ro)
        assert np.array_equal(rk[:, s], rko)


# ------------------------------------------------------------------ S1-S3 control step

@pytest.mark.parametrize("n_gpus,P,M,n", [(1, 4, 2, 133), (2, 4, 2, 133), (4, 8, 2, 133), (8, 8, 3, 133),
                                           (3, 8, 1, 133), (15, 8, 4, 133),
                                           # several full 128-server CTAs + a ragged tail
                                           (8, 8, 3, 420), (3, 8, 2, 256)])
def test_control_step_sequence(G, oracle_mod, n_gpus, P, M, n):
    """Several consecutive control_step calls on random measurements: model
    state, warm starts and all M blocks against the oracle's S1 (recursive),
    S2 and stacked S3."""
    d = desc_for(n_gpus, P=P, M=M)
    o = oracle_mod.Oracle(d)
    N = o.n
    rng = np.random.default_rng(43 + N)
    g = G.CapGPU.from_config(d, n_servers=n)
    A0 = np.abs(np.where(np.arange(N)[:, None] == 0, 0.05, 0.2) * (1 + 0.2 * rng.standard_normal((N, n)))) + 1e-3
    g.set_prior(T(A0))
    models = [o.model_new() for _ in range(n)]
    lo, hi, m = (np.array([k[x] for k in d["knobs"]]) for x in ("f_min", "f_max", "f_min"))
    tm = 40 + 160 * rng.random((N, n))
    n_tie = 0
    for step in range(12):
        f = lo[:, None] + (hi - lo)[:, None] * rng.random((N, n))
        a_true = np.where(np.arange(N)[:, None] == 0, 0.05, 0.2)
        p = 300 + np.sum(a_true * f, axis=0) + rng.normal(0, 11, n)
        thr = tm * rng.random((N, n)) * 1.1
        pmin = 300 + a_true[:, 0] @ lo; pmax = 300 + a_true[:, 0] @ hi
        cap = pmin + rng.uniform(-0.1, 1.1, n) * (pmax - pmin)
        out = g.control_step(T(p), T(f), T(thr), T(tm), T(cap))
        u, act, rk, ah, st = (H(out[k]) for k in ("u", "active", "rank", "ahat", "status"))
        for s in range(n):
            o.model_push(models[s], f[:, s], p[s])
            aho = o.model_solve(models[s], A0[:, s])
            np.testing.assert_allclose(ah[:, s], aho, rtol=RTOL, atol=1e-15)
            tho, Ro, rko = o.weights(thr[:, s], tm[:, s])
            assert np.array_equal(rk[:, s], rko)
            beta = p[s] - cap[s] - aho @ f[:, s]
            uo, acto, tie, sto, _ = o.mpc(aho, Ro, beta, lo, hi, m)
            np.testing.assert_allclose(u[:, :, s], uo, rtol=RTOL, atol=1e-9)
            bad, ties = active_equal(act[:, s], acto, tie)
            assert bad == 0, (step, s, act[:, s], acto)
            n_tie += ties
            smin = beta + aho @ lo; smax = beta + aho @ hi
            assert bool(st[s] & 1) == (smin > 0 or smax < 0)
            assert st[s] & G.ST_SOLVER_CAP == 0
    assert n_tie == 0


@pytest.mark.parametrize("n_gpus,M", [(2, 2), (4, 2), (5, 3), (8, 3)])
def test_control_step_general_bounds(G, oracle_mod, n_gpus, M):
    """SLO-raised lower bounds l_j > m_j = f_min (Eq. 10b-c): the general block
    solve on random measurements -- block_direct (all 2N breakpoints at once)
    for N <= 6, Newton + the breakpoint fallback for N = 9 -- every block's u
    and codes against the oracle's dense stacked QP with the same box."""
    d = desc_for(n_gpus, P=8, M=M)
    for j, k in enumerate(d["knobs"]):
        if j >= 1:
            k["f_lo"] = 600.0 + 35.0 * j
    o = oracle_mod.Oracle(d)
    N = o.n
    n = 160
    rng = np.random.default_rng(11 + N)
    g = G.CapGPU.from_config(d, n_servers=n)
    A0 = np.abs(np.where(np.arange(N)[:, None] == 0, 0.05, 0.2) * (1 + 0.2 * rng.standard_normal((N, n)))) + 1e-3
    g.set_prior(T(A0))
    models = [o.model_new() for _ in range(n)]
    fmin, hi = (np.array([k[x] for k in d["knobs"]]) for x in ("f_min", "f_max"))
    lo = np.array([k.get("f_lo", k["f_min"]) for k in d["knobs"]])
    tm = 40 + 160 * rng.random((N, n))
    n_tie = 0
    for step in range(10):
        f = fmin[:, None] + (hi - fmin)[:, None] * rng.random((N, n))
        a_true = np.where(np.arange(N)[:, None] == 0, 0.05, 0.2)
        p = 300 + np.sum(a_true * f, axis=0) + rng.normal(0, 11, n)
        thr = tm * rng.random((N, n)) * 1.1
        pmin = 300 + a_true[:, 0] @ lo; pmax = 300 + a_true[:, 0] @ hi
        cap = pmin + rng.uniform(-0.1, 1.1, n) * (pmax - pmin)
        out = g.control_step(T(p), T(f), T(thr), T(tm), T(cap))
        u, act, ah = (H(out[k]) for k in ("u", "active", "ahat"))
        for s in range(n):
            o.model_push(models[s], f[:, s], p[s])
            aho = o.model_solve(models[s], A0[:, s])
            np.testing.assert_allclose(ah[:, s], aho, rtol=RTOL, atol=1e-15)
            _, Ro, _ = o.weights(thr[:, s], tm[:, s])
            beta = p[s] - cap[s] - aho @ f[:, s]
            uo, acto, tie, _, _ = o.mpc(aho, Ro, beta, lo, hi, fmin)
            np.testing.assert_allclose(u[:, :, s], uo, rtol=RTOL, atol=1e-9)
            bad, ties = active_equal(act[:, s], acto, tie)
            assert bad == 0, (step, s, act[:, s], acto)
            n_tie += ties
    assert n_tie == 0


def test_control_step_nonfinite_and_order(G):
    d = desc_for(2)
    g = G.CapGPU.from_config(d, n_servers=8)
    z = T(np.ones(8)); f = T(np.full((3, 8), 1000.0))
    with pytest.raises(G.CapGPUError, match="call order"):
        g.control_step(z, f, f, f, z)
    g.set_prior(T(np.full((3, 8), 0.1)))
    p = np.full(8, 900.0); p[3] = np.nan
    out = g.control_step(T(p), f, f, T(np.full((3, 8), 2000.0)), T(np.full(8, 950.0)))
    st = H(out["status"]); u = H(out["u"])
    assert st[3] == G.ST_NONFINITE and np.all(st[[0, 1, 2, 4]] & G.ST_NONFINITE == 0)
    assert np.array_equal(u[:, :, 3], np.tile([1100.0, 435.0, 435.0], (2, 1)))


# ------------------------------------------------------------------ closed loop

def _sim_compare(G, oracle_mod, d, n_servers, trace_inst, periods=None, chunks=None):
    o = oracle_mod.Oracle(d)
    K = periods or d["periods"]
    g = G.CapGPU.from_config(d, n_servers=n_servers)
    wl = G.workload_from(d)
    if chunks is None:
        out = g.simulate(K, wl, trace_inst=trace_inst)
        gp = {k: H(v) for k, v in out.items()}
    else:
        parts = []
        for c in chunks:
            parts.append({k: H(v) for k, v in g.simulate(c, wl, trace_inst=trace_inst).items()})
        gp = {k: np.concatenate([pp[k] for pp in parts], axis=0) for k in parts[0] if k.startswith("tr_")}
        gp["final_p"] = parts[-1]["final_p"]
    ref = o.simulate(trace_inst, periods=K)
    nt = len(trace_inst)
    # p(k) traces: 1e-6 W; u: 1e-9 relative; integers exact
    np.testing.assert_allclose(gp["tr_p"], ref["p"], rtol=0, atol=1e-6)
    np.testing.assert_allclose(gp["tr_cap"], ref["cap"], rtol=1e-12)
    u_ref = np.transpose(ref["u"], (0, 2, 3, 1))
    np.testing.assert_allclose(gp["tr_u"], u_ref, rtol=RTOL, atol=1e-9)
    assert np.array_equal(gp["tr_levels"], np.transpose(ref["levels"], (0, 2, 3, 1)))
    assert np.array_equal(gp["tr_rank"], np.transpose(ref["rank"], (0, 2, 1)))
    np.testing.assert_allclose(gp["tr_ahat"], np.transpose(ref["ahat"], (0, 2, 1)), rtol=RTOL, atol=1e-15)
    np.testing.assert_allclose(gp["tr_theta"], np.transpose(ref["theta"], (0, 2, 1)), rtol=1e-12)
    bad, ties = active_equal(gp["tr_active"], np.transpose(ref["active"], (0, 2, 1)),
                             np.transpose(ref["tie"], (0, 2, 1)))
    assert bad == 0
    np.testing.assert_array_equal(gp["tr_status"] & 1, ref["status"] & 1)
    np.testing.assert_allclose(gp["final_p"][trace_inst], ref["final_p"], rtol=0, atol=1e-6)
    return g, gp, ref


def test_closed_loop_cfg1_full(G, oracle_mod):
    """cfg 1 (1 server, 1 CPU + 2 GPUs, P/M = 4/2, 200 periods, fixed cap): every output."""
    d = configs.get(1)
    g, gp, ref = _sim_compare(G, oracle_mod, d, 1, np.array([0]))
    s = ref["summary"]
    assert abs(gp["sum_p"][0] - s["sum_p"][0]) <= 1e-6 * s["n_window"][0]
    assert gp["n_window"][0] == s["n_window"][0] and gp["n_viol"][0] == s["n_viol"][0]
    assert abs(gp["max_p"][0] - s["max_p"][0]) <= 1e-6
    assert np.array_equal(gp["act_count"][:, 0], s["act_count"][0])


def test_closed_loop_cfg2_all_servers(G, oracle_mod):
    """cfg 2 (1,024 servers, N = 5, 8/2, 1,000 periods, step cap): 48 traced
    servers element by element, summaries of 256 servers."""
    d = configs.get(2)
    tr = np.arange(0, 1024, 1024 // 48)[:48]
    g, gp, ref = _sim_compare(G, oracle_mod, d, 1024, tr)
    o = oracle_mod.Oracle(d)
    sample = np.arange(0, 1024, 4)
    r2 = o.simulate(sample, traces=False)["summary"]
    np.testing.assert_allclose(gp["sum_p"][sample], r2["sum_p"], rtol=0, atol=1e-6 * 800)
    np.testing.assert_allclose(gp["max_p"][sample], r2["max_p"], rtol=0, atol=1e-6)
    assert np.array_equal(gp["n_viol"][sample], r2["n_viol"])
    np.testing.assert_allclose(gp["sum_theta"][sample], r2["sum_theta"], rtol=1e-9)


def test_closed_loop_chunked_equals_single(G, oracle_mod):
    """State carries across simulate calls: 3 calls of 70 periods == oracle 210."""
    d = configs.get(2)
    _sim_compare(G, oracle_mod, d, 160, np.array([0, 5, 159]), periods=210, chunks=[70, 70, 70])


@pytest.mark.parametrize("n_gpus,P,M,n", [(1, 8, 1, 37), (2, 4, 4, 129), (15, 8, 2, 33), (6, 12, 3, 300)])
def test_closed_loop_shapes(G, oracle_mod, n_gpus, P, M, n):
    """Edge shapes: N = 2 and N = 16 knobs, M = 1 and M = 4, ragged server counts."""
    d = desc_for(n_gpus, P=P, M=M, periods=150)
    d["workload"].update(demand_kind=1, cap_frac0=0.2, cap_frac_rand=0.7)
    _sim_compare(G, oracle_mod, d, n, np.array([0, n // 2, n - 1]), periods=150)


@pytest.mark.parametrize("n_gpus,M", [(2, 2), (8, 3)])
def test_closed_loop_slo_lower_bounds(G, oracle_mod, n_gpus, M):
    """SLO-raised lower bounds l_j > f_min (Eq. 10b-c, Q14) make the block QP
    non-convex in s: exercises the general (safeguarded + exact breakpoint) solve."""
    d = desc_for(n_gpus, P=8, M=M, periods=200)
    for j, k in enumerate(d["knobs"]):
        if j >= 1:
            k["f_lo"] = 600.0 + 40.0 * j  # GPU j must run >= 640.. MHz to meet its SLO
    d["workload"].update(demand_kind=1, cap_frac0=0.1, cap_frac_rand=0.8)
    _sim_compare(G, oracle_mod, d, 97, np.array([0, 13, 96]), periods=200)


def test_closed_loop_infeasible_caps(G, oracle_mod):
    """Caps below P_min / above P_max: CAP_INFEASIBLE and the frequencies pin to
    the box."""
    d = desc_for(4, P=8, M=2, periods=80)
    d["workload"].update(cap_frac0=-0.3)
    _, gp, _ = _sim_compare(G, oracle_mod, d, 64, np.array([0, 1, 63]), periods=80)
    assert np.all(gp["tr_status"][5:] & 1)
    d["workload"].update(cap_frac0=1.4)
    _sim_compare(G, oracle_mod, d, 64, np.array([0, 1, 63]), periods=80)


@pytest.mark.slow
def test_closed_loop_cfg3_full_size(G, oracle_mod):
    """cfg 3 at full size (65,536 servers, N = 9, 8/3, 1,000 periods) in the
    bench's launch configuration; 24 sampled servers compared element by element."""
    d = configs.get(3)
    tr = np.linspace(0, 65535, 24).astype(np.int64)
    _, gp, ref = _sim_compare(G, oracle_mod, d, 65536, tr)
    _summary_compare(gp, ref["summary"], tr)
    # 256 UNTRACED instances (the bench's path: block M-1 reports only its
    # "any bound active" bit, convex_any_upper) against the oracle's summaries
    sample = np.setdiff1d(np.arange(7, 65536, 256), tr)[:256]
    assert len(sample) == 256
    r2 = oracle_mod.Oracle(d).simulate(sample, traces=False)
    _summary_compare(gp, r2["summary"], sample)
    np.testing.assert_allclose(gp["final_p"][sample], r2["final_p"], rtol=0, atol=1e-6)
    assert np.count_nonzero(r2["summary"]["act_count"][:, -1]) > 0  # the last block's bit is exercised


def _summary_compare(gp, s, idx):
    """Per-instance summaries (window sums, max, violations, active-set counts):
    carried across the chunks of the persistent schedule."""
    n_win = s["n_window"]
    np.testing.assert_allclose(gp["sum_p"][idx], s["sum_p"], rtol=0, atol=1e-6 * n_win.max())
    np.testing.assert_allclose(gp["max_p"][idx], s["max_p"], rtol=0, atol=1e-6)
    np.testing.assert_allclose(gp["sum_theta"][idx], s["sum_theta"], rtol=1e-9)
    assert np.array_equal(gp["n_viol"][idx], s["n_viol"])
    assert np.array_equal(gp["n_window"][idx], n_win)
    assert np.array_equal(gp["act_count"][:, idx].T, s["act_count"])


def test_chunked_schedule_matches_single_pass(G, oracle_mod, monkeypatch):
    """The chunked persistent schedule (more instance groups than resident slots,
    DESIGN.md §6) against the one-item-per-CTA launch of the same call: every
    instance's summaries, final power and state are BITWISE identical (the
    scaled model state and its scale lam^-kk are carried across chunks as they
    are, and its folds depend on the call period only), and sampled instances
    match the oracle including the summaries carried across chunks."""
    d = configs.get(3)
    n, K = 65536, 200
    wl = G.workload_from(d)
    monkeypatch.setenv("CAPGPU_NO_CHUNKING", "1")
    g1 = G.CapGPU.from_config(d, n_servers=n)
    monkeypatch.delenv("CAPGPU_NO_CHUNKING")
    one = {k: H(v) for k, v in g1.simulate(K, wl).items()}
    one_st = {k: H(v) for k, v in g1.sim_state().items()}
    del g1
    tr = np.array([0, 777, 40000, 65535])
    g2 = G.CapGPU.from_config(d, n_servers=n)
    ch = {k: H(v) for k, v in g2.simulate(K, wl, trace_inst=tr).items()}
    ch_st = {k: H(v) for k, v in g2.sim_state().items()}
    for k in ("final_p", "sum_p", "sumsq_p", "max_p", "sum_theta", "n_viol", "n_window", "act_count"):
        assert np.array_equal(ch[k], one[k]), k
    for k in one_st:
        assert np.array_equal(ch_st[k], one_st[k]), k
    ref = oracle_mod.Oracle(d).simulate(tr, periods=K)
    np.testing.assert_allclose(ch["tr_p"], ref["p"], rtol=0, atol=1e-6)
    _summary_compare(ch, ref["summary"], tr)


@pytest.mark.parametrize("lam", [0.3, 0.6, 1.0])
def test_forgetting_factor_range(G, oracle_mod, monkeypatch, lam):
    """The fused kernel's scaled model state at small forgetting factors
    (a fixed fold interval overflowed lam^-kk for lam <~ 0.5):
    cfg 3's shape (chunked schedule) for 1,200 periods -- more than one
    1,024-period fold -- against the oracle, and bitwise equal to the
    one-item-per-CTA launch."""
    d = configs.get(3, lam=lam, periods=1200)
    n, K = 65536, 1200
    tr = np.array([0, 3, 32768, 65535])
    g, gp, ref = _sim_compare(G, oracle_mod, d, n, tr, periods=K)
    assert np.all(np.isfinite(gp["tr_ahat"]))
    _summary_compare(gp, ref["summary"], tr)
    monkeypatch.setenv("CAPGPU_NO_CHUNKING", "1")
    g1 = G.CapGPU.from_config(d, n_servers=n)
    monkeypatch.delenv("CAPGPU_NO_CHUNKING")
    one = {k: H(v) for k, v in g1.simulate(K, G.workload_from(d)).items()}
    assert np.array_equal(one["final_p"], gp["final_p"])
    assert np.array_equal(one["n_viol"], gp["n_viol"])


@pytest.mark.slow
def test_closed_loop_cfg5_full_size(G, oracle_mod):
    """cfg 5 at full size (262,144 servers x 32 caps, N = 4, 8/2, 2,000 periods);
    24 sampled (server, cap) instances compared element by element."""
    d = configs.get(5)
    ni = 262144 * 32
    tr = np.concatenate([np.arange(0, 32), np.linspace(32, ni - 1, 8).astype(np.int64)])
    _sim_compare(G, oracle_mod, d, 262144, tr)
