"""Pins of the oracle's baseline controllers (NEXT-2: §6.1, §6.2
P:293-305; Q32-Q35).  P:NNN = /root/reference/PAPER.md line.

Independent of the oracle's controller code:
  * the plant in closed form: with no meter noise a command on a grid level
    passes the delta-sigma modulator unchanged, so p(k+1) - p(k) equals
    sum_j a_j (u_j(k) - u_j(k-1)) with the TRUE gains from the generator;
  * the Fixed-step rule re-implemented here from the traced weights
    (argmax / argmin over the knobs that can move, round-robin ties) and its
    limit cycle: once the set point is crossed, |p - P_s| stays within the
    largest single-step power change;
  * the pole-placed P loop: with the exact model, e(k+1) = z e(k) up to
    the modulator's quantisation, |e(k+1) - z e(k)| <= sum_J a_j 2 step_j / S,
    on every period where the command does not saturate; zero mean error
    (integral action) in steady state;
  * CPU-only's narrow control range (Fig. 3): the cap below its reach
    pins the CPU at f_min and violates every period.
"""
import numpy as np
import pytest

from gen import configs


def _quiet(kind, n=6, periods=160, **kw):
    d = configs.baseline(kind, n_servers=n, periods=periods, **kw)
    d["controller"]["noise_std"] = 0.0
    d["workload"].update(demand_kind=0, cap_period=0)
    return d


def _grid(d):
    return [np.array([k["f_min"] + l * (k["f_max"] - k["f_min"]) / (k["n_levels"] - 1)
                      for l in range(k["n_levels"])]) for k in d["knobs"]]


@pytest.mark.parametrize("steps", [1, 3])
def test_fixed_step_rule_plant_and_limit_cycle(oracle_mod, steps):
    d = _quiet("fixed", fs_levels=steps)
    o = oracle_mod.Oracle(d)
    n_inst = 6
    out = o.simulate_baseline(range(n_inst))
    grid = _grid(d)
    N = o.n
    for i in range(n_inst):
        g = o.gen_server(i)
        a = g["a_true"]
        u, p, th, cap = out["u"][:, i], out["p"][:, i], out["theta"][:, i], out["cap"][:, i]
        lev = np.array([[int(np.argmin(np.abs(grid[j] - u[k, j]))) for j in range(N)] for k in range(len(u))])
        assert np.array_equal(u, np.array([[grid[j][lev[k, j]] for j in range(N)] for k in range(len(u))]))
        prev = np.zeros(N, dtype=int)  # every knob starts at its lowest level
        rr = 0
        for k in range(len(u)):
            err = cap[k] - p[k]
            exp = prev.copy()
            if err != 0:
                cand = [(rr + q) % N for q in range(N)]
                cand = [j for j in cand if (prev[j] < len(grid[j]) - 1 if err > 0 else prev[j] > 0)]
                if cand:
                    best = cand[0]
                    for j in cand[1:]:
                        if (th[k, j] > th[k, best]) if err > 0 else (th[k, j] < th[k, best]):
                            best = j
                    exp[best] = min(prev[best] + steps, len(grid[best]) - 1) if err > 0 else max(prev[best] - steps, 0)
                    rr = (best + 1) % N
            assert np.array_equal(lev[k], exp), (i, k)
            prev = lev[k]
        # closed-form plant: p(k+1) - p(k) = a . (u(k) - u(k-1)) (no noise, grid commands)
        du = np.diff(np.vstack([[gr[0] for gr in grid], u]), axis=0)[:-1]
        np.testing.assert_allclose(np.diff(p), du @ a, rtol=0, atol=1e-9)
        # limit cycle once the set point was crossed
        big = max(a[j] * steps * (grid[j][1] - grid[j][0]) for j in range(N))
        k0 = int(np.argmax(p >= cap))
        assert p[k0] >= cap[k0]
        assert np.all(np.abs(p[k0:] - cap[k0:]) <= big + 1e-9)


def test_safe_fixed_step_stays_below_the_cap_on_average(oracle_mod):
    d = _quiet("safe", fs_levels=1, safe_margin=30.0, periods=300)
    out = oracle_mod.Oracle(d).simulate_baseline(range(6))
    s = out["summary"]
    mean = s["sum_p"] / s["n_window"]
    assert np.all(mean < out["cap"][-1])
    assert np.all(mean > out["cap"][-1] - 30.0 - 60.0)


@pytest.mark.parametrize("kind,z", [("gpuonly", 0.5), ("gpuonly", 0.0), ("gpuonly", 0.8)])
def test_p_loop_pole_placement(oracle_mod, kind, z):
    d = _quiet(kind, p_pole=z, periods=200)
    o = oracle_mod.Oracle(d)
    out = o.simulate_baseline(range(6))
    N, S = o.n, d["controller"]["substeps"]
    steps = np.array([(k["f_max"] - k["f_min"]) / (k["n_levels"] - 1) for k in d["knobs"]])
    fmin = np.array([k["f_min"] for k in d["knobs"]]); fmax = np.array([k["f_max"] for k in d["knobs"]])
    J = np.arange(1, N)
    for i in range(6):
        a = o.gen_server(i)["a_true"]
        u, p, cap = out["u"][:, i], out["p"][:, i], out["cap"][:, i]
        assert np.all(u[:, 0] == fmax[0])  # CPU held at f_max
        assert np.all(u[:, J] == u[:, [1]])  # one common GPU frequency
        e = cap - p
        bound = np.sum(a[J] * 2 * steps[J] / S) + 1e-9
        g = u[:, 1]
        free = (g > fmin[1]) & (g < fmax[1])
        n_chk = 0
        for k in range(2, len(p) - 1):
            if free[k] and free[k - 1]:
                assert abs(e[k + 1] - z * e[k]) <= bound, (i, k, e[k + 1], z * e[k], bound)
                n_chk += 1
        assert n_chk > 100
        s = out["summary"]
        assert abs(s["sum_p"][i] / s["n_window"][i] - cap[-1]) <= bound


def test_cpu_only_range_is_too_narrow(oracle_mod):
    d = _quiet("cpuonly", periods=100)
    out = oracle_mod.Oracle(d).simulate_baseline(range(6))
    assert np.all(out["u"][20:, :, 0] == d["knobs"][0]["f_min"])
    assert np.all(out["u"][:, :, 1:] == d["knobs"][1]["f_max"])
    assert np.all(out["summary"]["n_viol"] == out["summary"]["n_window"])


def test_baselines_ignore_slo_but_misses_are_counted(oracle_mod):
    """With the §6.4 SLO schedule the GPU-only loop (one shared GPU frequency)
    misses SLOs that CapGPU's MPC meets on the same servers (Fig. 8/9)."""
    n, K = 16, 400
    gp = oracle_mod.Oracle(configs.baseline("gpuonly", n_servers=n, periods=K, slo=True))
    b = gp.simulate_baseline(range(n), traces=False)["summary"]["n_miss"]
    cg = oracle_mod.Oracle(configs.baseline("capgpu", n_servers=n, periods=K, slo=True))
    m = cg.simulate(range(n), traces=False)["summary"]["n_miss"]
    assert m.sum() == 0 and b.sum() > 0


@pytest.mark.parametrize("share,z", [(0.82, 0.5), (0.8, 0.0), (0.83, 0.7)])
def test_cpu_gpu_two_loops(oracle_mod, share, z):
    """CPU+GPU (Q39): the CPU loop tracks (1 - share) P_s on the CPU
    meter, the GPU loop share * P_s on the GPU meter, each with its own
    pole-placed gain.  The meters are recomputed here from the traced level
    indices with the grid formula and the TRUE gains (CPU meter
    0.3 C + a_0 fbar_0 without noise); each loop's error obeys
    |e(k+1) - z e(k)| <= sum_J a_j 2 step_j / S on unsaturated periods."""
    d = _quiet("cpugpu", p_pole=z, periods=200, gpu_share=share)
    o = oracle_mod.Oracle(d)
    out = o.simulate_baseline(range(6))
    N, S = o.n, d["controller"]["substeps"]
    grid = _grid(d)
    steps = np.array([(k["f_max"] - k["f_min"]) / (k["n_levels"] - 1) for k in d["knobs"]])
    fmin = np.array([k["f_min"] for k in d["knobs"]]); fmax = np.array([k["f_max"] for k in d["knobs"]])
    for i in range(6):
        g = o.gen_server(i)
        a, c0 = g["a_true"], g["c_true"]
        u, p, cap, lv = out["u"][:, i], out["p"][:, i], out["cap"][:, i], out["levels"][:, i]
        assert np.all(u[:, 1:] == u[:, [1]])  # one common GPU frequency
        # fbar(k+1) from the levels applied in period k (grid formula, not the oracle's tables)
        fb0 = np.array([np.mean(grid[0][lv[k, :, 0]]) for k in range(len(p))])
        pc = 0.3 * c0 + a[0] * fb0[:-1]          # CPU meter at instants 1..K-1
        pg = p[1:] - pc                           # GPU meter
        ec = (1 - share) * cap[1:] - pc
        eg = share * cap[1:] - pg
        bc = a[0] * 2 * steps[0] / S + 1e-9
        bg = np.sum(a[1:] * 2 * steps[1:] / S) + 1e-9
        n_c = n_g = 0
        for k in range(2, len(ec) - 1):
            if fmin[0] < u[k + 1, 0] < fmax[0] and fmin[0] < u[k, 0] < fmax[0]:
                assert abs(ec[k + 1] - z * ec[k]) <= bc, (i, k, ec[k + 1], z * ec[k])
                n_c += 1
            if fmin[1] < u[k + 1, 1] < fmax[1] and fmin[1] < u[k, 1] < fmax[1]:
                assert abs(eg[k + 1] - z * eg[k]) <= bg, (i, k, eg[k + 1], z * eg[k])
                n_g += 1
        assert n_c + n_g > 100


def test_cpu_gpu_fixed_split_misses_the_cap(oracle_mod):
    """P:282 "it is hard to find the perfect ratio": the paper's 50/50 split
    asks the CPU for more than it can draw (CPU meter 150-265 W of a ~1 kW
    cap), the CPU saturates at f_max and the server settles below the cap; a
    95 % GPU share pins the CPU at f_min and the GPU loop drives the server
    over the cap."""
    for share, cpu_pin, sign in [(0.5, "f_max", -1.0), (0.95, "f_min", 1.0)]:
        d = _quiet("cpugpu", periods=200, gpu_share=share)
        out = oracle_mod.Oracle(d).simulate_baseline(range(6))
        assert np.all(out["u"][50:, :, 0] == d["knobs"][0][cpu_pin])
        s = out["summary"]
        dev = s["sum_p"] / s["n_window"] - out["cap"][-1]
        assert np.all(sign * dev > 5.0), (share, dev)
