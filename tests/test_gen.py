"""The seeded input generator (gen/capgpu_gen.h) through the oracle's exports:
splitmix64 known-answer vector, distributions and ranges of the recipe in
DESIGN.md §3.  (The device copy is checked bit-for-bit in test_gpu_parity.py.)"""
import numpy as np

from gen import configs


def test_splitmix64_known_answer(oracle_mod):
    # splitmix64 with state 0: first output = mix(0x9E3779B97F4A7C15)
    L = oracle_mod.lib()
    assert L.ora_gen_mix64(0x9E3779B97F4A7C15) == 0xE220A8397B1DCDAF
    # second output of the same sequence
    assert L.ora_gen_mix64((2 * 0x9E3779B97F4A7C15) % 2**64) == 0x6E789E6AA1B965F4


def test_param_ranges(oracle_mod):
    o = oracle_mod.oracle_for(3)
    a, c, tm, b, am = [], [], [], [], []
    for s in range(2000):
        g = o.gen_server(s)
        a.append(g["a_true"]); c.append(g["c_true"]); tm.append(g["thr_max"])
        b.append(g["base"]); am.append(g["amp"])
    a, c, tm, b, am = map(np.array, (a, c, tm, b, am))
    assert a[:, 0].min() >= 0.03 and a[:, 0].max() < 0.08
    assert a[:, 1:].min() >= 0.15 and a[:, 1:].max() < 0.25
    assert c.min() >= 250 and c.max() < 350
    assert tm[:, 0].min() >= 50 and tm[:, 1:].min() >= 40 and tm[:, 1:].max() < 200
    assert b.min() >= 0.2 and b.max() < 0.9 and am.min() >= 0.2 and am.max() < 0.6
    # uniformity: means near the middle of the ranges
    assert abs(a[:, 1:].mean() - 0.20) < 0.003 and abs(c.mean() - 300) < 2.0


def test_noise_moments(oracle_mod):
    o = oracle_mod.oracle_for(2)
    x = np.array([o.gen_noise(s, k) for s in range(50) for k in range(400)])
    assert abs(x.mean()) < 0.3
    assert abs(x.std() - 11.0) < 0.3
    assert np.abs(x).max() <= 2 * 11.0 * np.sqrt(3.0) + 1e-9  # Irwin-Hall-4 support


def test_demand_and_caps(oracle_mod):
    o = oracle_mod.oracle_for(2)
    d = configs.get(2)
    burst_frac = []
    for s in range(40):
        g = o.gen_server(s)
        for k in range(0, 300, 7):
            dem = o.gen_demand(s, k)
            assert np.all(dem >= 0) and np.all(dem <= 1.5 * g["thr_max"] + 1e-9)
            burst_frac.append(np.mean(dem / g["thr_max"] > g["base"] + 0.06))
        cb = o.gen_cap_base(s)
        lo = np.array([k["f_min"] for k in d["knobs"]]); hi = np.array([k["f_max"] for k in d["knobs"]])
        pmin = g["c_true"] + g["a_true"] @ lo; pmax = g["c_true"] + g["a_true"] @ hi
        assert abs(cb - (pmin + 0.45 * (pmax - pmin))) <= 1e-9 * cb
    assert 0.1 < np.mean(burst_frac) < 0.3  # bursts on ~20 % of the 10-period windows


def test_sweep_rows_design(oracle_mod):
    """one knob varies over all its levels, others at base."""
    o = oracle_mod.oracle_for(3)
    F, p = o.sweep_rows(0, noisy=False)
    d = configs.get(3)
    r = 0
    for j, k in enumerate(d["knobs"]):
        lv, _, _ = o.levels(j)
        for l in range(k["n_levels"]):
            for jj, kk in enumerate(d["knobs"]):
                lvj, _, _ = o.levels(jj)
                want = lv[l] if jj == j else lvj[kk["sweep_base"]]
                assert F[r, jj] == want
            r += 1
    assert r == F.shape[0] == 14 + 8 * 11
