"""The five BASELINE.json workloads as plain data.

No method arithmetic lives here: only bounds, horizons, controller constants and
the workload recipe (cap schedule, demand kind, seeds).  Both the oracle wrapper
(oracle/oracle.py) and the product binding read these dictionaries.

Citations: P:NNN = /root/reference/PAPER.md line.
"""
from __future__ import annotations

import copy

# Knob classes (Q15): CPU 1.1-2.4 GHz in 100 MHz steps, V100-class
# GPU 435-1350 MHz (nvidia-smi -ac 877,435-1350) on 11 levels (91.5 MHz).
CPU_KNOB = dict(f_min=1100.0, f_max=2400.0, n_levels=14, sweep_base=3)  # base 1400 MHz
GPU_KNOB = dict(f_min=435.0, f_max=1350.0, n_levels=11, sweep_base=0)   # base = lowest level

# Controller constants (Q1, Q4, Q6, Q8, Q21; P = 8 / M = 2 from P:264; gamma P:190)
CONTROLLER = dict(q=1.0, r0=1e-4, theta_min=0.05, lam=0.95, rho=100.0, a_lo=0.25, a_hi=4.0,
                  a_floor=1e-3, gamma=0.91, noise_std=11.0, substeps=4, wmove=0.0,
                  ref_alpha=0.0)

_BASE_WORKLOAD = dict(n_caps=1, demand_kind=1, demand_frac=0.7, cap_frac0=0.5, cap_frac_rand=0.0,
                      cap_frac_step=0.0, cap_period=0, cap_lo=0, cap_hi=0, cap_mult=1.0,
                      hierarchical=False, gain_dlo=0.0, gain_step=0.0,
                      slo_period=0, slo_lo=0, slo_hi=0, slo_a=None, slo_b=None,
                      controller=0, fs_levels=1, safe_margin=0.0, p_pole=0.5, gpu_share=0.5)

# NEXT-2 baseline controllers (§6.1): workload["controller"]
CONTROLLERS = {"capgpu": 0, "fixed": 1, "safe": 2, "gpuonly": 3, "cpuonly": 4, "cpugpu": 5}

# NEXT-1 (§6.4): latency SLOs as ratios SLO_j / e_min,j for the three
# tail levels the paper switches between ("30 %", "50 %", "80 % tail").  The
# paper's percentiles come from measured latency distributions; these ratios
# are the synthetic stand-ins (Q29): a higher tail = a looser SLO.
SLO_TAIL = {30: 1.15, 50: 1.35, 80: 1.6}

CONFIGS = {
    # 1 server, 1 CPU + 2 GPUs, P/M = 4/2, 200 periods, fixed cap
    1: dict(n_servers=1, n_gpus=2, P=4, M=2, periods=200, seed=1,
            workload=dict(demand_kind=0, demand_frac=0.7, cap_frac0=0.6)),
    # 1,024 servers, 1 CPU + 4 GPUs, 8/2, 1000 periods, step changes in cap
    # (800 -> 900 -> 800 W analogue of Fig. 10: x 900/800 in [40, 80) mod 200)
    2: dict(n_servers=1024, n_gpus=4, P=8, M=2, periods=1000, seed=2,
            workload=dict(cap_frac0=0.45, cap_period=200, cap_lo=40, cap_hi=80, cap_mult=1.125)),
    # 65,536 servers, 1 CPU + 8 GPUs (9 knobs), 8/3, 1000 periods, throughput-driven weights
    3: dict(n_servers=65536, n_gpus=8, P=8, M=3, periods=1000, seed=3,
            workload=dict(cap_frac0=0.3, cap_frac_rand=0.5)),
    # 1,048,576 servers sharded over 8 GPUs, hierarchical rack budget (Q16)
    4: dict(n_servers=1048576, n_gpus=8, P=8, M=2, periods=1000, seed=4,
            workload=dict(hierarchical=True, rack=16, block=1024, cluster_frac=0.55,
                          rack_frac=0.9)),
    # cap sweep: 262,144 servers x 32 caps x 2,000 periods (Fig. 6 analogue)
    5: dict(n_servers=262144, n_gpus=3, P=8, M=2, periods=2000, seed=5,
            workload=dict(n_caps=32, cap_frac0=0.0, cap_frac_step=1.0 / 32.0)),
}


def stability_sweep(n_servers: int = 64, n_gains: int = 24, g_lo: float = 0.2, g_hi: float = 6.0,
                    periods: int = 1000, r0: float = 0.1) -> dict:
    """NEXT-4: batched gain-mismatch sweep of §4.4.  The paper's
    1 CPU + 3 GPU server, frozen model (ridge -> inf, so Ahat = A0), noiseless
    plant and identification (A0 = a exactly), all weights 1 (theta_min = 1,
    R = r0), constant demand; cap column c runs the plant with true gains g_c a,
    g_c = g_lo + c (g_hi - g_lo)/(n_gains - 1), set point at the middle of the
    true plant's range (feasible).  The closed form (tests/stability.py)
    says the loop converges iff g < 2 + 1/(c_0 kappa), kappa = sum_j A0_j^2 / r0;
    r0 = 0.1 puts c_0 kappa near 1 so the bound differs visibly from 2.  The
    default grid avoids g = 2 exactly: there the nominal model's reachable
    maximum a.(f_max - f_min) + beta sits exactly on the set point, a floating
    tie of the CAP_INFEASIBLE flag (Q28)."""
    d = get(5, n_servers=n_servers, periods=periods, noise_std=0.0, rho=1e30, theta_min=1.0,
            a_lo=0.0, a_hi=1e30, r0=r0, P=8, M=2)
    step = (g_hi - g_lo) / (n_gains - 1)
    d["workload"].update(n_caps=n_gains, demand_kind=0, demand_frac=0.7, cap_frac0=0.5, cap_frac_rand=0.0,
                         cap_frac_step=0.0, gain_dlo=g_lo - 1.0, gain_step=step)
    d["cfg"] = "stability"
    return d


def slo_schedule(n_servers: int = 64, periods: int = 1000, slo_period: int = 200, slo_lo: int = 14,
                 slo_hi: int = 114) -> dict:
    """NEXT-1: time-varying SLOs (§6.4) on the paper's 1 CPU + 3 GPU
    server (P/M = 8/2).  Phase A: every GPU task at the 50 %-tail SLO;
    phase B (k mod slo_period in [slo_lo, slo_hi), the paper switches at period
    14): GPU 0 tightened to the 30 % tail, GPUs 1-2 relaxed to the 80 % tail.
    The CPU task has no SLO.  Set points P_min + (0.55 + 0.4 U) dP per
    server: most servers can meet every SLO, some cannot reach their cap with
    the raised bounds (CAP_INFEASIBLE).  Bursty demand."""
    d = get(5, n_servers=n_servers, periods=periods)
    d["workload"].update(n_caps=1, cap_frac0=0.55, cap_frac_rand=0.4, cap_frac_step=0.0,
                         slo_period=slo_period, slo_lo=slo_lo, slo_hi=slo_hi,
                         slo_a=[0.0] + [SLO_TAIL[50]] * 3,
                         slo_b=[0.0, SLO_TAIL[30], SLO_TAIL[80], SLO_TAIL[80]])
    d["cfg"] = "slo"
    return d


def baseline(controller: str, n_servers: int = 1024, periods: int = 1000, fs_levels: int = 1,
             safe_margin: float = 25.0, p_pole: float = 0.5, slo: bool = False, gpu_share: float = 0.5) -> dict:
    """NEXT-2: a comparison controller (§6.1) on the cfg 2 plant and
    set-point schedule (1 CPU + 4 GPUs, P_min + 0.45 dP, x 900/800 in [40, 80)
    mod 200: the Fig. 10 step).  "fixed" / "safe" = Fixed-step /
    Safe Fixed-step (step `fs_levels` grid levels; safe set point
    P_s - safe_margin), "gpuonly" / "cpuonly" = pole-placed P loops
    (pole p_pole), "cpugpu" = CPU+GPU, two such loops on separately
    metered CPU and GPU power with the budget split gpu_share : 1 - gpu_share
    (50/50 and 60/40; Q39), "capgpu" = the MPC on the same workload.
    slo=True adds the §6.4 SLO schedule (the baselines ignore it; misses count)."""
    d = get(2, n_servers=n_servers, periods=periods)
    d["workload"].update(controller=CONTROLLERS[controller], fs_levels=fs_levels, safe_margin=safe_margin,
                         p_pole=p_pole, gpu_share=gpu_share)
    if slo:
        d["workload"].update(slo_period=200, slo_lo=14, slo_hi=114, slo_a=[0.0] + [SLO_TAIL[50]] * 4,
                             slo_b=[0.0, SLO_TAIL[30], SLO_TAIL[80], SLO_TAIL[80], SLO_TAIL[80]])
    d["cfg"] = "baseline-" + controller
    return d


def move_suppression(n_servers: int = 64, periods: int = 1000, wmove: float = 2e-4, n_gpus: int = 3,
                     P: int = 8, M: int = 2) -> dict:
    """NEXT-3: the horizon-active MPC (Q36) on the paper's 1 CPU + 3 GPU
    server (P/M = 8/2): Eq. 9 plus wmove |d(k+t|k)|^2 per control step,
    set points P_min + (0.3 + 0.5 U) dP, bursty demand.  wmove = 2e-4 W^2/MHz^2
    is twice the base frequency penalty r0 (Q6)."""
    d = get(5, n_servers=n_servers, periods=periods, wmove=wmove, n_gpus=n_gpus, P=P, M=M)
    d["knobs"] = knobs(n_gpus)
    d["workload"].update(n_caps=1, cap_frac0=0.3, cap_frac_rand=0.5, cap_frac_step=0.0)
    d["cfg"] = "move"
    return d


def by_name(name) -> dict:
    """bench.py --config: "1".."5" (BASELINE.json configs), "stab" (the NEXT-4
    gain sweep at bench size: 16,384 servers x 24 gains x 1,000 periods) or
    "slo" (the NEXT-1 SLO schedule: 1,048,576 servers x 1,000 periods), or a
    NEXT-2 baseline "fixed" / "safe" / "gpuonly" / "cpuonly" / "cpugpu" (1,048,576 servers
    of the cfg 2 plant x 1,000 periods)."""
    if str(name) == "stab":
        return stability_sweep(n_servers=16384)
    if str(name) == "slo":
        return slo_schedule(n_servers=1048576)
    if str(name) == "move":
        return move_suppression(n_servers=1048576)
    if str(name) in CONTROLLERS and str(name) != "capgpu":
        return baseline(str(name), n_servers=1048576)
    return get(int(name))


def knobs(n_gpus: int) -> list[dict]:
    """Knob list: knob 0 = CPU, knobs 1..n_gpus = GPUs (paper order)."""
    return [dict(CPU_KNOB)] + [dict(GPU_KNOB) for _ in range(n_gpus)]


def get(cfg: int, **overrides) -> dict:
    """Full description of config `cfg` (1..5) with optional overrides."""
    c = copy.deepcopy(CONFIGS[cfg])
    wl = dict(_BASE_WORKLOAD)
    wl.update(c.pop("workload"))
    c["workload"] = wl
    c["controller"] = dict(CONTROLLER)
    c["cfg"] = cfg
    for k, v in overrides.items():
        if k in c["controller"]:
            c["controller"][k] = v
        elif k in wl:
            wl[k] = v
        else:
            c[k] = v
    c["knobs"] = knobs(c["n_gpus"])
    return c
