"""Closed-form stability analysis of the CapGPU loop under gain mismatch
(§4.4), written out from the mathematics -- NOT from the oracle or
the CUDA path.  Used by tests/test_oracle_stability.py (pins the oracle's
closed loop) and tests/test_gpu_stability.py (property checks at scale).

Setting (gen.configs.stability_sweep): frozen model Ahat = A0 = a (noiseless
identification, ridge -> inf), all weights theta = 1 so R_j = r0_j, penalty
reference m = f_min (Q7), lower bound lo = f_min, P/M = 8/2.

Step 1 of P:221 (nominal control input).  The stacked cost (Eq. 9 with the
block structure of Q11) gives block 0 the weight c_0 = Q; with
beta = p(k) - P_s - A.fbar(k) its unconstrained minimiser is

    u_j = m_j - c_0 a_j s / R_j,   s = beta + a.u = (beta + a.m) / (1 + c_0 kappa),
    kappa = sum_j a_j^2 / R_j.

Steps 2-3 (actual plant p = C + g a.F): with x(k) = a.fbar(k) and
fbar(k+1) = u(k) + e(k+1) (delta-sigma error e, |e_j| <= step_j / S telescoping),

    x(k+1) = x* + rho (x(k) - x*) + a.e(k+1),
    rho    = -(g - 1) c_0 kappa / (1 + c_0 kappa),
    x*     = (a.m + c_0 kappa (P_s - C)) / (1 + g c_0 kappa),   p* = C + g x*.

Step 4 (pole): the loop converges iff |rho| < 1, i.e.
-1/(c_0 kappa) < g < g* = 2 + 1/(c_0 kappa).

Disturbance bounds used by the pins, with E = sum_j a_j step_j / S and
delta(k) = x(k) - x* (valid while u stays inside the box):
  |delta| <= E / (1 - |rho|) after the transient,
  |mean of delta over W periods| <= (E + 2 |rho| max|delta|) / ((1 - rho) W).
p - p* = g delta.
"""
from __future__ import annotations

import numpy as np


def knob_arrays(desc):
    ks = desc["knobs"]
    fmin = np.array([k["f_min"] for k in ks])
    fmax = np.array([k["f_max"] for k in ks])
    step = (fmax - fmin) / np.array([k["n_levels"] - 1 for k in ks])
    r0 = np.array([k.get("r0", desc["controller"]["r0"]) for k in ks])
    return fmin, fmax, step, r0


def gains(desc):
    wl = desc["workload"]
    return (1.0 + wl["gain_dlo"]) + np.arange(wl["n_caps"]) * wl["gain_step"]


def analyse(desc, a, C, cap, g):
    """Closed-form quantities for one (server, gain) instance.  a, C: the true
    (= identified) plant; cap: the set point P_s; g: the gain factor."""
    fmin, fmax, step, r0 = knob_arrays(desc)
    c0 = desc["controller"]["q"]  # block 0 weight for M = 2 (Q11)
    S = desc["controller"]["substeps"]
    kappa = float(np.sum(a * a / r0))
    ck = c0 * kappa
    rho = -(g - 1.0) * ck / (1.0 + ck)
    x_star = (a @ fmin + ck * (cap - C)) / (1.0 + g * ck)
    p_star = C + g * x_star
    s_star = (a @ fmin - x_star) / ck
    u_star = fmin - c0 * a * s_star / r0
    E = float(np.sum(a * step)) / S
    return dict(kappa=kappa, g_star=2.0 + 1.0 / ck, rho=rho, p_star=p_star, u_star=u_star,
                interior=bool(np.all(u_star > fmin) and np.all(u_star < fmax)), E=E,
                dev_bound=g * E / (1.0 - abs(rho)) if abs(rho) < 1 else np.inf,
                p_range=g * float(a @ (fmax - fmin)))


def mean_bound(info, g, W):
    """Bound on |mean(p) - p*| over a W-period window after the transient."""
    rho = info["rho"]
    dmax = info["E"] / (1.0 - abs(rho))
    return g * (info["E"] + 2.0 * abs(rho) * dmax) / ((1.0 - rho) * W)
