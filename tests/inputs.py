"""Seeded random inputs for unit-level parity tests (oracle vs CUDA).

A module of its own: holds no method arithmetic, only numpy random draws shaped
like the paper's workloads.  Both the oracle and the CUDA path
receive exactly these arrays.
"""
from __future__ import annotations

import numpy as np

from gen import configs


def bounds(desc):
    ks = desc["knobs"]
    lo = np.array([k.get("f_lo", k["f_min"]) for k in ks])
    hi = np.array([k["f_max"] for k in ks])
    m = np.array([k["f_min"] for k in ks])
    return lo, hi, m


def mpc_problem(rng, desc, active_mix=True):
    """Random S3 instance: Ahat > 0 in the synthetic gain ranges, theta-derived
    R, current frequencies inside the box, and a cap that is reachable, or on
    purpose out of reach (so that bounds become active)."""
    n = len(desc["knobs"])
    lo, hi, m = bounds(desc)
    ahat = np.where(np.arange(n) == 0, 0.03 + 0.05 * rng.random(n), 0.15 + 0.10 * rng.random(n))
    theta = np.clip(rng.random(n), desc["controller"]["theta_min"], 1.0)
    if active_mix and rng.random() < 0.3:
        theta = rng.choice([desc["controller"]["theta_min"], 1.0], size=n)
    R = desc["controller"]["r0"] / theta
    f = lo + (hi - lo) * rng.random(n)
    c_true = 250 + 100 * rng.random()
    p = c_true + ahat @ f + rng.normal(0, 11)
    pmin, pmax = c_true + ahat @ lo, c_true + ahat @ hi
    frac = rng.uniform(-0.1, 1.1) if active_mix else rng.uniform(0.2, 0.8)
    cap = pmin + frac * (pmax - pmin)
    beta = p - ahat @ f - cap
    return dict(ahat=ahat, R=R, theta=theta, beta=beta, lo=lo, hi=hi, m=m, f=f, p=p, cap=cap)


def desc_for(n_gpus, P=8, M=2, **kw):
    d = configs.get(1, n_gpus=n_gpus, P=P, M=M, **kw)
    d["knobs"] = configs.knobs(n_gpus)
    return d
