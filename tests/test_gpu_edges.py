"""GPU parity at the edges of the ABI and of the method:
the largest shapes the C ABI accepts (N = 16 knobs, M = 4, P = 64), the
smallest frequency grid (two levels per knob), level grids whose spacing is
not representable in binary (the threshold tables are then inexact, level
indices must still match the oracle bit for bit), one-period calls, several
caps per server with a ragged instance count, and the smallest horizons
(P = M = 1).  Same bars as test_gpu_parity: u 1e-9 relative, p 1e-6 W,
integers exact except oracle-flagged ties."""
import numpy as np
import pytest

from gen import configs
from tests.inputs import desc_for
from tests.test_gpu_parity import G, H, _sim_compare  # noqa: F401  (fixture + helpers)

pytestmark = pytest.mark.gpu


def _bursty(d):
    d["workload"].update(demand_kind=1, cap_frac0=0.15, cap_frac_rand=0.75)
    return d


def test_abi_maxima_n16_m4_p64(G, oracle_mod):
    """15 GPUs + 1 CPU (CAPGPU_MAX_KNOBS), M = 4 (the largest control horizon),
    P = 64 (the largest prediction horizon): the last block's weight is 61 Q."""
    d = _bursty(desc_for(15, P=64, M=4, periods=60))
    _sim_compare(G, oracle_mod, d, 33, np.array([0, 16, 32]), periods=60)


def test_two_level_grids(G, oracle_mod):
    """Every knob has only its two end levels (the coarsest delta-sigma)."""
    d = _bursty(desc_for(3, P=8, M=2, periods=120))
    for k in d["knobs"]:
        k["n_levels"] = 2
        k["sweep_base"] = 0
    _sim_compare(G, oracle_mod, d, 40, np.array([0, 19, 39]), periods=120)


def test_inexact_level_spacing(G, oracle_mod):
    """Spacings 1000/6 and 1000/7 MHz are not binary fractions: the midpoints
    and levels in the host tables are rounded, the decisions still exact."""
    d = _bursty(desc_for(4, P=8, M=2, periods=150))
    d["knobs"][0].update(f_min=1000.0, f_max=2000.0, n_levels=7, sweep_base=2)
    for k in d["knobs"][1:]:
        k.update(f_min=400.0, f_max=1400.0, n_levels=8, sweep_base=0)
    _sim_compare(G, oracle_mod, d, 50, np.array([0, 25, 49]), periods=150)


def test_one_period_calls(G, oracle_mod):
    """Twelve calls of one period each: state, warm starts and the summary
    window carry across calls (here every call is its own 1-period window)."""
    d = configs.get(2, n_servers=96, periods=12)
    _sim_compare(G, oracle_mod, d, 96, np.array([0, 47, 95]), periods=12, chunks=[1] * 12)


def test_caps_per_server_ragged(G, oracle_mod):
    """cfg 5's structure (read-only server parameters shared by its caps) at a
    ragged size: 13 servers x 32 caps = 416 instances."""
    d = configs.get(5, n_servers=13, periods=200)
    tr = np.array([0, 31, 32, 200, 415])
    _sim_compare(G, oracle_mod, d, 13, tr, periods=200)


def test_shortest_horizons(G, oracle_mod):
    """P = M = 1: one block with weight Q, no prediction beyond the next period."""
    d = _bursty(desc_for(2, P=1, M=1, periods=150))
    _sim_compare(G, oracle_mod, d, 30, np.array([0, 29]), periods=150)
