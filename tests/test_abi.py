"""CPU-side checks of the C-ABI boundary: the library loads, exports every
symbol include/capgpu.h declares, and its host-only helpers behave."""
import ctypes
import os
import re

import pytest

from paper_conf_icpp_masw25_b200 import build as B
from paper_conf_icpp_masw25_b200 import capgpu as G

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def L():
    B.build()
    return G.lib()


def _declared():
    src = open(os.path.join(ROOT, "include", "capgpu.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(capgpu_[a-z0-9_]+)\s*\(", src)))


def test_exports_every_declared_symbol(L):
    decl = _declared()
    assert len(decl) >= 15
    for name in decl:
        assert hasattr(L, name), name
    assert set(decl) == set(G.SYMBOLS)


def test_version_and_status_strings(L):
    assert b"sm_100a" in L.capgpu_version()
    assert L.capgpu_status_string(G.E_ORDER).startswith(b"call order")


def test_default_params(L):
    p = G.default_params()
    assert (p.q, p.r0, p.theta_min, p.lam, p.rho) == (1.0, 1e-4, 0.05, 0.95, 100.0)
    assert (p.a_lo, p.a_hi, p.substeps, p.caps_per_server) == (0.25, 4.0, 4, 1)


def test_shard_range_partition(L):
    for n, world, gran in [(1048576, 8, 1024), (65536, 3, 1024), (1000, 4, 7), (5, 8, 1)]:
        spans = [G.shard_range(n, world, r, gran) for r in range(world)]
        assert spans[0][0] == 0
        for (b0, n0), (b1, _) in zip(spans, spans[1:]):
            assert b0 + n0 == b1
        assert sum(s[1] for s in spans) == n
        for b, _ in spans:
            assert b % gran == 0


def test_create_validation_before_device_work(L):
    """Validation failures return E_INVALID before any CUDA call (works on a CPU box)."""
    kb = (G.KnobBounds * 2)()
    kb[0].f_min, kb[0].f_max, kb[0].n_levels = 1100.0, 2400.0, 14
    kb[1].f_min, kb[1].f_max, kb[1].n_levels = 1350.0, 435.0, 11  # f_min > f_max
    ctx = ctypes.c_void_p()
    rc = L.capgpu_create(ctypes.byref(ctx), 4, 1, G.Horizons(8, 2), kb, None, None)
    assert rc == G.E_INVALID and not ctx
    assert b"f_min < f_max" in L.capgpu_last_error(None)
    kb[1].f_min, kb[1].f_max = 435.0, 1350.0
    rc = L.capgpu_create(ctypes.byref(ctx), 4, 1, G.Horizons(2, 3), kb, None, None)  # M > P
    assert rc == G.E_INVALID
    rc = L.capgpu_create(ctypes.byref(ctx), 0, 1, G.Horizons(8, 2), kb, None, None)
    assert rc == G.E_INVALID
    rc = L.capgpu_create(ctypes.byref(ctx), 4, 1, G.Horizons(8, 6), kb, None, None)
    assert rc == G.E_UNSUPPORTED


def test_no_oracle_in_product():
    """The product package never imports, links or executes oracle/."""
    pkg = os.path.join(ROOT, "paper_conf_icpp_masw25_b200")
    for dp, _, fs in os.walk(pkg):
        for f in fs:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                txt = open(os.path.join(dp, f)).read()
                for pat in ("import oracle", "from oracle", "capgpu_oracle", "oracle/", "oracle.py", "ora_"):
                    assert pat not in txt, (f, pat)
