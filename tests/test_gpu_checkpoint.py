"""Checkpoint / resume and the state setter through the C ABI:
a run split by a checkpoint, restored into a fresh context, continues
bitwise identically; set_state validates before it writes."""
import numpy as np
import pytest
import torch

from gen import configs
from tests.test_gpu_parity import G, H  # noqa: F401

pytestmark = pytest.mark.gpu

KEYS = ("final_p", "sum_p", "max_p", "n_viol", "act_count")


@pytest.mark.parametrize("cfg,n", [(2, 2048), (3, 4096)])
def test_checkpoint_resume_bitwise(G, cfg, n):
    d = configs.get(cfg, n_servers=n)
    wl = G.workload_from(d)
    a = G.CapGPU.from_config(d, n_servers=n)
    a.simulate(120, wl)
    blob = a.checkpoint().cpu()  # persisted on the host
    ref = {k: H(v) for k, v in a.simulate(150, wl).items()}
    ref_st = {k: H(v) for k, v in a.sim_state().items()}
    b = G.CapGPU.from_config(d, n_servers=n)
    b.restore(blob)
    out = {k: H(v) for k, v in b.simulate(150, wl).items()}
    for k in KEYS:
        assert np.array_equal(out[k], ref[k]), k
    for k, v in b.sim_state().items():
        assert np.array_equal(H(v), ref_st[k]), k


def test_checkpoint_shape_mismatch(G):
    d = configs.get(2, n_servers=1024)
    a = G.CapGPU.from_config(d, n_servers=1024)
    a.simulate(10, G.workload_from(d))
    blob = a.checkpoint()
    b = G.CapGPU.from_config(d, n_servers=2048)
    with pytest.raises(G.CapGPUError, match="shape"):
        b.restore(blob)


def test_set_state_validates_and_roundtrips(G):
    d = configs.get(2, n_servers=1024)
    g = G.CapGPU.from_config(d, n_servers=1024)
    wl = G.workload_from(d)
    with pytest.raises(G.CapGPUError):
        g.set_state(p=torch.zeros(1024, dtype=torch.float64, device="cuda"))  # before the first simulate
    g.simulate(20, wl)
    st = g.sim_state()
    bad = st["acc"].clone()
    bad[1, 7] = 1e3  # far beyond half a grid step
    with pytest.raises(G.CapGPUError, match="acc"):
        g.set_state(acc=bad)
    nan = st["p"].clone()
    nan[3] = float("nan")
    with pytest.raises(G.CapGPUError, match="finite"):
        g.set_state(p=nan)
    assert torch.equal(g.sim_state()["acc"], st["acc"])  # nothing written
    # a second context driven to the same state continues identically
    h = G.CapGPU.from_config(d, n_servers=1024)
    h.simulate(20, wl)
    p2 = st["p"].clone()
    p2 += 1.0
    g.set_state(p=p2)
    h.set_state(p=p2)
    a = {k: H(v) for k, v in g.simulate(30, wl).items()}
    b = {k: H(v) for k, v in h.simulate(30, wl).items()}
    assert np.array_equal(a["final_p"], b["final_p"])
