"""One fused-kernel call at a chosen instance count (GPU box; for ncu captures
of the single-warp latency chain).  usage: python tools/exp_single.py cfg n_servers periods"""
import os
import sys

os.environ.setdefault("CAPGPU_LP_MAX_INST", "0")
os.environ.setdefault("CAPGPU_NO_CHUNKING", "1")
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from gen import configs  # noqa: E402
from paper_conf_icpp_masw25_b200 import CapGPU, workload_from  # noqa: E402

cfg, n_srv, K = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3])
d = configs.get(cfg)
g = CapGPU.from_config(d, n_servers=n_srv)
wl = workload_from(d)
bufs = g.summary_buffers()
g.simulate(K, wl, out=bufs)
g.simulate(K, wl, out=bufs)
torch.cuda.synchronize()
print("ok", g.n_inst)
