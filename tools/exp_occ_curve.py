"""Per-period time of the fused kernel vs resident warps per SM (GPU box).

cfg 3 (N = 9) and cfg 5 (N = 4) shapes with 148 x 32 x w instances for
w = 1, 2, 4, 8, (16): one warp per SM, then more.  CAPGPU_LP_MAX_INST=0 and
CAPGPU_NO_CHUNKING=1 keep every run on the plain thread-per-instance kernel.
usage: python tools/exp_occ_curve.py [periods]"""
import os
import sys

os.environ.setdefault("CAPGPU_LP_MAX_INST", "0")
os.environ.setdefault("CAPGPU_NO_CHUNKING", "1")
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from gen import configs  # noqa: E402
from paper_conf_icpp_masw25_b200 import CapGPU, workload_from  # noqa: E402

K = int(sys.argv[1]) if len(sys.argv) > 1 else 200
for cfg, ws in ((3, (1, 2, 4, 6, 8)), (5, (1, 2, 4, 8, 12, 16))):
    d = configs.get(cfg)
    caps = d["workload"]["n_caps"]
    for w in ws:
        n_inst = 148 * 32 * w
        g = CapGPU.from_config(d, n_servers=max(1, n_inst // caps))
        wl = workload_from(d)
        bufs = g.summary_buffers()
        g.simulate(K, wl, out=bufs)
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        for _ in range(3):
            g.simulate(K, wl, out=bufs)
        b.record()
        torch.cuda.synchronize()
        ms = a.elapsed_time(b) / 3
        us_per = ms * 1e3 / K
        cyc = us_per * 1965
        print(f"cfg{cfg} warps/SM {w:2d} inst {g.n_inst:7d}: {us_per:7.3f} us/period = {cyc:8.0f} cycles/period; "
              f"{g.n_inst * K / ms / 1e6:.3f} G steps/s", flush=True)
        g.close()
