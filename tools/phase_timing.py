"""Per-phase cycle breakdown of the fused kernel (profiling build
libcapgpu_timing.so, -DCAPGPU_PHASE_TIMING).  Prints the share of each phase
of the period loop, averaged over instances.

    python -m paper_conf_icpp_masw25_b200.build --variant=timing
    CAPGPU_LIB_VARIANT=timing python tools/phase_timing.py [cfg] [periods] [n_servers]
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
os.environ.setdefault("CAPGPU_LIB_VARIANT", "timing")

import torch  # noqa: E402

from gen import configs  # noqa: E402
from paper_conf_icpp_masw25_b200 import capgpu as G  # noqa: E402

NAMES = {1: "S1 Welford push", 2: "S1 LDL^T solve + clamp", 3: "S2 weights (+trace)", 0: "S1-S3 total (caller)",
         4: "S4 demand generation (+trace rows)", 5: "S4 delta-sigma plant", 6: "S4 noise + power",
         7: "loop: summaries, trace checks"}

cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 3
periods = int(sys.argv[2]) if len(sys.argv) > 2 else 200
n_srv = int(sys.argv[3]) if len(sys.argv) > 3 else None  # e.g. 4736 = one warp per SM (latency chain alone)
d = configs.get(cfg)
g = G.CapGPU.from_config(d, n_servers=n_srv)
wl = G.workload_from(d)
g.simulate(periods, wl)  # init + warm
cnt = torch.zeros(8, g.n_inst, dtype=torch.int64, device="cuda")
G._check(G.lib().capgpu_debug_phase_counters(g._ctx, G._ptr(cnt)))
g.simulate(periods, wl)
torch.cuda.synchronize()
m = cnt.double().mean(dim=1).cpu().tolist()
s3 = m[0] - m[1] - m[2] - m[3]
tot = m[0] + m[4] + m[5] + m[6] + m[7]
print(f"cfg {cfg}: cycles per instance-period (sum over phases {tot / periods:.0f})")
for k in (1, 2, 3):
    print(f"  {NAMES[k]:40s} {m[k] / periods:8.0f}  {m[k] / tot * 100:5.1f} %")
print(f"  {'S3 block QPs (= total - S1 - S2)':40s} {s3 / periods:8.0f}  {s3 / tot * 100:5.1f} %")
for k in (4, 5, 6, 7):
    print(f"  {NAMES[k]:40s} {m[k] / periods:8.0f}  {m[k] / tot * 100:5.1f} %")
