import os, sys
sys.path.insert(0, '/root/repo')
import torch
from gen import configs
from paper_conf_icpp_masw25_b200 import CapGPU, workload_from
K = 200
for cfg, ns in ((3, 296), (3, 1184), (3, 2048), (3, 8192), (2, 1024)):
    d = configs.get(cfg)
    g = CapGPU.from_config(d, n_servers=ns)
    wl = workload_from(d); bufs = g.summary_buffers()
    g.simulate(K, wl, out=bufs); torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(3): g.simulate(K, wl, out=bufs)
    b.record(); torch.cuda.synchronize()
    us = a.elapsed_time(b) / 3 * 1e3 / K
    print(f"cfg{cfg} n={ns} lp_max={os.environ.get('CAPGPU_LP_MAX_INST')}: {us:.3f} us/period = {us*1965:.0f} cycles; {ns*K/(a.elapsed_time(b)/3*1e-3)/1e9:.3f} G/s", flush=True)
    g.close()
