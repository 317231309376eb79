"""cfg 4 period-loop overhead on one GPU: `world` loopback shards of the
1,048,576-server cluster (capgpu_simulate_group) timed with CUDA events, with
and without CUDA-graph replay of the period loop (CAPGPU_NO_GRAPH), against the
k_period kernel time alone (from the same run's per-shard launch count).
usage: python tools/group_timing.py [world] [periods]"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from gen import configs  # noqa: E402
from paper_conf_icpp_masw25_b200 import capgpu as G  # noqa: E402

world = int(sys.argv[1]) if len(sys.argv) > 1 else 8
K = int(sys.argv[2]) if len(sys.argv) > 2 else 200
n_glob = 1048576 // (8 // world) if world < 8 else 1048576
per = n_glob // world
d = configs.get(4, periods=K)
wl = G.workload_from(d)
res = {}
for mode in ("graph", "stream"):
    if mode == "stream":
        os.environ["CAPGPU_NO_GRAPH"] = "1"
    else:
        os.environ.pop("CAPGPU_NO_GRAPH", None)
    ctxs = [G.CapGPU.from_config(d, n_servers=per, srv_begin=r * per, world=world, rank=r, n_servers_global=n_glob)
            for r in range(world)]
    G.simulate_group(ctxs, 20, wl, summaries=False)  # warm-up (+ setup)
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    G.simulate_group(ctxs, K, wl, summaries=False)
    b.record()
    torch.cuda.synchronize()
    res[mode] = a.elapsed_time(b) / K * 1e3  # us per period
    del ctxs
print(json.dumps({"world": world, "servers": n_glob, "periods": K, "us_per_period": res}))
