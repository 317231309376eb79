"""Projected strong-scaling curve of cfgs 3 and 5 from one GPU (GPU box).

cfgs 3 and 5 shard with no data-path collective, so an N-GPU
run is N independent shards of the global problem: this times, on one GPU,
the rank-0 shard that `bench.py --gpus N` would give each rank (contiguous
1024-server shards, capgpu_shard_range) and reports the per-GPU rate and the
N x per-GPU aggregate.  usage: python tools/exp_shard_rates.py [reps]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from gen import configs  # noqa: E402
from paper_conf_icpp_masw25_b200 import CapGPU, workload_from  # noqa: E402
from paper_conf_icpp_masw25_b200 import capgpu as G  # noqa: E402

reps = int(sys.argv[1]) if len(sys.argv) > 1 else 3
for cfg in (3, 5):
    d = configs.get(cfg)
    caps = d["workload"]["n_caps"]
    n_global, K = d["n_servers"], d["periods"]
    base = None
    for world in (1, 2, 4, 8):
        begin, n_srv = G.shard_range(n_global, world, 0, 1024)
        g = CapGPU.from_config(d, n_servers=n_srv, srv_begin=begin, world=world, rank=0, n_servers_global=n_global)
        wl = workload_from(d)
        bufs = g.summary_buffers()
        g.simulate(K, wl, out=bufs)
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        for _ in range(reps):
            g.simulate(K, wl, out=bufs)
        b.record()
        torch.cuda.synchronize()
        ms = a.elapsed_time(b) / reps
        per_gpu = n_srv * caps * K / (ms * 1e-3)
        base = base or per_gpu
        print(json.dumps({"cfg": cfg, "gpus": world, "instances_per_gpu": n_srv * caps, "ms_per_step": round(ms, 3),
                          "per_gpu_steps_per_s": per_gpu, "aggregate_steps_per_s": world * per_gpu,
                          "efficiency_vs_1gpu": round(per_gpu / base, 3)}), flush=True)
        g.close()
