"""Multi-process host logic of the N > 1 path on CPU (gloo, world size 2):
contiguous 1024-aligned shards, the NCCL unique-id broadcast, and the
deterministic cluster aggregation (zero-padded block vector -> all-reduce ->
the library's fixed-order tree), which must be bitwise identical to one
process holding every server."""
import math
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_icpp_masw25_b200 import capgpu as G

BLOCK = 1024


def _values(n_global):
    # seeded per-server values (e.g. the w_i of an instant), indexed by global id
    rng = np.random.default_rng(1234)
    return 0.05 + 0.95 * rng.random(n_global)


def _block_sums(vals, begin, count):
    nb = (count + BLOCK - 1) // BLOCK
    out = np.zeros(nb)
    for b in range(nb):
        s = 0.0
        for x in vals[begin + b * BLOCK: begin + min((b + 1) * BLOCK, count)]:
            s += x  # fixed (ascending) order within a block
        out[b] = s
    return out


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, n_global, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    begin, count = G.shard_range(n_global, world, rank, BLOCK)
    vals = _values(n_global)
    nb_g = (n_global + BLOCK - 1) // BLOCK
    vec = torch.zeros(nb_g, dtype=torch.float64)
    vec[begin // BLOCK: begin // BLOCK + (count + BLOCK - 1) // BLOCK] = torch.from_numpy(_block_sums(vals, begin, count))
    dist.all_reduce(vec)  # one non-zero contributor per element: exact in any order
    W = G.tree_sum_host(vec.numpy())
    # NCCL unique id created on rank 0 and broadcast (what bench.py / the ABI use)
    uid = torch.zeros(128, dtype=torch.uint8)
    if rank == 0:
        uid = torch.tensor(list(G.nccl_unique_id()), dtype=torch.uint8)
    dist.broadcast(uid, 0)
    q.put((rank, begin, count, W, bytes(uid.tolist())))
    dist.destroy_process_group()


@pytest.mark.parametrize("n_global", [8192, 9 * 1024 + 300])
def test_two_rank_aggregation_bitwise(n_global):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, n_global, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = sorted(q.get(timeout=120) for _ in range(2))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    # shards: contiguous, 1024-aligned, covering everything
    assert res[0][1] == 0 and res[0][1] + res[0][2] == res[1][1] and res[1][1] + res[1][2] == n_global
    assert res[1][1] % BLOCK == 0
    # bitwise identical cluster sums on both ranks and vs one process
    vals = _values(n_global)
    W1 = G.tree_sum_host(_block_sums(vals, 0, n_global))
    assert res[0][3] == res[1][3] == W1
    assert abs(W1 - math.fsum(vals)) <= 1e-12 * W1
    assert res[0][4] == res[1][4] and len(res[0][4]) == 128


def test_tree_order():
    """The library tree = zero-padded pairwise v[i] += v[i + h]; exact on
    integers and within rounding of fsum otherwise."""
    v = np.arange(1, 1001, dtype=np.float64)
    assert G.tree_sum_host(v) == 500500.0
    rng = np.random.default_rng(7)
    x = rng.random(777) * 1e3
    n = 1
    while n < len(x):
        n *= 2
    w = np.zeros(n)
    w[:len(x)] = x
    h = n // 2
    while h >= 1:
        w[:h] = w[:h] + w[h:2 * h]
        h //= 2
    assert G.tree_sum_host(x) == w[0]
    assert abs(w[0] - math.fsum(x)) < 1e-9
