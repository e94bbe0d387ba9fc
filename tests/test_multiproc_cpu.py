"""World-size-2 gloo test of the multi-GPU host logic (sharding, record gather, un-sharding)
on CPU -- the GPU box has one device, so the NCCL path is covered by construction."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as tmp

from paper_conf_isca_libwmvgjbj025_b200 import dist as D, workloads as W


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _fake_records(idx):
    r = np.zeros(len(idx), W.RESULT_DTYPE)
    r["iter_time_s"] = np.asarray(idx, float) * 0.5
    r["order_hash"] = np.asarray(idx, np.uint64) * 2654435761
    r["status"] = 0
    return r


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    sw = W.sweep_c2()
    tr = sw.trace
    wg = tr.tensors[tr.tensors["category"] == W.CAT_WGRAD]
    costs = D.point_cost(sw.points, len(tr.ops), len(wg), int(wg["bytes_b0"].sum()))
    mine = D.shard_points(costs, world, rank)
    maxc = max(D.shard_sizes(len(costs), world, costs))
    local = torch.from_numpy(_fake_records(mine).view(np.uint8).copy())
    g = D.gather_records(local, world, maxc)
    if rank == 0:
        res = D.unshard(g.numpy(), costs, world, maxc)
        q.put((res["iter_time_s"].tolist(), res["order_hash"].tolist(),
               [float(costs[D.shard_points(costs, world, r)].sum()) for r in range(world)]))
    # weak scaling: rank-major concatenation of full sweeps
    full = torch.from_numpy(_fake_records(np.arange(16) + 100 * rank).view(np.uint8).copy())
    g2 = D.gather_records(full, world, 16)
    if rank == 0:
        q.put(g2.numpy().view(W.RESULT_DTYPE)["iter_time_s"].tolist())
    dist.barrier()
    dist.destroy_process_group()


def test_shard_gather_unshard_world2():
    ctx = tmp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    it, h, loads = q.get(timeout=120)
    weak = q.get(timeout=120)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    n = len(it)
    assert it == [0.5 * i for i in range(n)]            # every point exactly once, in sweep order
    assert h == [i * 2654435761 for i in range(n)]
    assert max(loads) / min(loads) < 1.05                # cost-balanced shards
    assert weak == [0.5 * (i + 100 * r) for r in range(2) for i in range(16)]


def test_shard_partition_properties():
    rng = np.random.Generator(np.random.PCG64(1))
    costs = rng.lognormal(0, 2, 1001)
    for world in (1, 2, 3, 8):
        parts = [D.shard_points(costs, world, r) for r in range(world)]
        allidx = np.concatenate(parts)
        assert sorted(allidx.tolist()) == list(range(1001))
        assert max(len(p) for p in parts) - min(len(p) for p in parts) <= 1
