"""World-size-2/3 gloo tests of bench.py's multi-GPU path (its sweep, cost-balanced sharding, record
all-gather, scatter into sweep order) on CPU -- the GPU box has one device, so the NCCL path is covered
by construction and by a shared-GPU gloo run of bench.py itself (tools/)."""
import os
import socket

import ctypes
import zlib
import sys

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as tmp

from paper_conf_isca_libwmvgjbj025_b200 import dist as D, workloads as W

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


class FakeCtx:
    """Stands in for triosim.Context on CPU: a record is a pure function of the point (as on the GPU, where
    results are per point and independent of the batch or device that simulated them)."""

    def triosim_load_trace(self, tr):
        return 1

    def triosim_build_sweep(self, tid, topos, points, plans=None):
        self.pts = np.array(points, copy=True)
        return 2

    def triosim_simulate_batch(self, sid, first, count, stream=0):
        pass

    def triosim_results(self, sid, first, count, device_ptr=None, stream=0):
        p = self.pts[first:first + count]
        r = np.zeros(count, W.RESULT_DTYPE)
        r["iter_time_s"] = p["bw_scale"] * p["dp"] + p["lat_scale"]
        r["n_compute"] = p["global_batch"]
        r["order_hash"] = [zlib.crc32(x.tobytes()) for x in p]
        ctypes.memmove(device_ptr, r.ctypes.data, r.nbytes)

    def triosim_release(self, h):
        pass


def _worker(rank, world, port, q, scale):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    sw = bench.make_sweep("c2", scale)        # bench's own weak-scaling sweep at this world size
    plan = D.ShardPlan(D.sweep_cost(sw), world, rank)
    got = D.simulate_sharded(FakeCtx(), sw, plan, device="cpu", host_on_rank0=True)
    if rank == 0:
        q.put((got.tobytes(), [float(D.sweep_cost(sw)[s].sum()) for s in plan.shards], [len(s) for s in plan.shards]))
    else:
        assert got is None
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_bench_shard_gather_unshard_matches_one_rank(world):
    """bench.py's N-rank path (its sweep at N x 10k distinct points, cost-balanced snake shards, one
    all-gather, scatter into sweep order, rank-0 D2H) gives byte for byte the records of one rank
    simulating the same sweep, with every point exactly once."""
    ctx = tmp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q, world)) for r in range(world)]
    for p in procs:
        p.start()
    got, loads, sizes = q.get(timeout=300)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    sw = bench.make_sweep("c2", world)
    assert len(sw.points) == 10000 * world
    one = D.simulate_sharded(FakeCtx(), sw, D.ShardPlan(D.sweep_cost(sw), 1, 0), device="cpu")
    assert got == one.tobytes()
    assert max(loads) / min(loads) < 1.01 and max(sizes) - min(sizes) <= 1
    # distinct points: the refined sweep has no duplicates and contains configs[1] at scale 1's size
    key = sw.points[["topo", "global_batch", "bucket_bytes", "bw_scale", "lat_scale"]]
    assert len(np.unique(key)) == len(key)


def test_bench_scale_one_is_configs1():
    assert bench.make_sweep("c2", 1).points.tobytes() == W.sweep_c2().points.tobytes()


def test_shard_partition_properties():
    rng = np.random.Generator(np.random.PCG64(1))
    costs = rng.lognormal(0, 2, 1001)
    for world in (1, 2, 3, 8):
        parts = [D.shard_points(costs, world, r) for r in range(world)]
        allidx = np.concatenate(parts)
        assert sorted(allidx.tolist()) == list(range(1001))
        assert max(len(p) for p in parts) - min(len(p) for p in parts) <= 1
