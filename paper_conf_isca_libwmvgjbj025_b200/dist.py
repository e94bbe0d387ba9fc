"""Multi-GPU plumbing: design points are independent, so the
ranks exchange nothing but the per-point result records -- one all-gather per sweep over NCCL (NVLink)
on B200, gloo on CPU in the tests.  One process per GPU.

A sweep is dealt to the ranks by estimated cost (``shard_points``: sorted by cost, dealt in snake order,
so every rank gets a similar amount of work and every point exactly once); each rank simulates its shard
through the C ABI; ``ShardPlan.gather`` all-gathers the fixed-size 112-B records (zero padded to the
largest shard) and scatters them back into sweep order on the device, so rank 0 ends with the records
of the whole sweep, byte for byte those of a one-GPU run (results are per point and do not depend on
which GPU or batch simulated them).  ``simulate_sharded`` is the public entry point.
"""
from __future__ import annotations

import numpy as np

from . import workloads as W


def point_cost(points: np.ndarray, n_ops: int, n_wgrad: int, wgrad_bytes: int) -> np.ndarray:
    """Rough per-point work estimate (compute tasks + flows), used only for balancing."""
    dp, tp, pp = points["dp"].astype(float), points["tp"].astype(float), points["pp"].astype(float)
    m = np.maximum(points["microbatches"].astype(float), 1.0)
    lanes = np.where(points["strategy"] == W.ST_TP, tp, np.where(points["strategy"] == W.ST_PP, pp, dp))
    lanes = np.where(points["strategy"] == W.ST_HYBRID, dp * tp * pp, lanes)
    bucket = points["bucket_bytes"].astype(float)
    ncoll = np.where(bucket > 0, np.ceil(wgrad_bytes / np.maximum(bucket, 1.0)), float(n_wgrad))
    coll = ncoll * 2.0 * np.maximum(lanes - 1.0, 0.0) * lanes
    piped = (points["strategy"] == W.ST_PP) | (points["strategy"] == W.ST_HYBRID)
    return np.where(piped, m * n_ops * np.maximum(lanes / np.maximum(pp, 1.0), 1.0), lanes * n_ops + coll)


def sweep_cost(sw: W.Sweep) -> np.ndarray:
    tr = sw.trace
    wg = tr.tensors[tr.tensors["category"] == W.CAT_WGRAD]
    return point_cost(sw.points, len(tr.ops), len(wg), int(wg["bytes_b0"].sum()))


def shard_points(costs: np.ndarray, world: int, rank: int) -> np.ndarray:
    """Indices of the points rank `rank` simulates: sort by cost descending and deal in snake
    order (0..w-1, w-1..0, ...), then keep the original order within the shard."""
    order = np.argsort(-costs, kind="stable")
    r = np.arange(len(order)) % (2 * world)
    owner = np.where(r < world, r, 2 * world - 1 - r)
    return np.sort(order[owner == rank])


def shard_sizes(n: int, world: int, costs: np.ndarray) -> list:
    return [len(shard_points(costs, world, r)) for r in range(world)]


class ShardPlan:
    """Who simulates which point, and the device-side index map that restores sweep order."""

    def __init__(self, costs: np.ndarray, world: int, rank: int):
        self.n = len(costs)
        self.world, self.rank = world, rank
        self.shards = [shard_points(costs, world, r) for r in range(world)]
        self.mine = self.shards[rank]
        self.max_count = max(1, max(len(s) for s in self.shards))
        self._dst = None

    def sub_sweep(self, sw: W.Sweep) -> W.Sweep:
        return W.Sweep(sw.name, sw.trace, sw.topos, sw.points[self.mine], sw.plans)

    def gather(self, local, out=None):
        """All-gather this rank's records (uint8 tensor, len(mine) x 112 B) and scatter every rank's
        records into sweep order: returns (or fills) an n x 112 uint8 tensor on local's device, the same
        on every rank.  NCCL: one all_gather_into_tensor; gloo: all_gather over a list."""
        import torch
        import torch.distributed as dist
        rec = W.RESULT_DTYPE.itemsize
        dev = local.device
        if self._dst is None or self._dst.device != dev:
            src, dst = [], []
            for r, s in enumerate(self.shards):
                src.append(r * self.max_count + np.arange(len(s)))
                dst.append(s)
            self._src = torch.from_numpy(np.concatenate(src).astype(np.int64)).to(dev)
            self._dst = torch.from_numpy(np.concatenate(dst).astype(np.int64)).to(dev)
            self._buf = torch.zeros(self.max_count * rec, dtype=torch.uint8, device=dev)
            self._all = torch.empty(self.world * self.max_count * rec, dtype=torch.uint8, device=dev)
        self._buf[: local.numel()].copy_(local)
        if self.world > 1:
            if dist.get_backend() == "nccl":
                dist.all_gather_into_tensor(self._all, self._buf)
            else:   # gloo (CPU tests; test-only GPU sharing): through host memory
                hb, ha = self._buf.cpu(), self._all.cpu()
                dist.all_gather(list(ha.chunk(self.world)), hb)
                self._all.copy_(ha)
        else:
            self._all.copy_(self._buf)
        if out is None:
            out = torch.empty(self.n * rec, dtype=torch.uint8, device=dev)
        out.view(self.n, rec).index_copy_(0, self._dst, self._all.view(-1, rec).index_select(0, self._src))
        return out


def simulate_sharded(ctx, sw: W.Sweep, plan: ShardPlan, device="cuda", sub: W.Sweep = None, host_on_rank0=False):
    """Public multi-GPU call: this rank simulates its shard of `sw` through the C ABI (load_trace,
    build_sweep, simulate_batch, results into device memory), all on torch's current stream, then the
    records of the whole sweep are all-gathered and put in sweep order.  Returns the sweep's RESULT_DTYPE
    records (numpy; with host_on_rank0 only rank 0 copies them to the host, the others return None).  `sub` may pass this rank's shard prepared in advance (e.g. in pinned
    host memory)."""
    import torch
    rec = W.RESULT_DTYPE.itemsize
    stream = torch.cuda.current_stream().cuda_stream if device != "cpu" else 0
    sub = sub if sub is not None else plan.sub_sweep(sw)
    tid = ctx.triosim_load_trace(sub.trace)
    sid = ctx.triosim_build_sweep(tid, sub.topos, sub.points, sub.plans or None)
    n = len(sub.points)
    local = torch.zeros(max(n, 1) * rec, dtype=torch.uint8, device=device)
    if n:
        ctx.triosim_simulate_batch(sid, 0, n, stream)
        ctx.triosim_results(sid, 0, n, device_ptr=local.data_ptr(), stream=stream)
    out = plan.gather(local[: n * rec])
    host = None if (host_on_rank0 and plan.rank != 0) else out.cpu().numpy().view(W.RESULT_DTYPE)
    ctx.triosim_release(sid)
    ctx.triosim_release(tid)
    return host
