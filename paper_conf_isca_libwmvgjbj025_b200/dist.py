"""Multi-GPU plumbing: design points are independent, so ranks only
exchange the per-point result records -- one all-gather per sweep over NCCL (NVLink) on B200,
gloo on CPU in the tests.

* weak scaling (bench default): every rank simulates its own full sweep; the gathered buffer is
  the rank-major concatenation of the records.
* strong scaling (``shard_points``): one sweep is dealt to the ranks by estimated cost
  (snake / LPT order) so every rank gets a similar amount of work; ``unshard`` restores the
  sweep order from the gathered records.
"""
from __future__ import annotations

import numpy as np

from . import workloads as W


def point_cost(points: np.ndarray, n_ops: int, n_wgrad: int, wgrad_bytes: int) -> np.ndarray:
    """Rough per-point work estimate (compute tasks + flows), used only for balancing."""
    dp, tp, pp = points["dp"].astype(float), points["tp"].astype(float), points["pp"].astype(float)
    m = np.maximum(points["microbatches"].astype(float), 1.0)
    lanes = np.where(points["strategy"] == W.ST_TP, tp, np.where(points["strategy"] == W.ST_PP, pp, dp))
    bucket = points["bucket_bytes"].astype(float)
    ncoll = np.where(bucket > 0, np.ceil(wgrad_bytes / np.maximum(bucket, 1.0)), float(n_wgrad))
    coll = ncoll * 2.0 * np.maximum(lanes - 1.0, 0.0) * lanes
    return np.where(points["strategy"] == W.ST_PP, m * n_ops, lanes * n_ops + coll)


def shard_points(costs: np.ndarray, world: int, rank: int) -> np.ndarray:
    """Indices of the points rank `rank` simulates: sort by cost descending and deal in snake
    order (0..w-1, w-1..0, ...), then keep the original order within the shard."""
    order = np.argsort(-costs, kind="stable")
    r = np.arange(len(order)) % (2 * world)
    owner = np.where(r < world, r, 2 * world - 1 - r)
    return np.sort(order[owner == rank])


def shard_sizes(n: int, world: int, costs: np.ndarray) -> list:
    return [len(shard_points(costs, world, r)) for r in range(world)]


def gather_records(local: "torch.Tensor", world: int, max_count: int) -> "torch.Tensor":
    """All-gather fixed-size result records (uint8 tensors of max_count records, zero padded)."""
    import torch
    import torch.distributed as dist
    rec = W.RESULT_DTYPE.itemsize
    buf = torch.zeros(max_count * rec, dtype=torch.uint8, device=local.device)
    buf[: local.numel()] = local
    out = torch.empty(world * max_count * rec, dtype=torch.uint8, device=local.device)
    if dist.get_backend() == "nccl":
        dist.all_gather_into_tensor(out, buf)
    else:
        dist.all_gather(list(out.chunk(world)), buf)
    return out


def unshard(gathered: np.ndarray, costs: np.ndarray, world: int, max_count: int) -> np.ndarray:
    """Sweep-ordered RESULT_DTYPE records from the rank-major gathered buffer."""
    recs = gathered.view(W.RESULT_DTYPE).reshape(world, max_count)
    out = np.zeros(len(costs), W.RESULT_DTYPE)
    for r in range(world):
        idx = shard_points(costs, world, r)
        out[idx] = recs[r, : len(idx)]
    return out
